import torch, numpy as np, sys, ctypes
sys.path.insert(0, '.')
import synth
from paper_conf_conext_dhakalrwcr22_b200 import ss
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline
pipe = OrbPipeline(752, 480, 1000, 8, max_frames=4)
fr = torch.from_numpy(synth.make_frames(752, 480, 4)).cuda()
for name, st in [("default", None), ("current", torch.cuda.current_stream()), ("new", torch.cuda.Stream())]:
    try:
        pipe.extract(fr, stream=st); torch.cuda.synchronize(); print(name, "ok", flush=True)
    except Exception as e:
        print(name, "FAIL", e, flush=True)
s = torch.cuda.Stream()
print("stream handle", hex(s.cuda_stream))
rt = ctypes.CDLL("libcudart.so.12")
fl = ctypes.c_uint()
print("torch-rt cudaStreamGetFlags", rt.cudaStreamGetFlags(ctypes.c_void_p(s.cuda_stream), ctypes.byref(fl)))
import os
print(open('/proc/self/maps').read().count('libcudart'), [l.split()[-1] for l in open('/proc/self/maps') if 'libcudart' in l][:3])
