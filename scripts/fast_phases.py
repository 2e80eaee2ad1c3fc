"""Per-CTA phase timeline of fast_bands_kernel (instrumented build: SS_NVCC_EXTRA=-DSS_FAST_PHASES).
Prints, per launch (level 0 / levels >= 1), the CTA count, launch span, and the median / max
of each phase: stage, score, nms, output."""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["SS_NVCC_EXTRA"] = os.environ.get("SS_NVCC_EXTRA", "") + " -DSS_FAST_PHASES"
from paper_conf_conext_dhakalrwcr22_b200 import build as b  # noqa: E402

b.build(force=True)
import torch  # noqa: E402

import synth  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200 import ss  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline  # noqa: E402

shape = sys.argv[1] if len(sys.argv) > 1 else "euroc"
B = int(sys.argv[2]) if len(sys.argv) > 2 else 4
w, h = synth.SHAPES[shape]
pipe = OrbPipeline(w, h, 1000, 8, max_frames=B)
fr = torch.from_numpy(synth.make_frames(w, h, B, cfg=2)).cuda()
for _ in range(5):
    pipe.extract(fr)
torch.cuda.synchronize()
buf = np.zeros((2, 4096, 8), np.uint64)
assert ss.lib().ss_dbg_fast_ts(buf.ctypes.data_as(ctypes.c_void_p)) == 0
for li, name in enumerate(["level 0", "levels >= 1"]):
    t = buf[li].astype(np.int64)
    t = t[t[:, 0] > 0]  # the launch's CTAs of this group (indices follow the launch's band order)
    n = len(t)
    t0 = t[:, 0].min()
    ph = np.diff(t[:, 0:5], axis=1)
    print(f"{name}: {n} CTAs, span {(t[:, 4].max() - t0) / 1000:.2f} us, last start {(t[:, 0].max() - t0) / 1000:.2f} us, "
          f"SMs used {len(set(t[:, 5].tolist()))}")
    for j, pn in enumerate(["stage", "score", "nms", "output"]):
        print(f"   {pn:7s} median {np.median(ph[:, j]) / 1000:.2f} us  max {ph[:, j].max() / 1000:.2f} us")
    cta = (t[:, 4] - t[:, 0]) / 1000
    print(f"   CTA total median {np.median(cta):.2f} max {cta.max():.2f} us")
    per_sm = np.bincount(t[:, 5].astype(np.int64))
    print(f"   CTAs per SM: max {per_sm.max()} mean {per_sm[per_sm > 0].mean():.2f}")
