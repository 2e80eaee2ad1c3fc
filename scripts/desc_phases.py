"""Per-warp phase timeline of describe_kernel (instrumented build: -DSS_DESC_PHASES): entry,
after the PDL wait, after the level-offset barrier, patch staged, moments + vertical blur
done, descriptor written, end.  Usage: python scripts/desc_phases.py [shape] [frames]"""
import ctypes
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["SS_NVCC_EXTRA"] = os.environ.get("SS_NVCC_EXTRA", "") + " -DSS_DESC_PHASES"
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
buf = np.zeros((16384, 8), np.uint64)
assert ss.lib().ss_dbg_desc_ts(buf.ctypes.data_as(ctypes.c_void_p)) == 0
t = buf.astype(np.int64)
ok = (t[:, 6] > 0) & (t[:, 0] > 0)
t = t[ok]
t0 = t[:, 0].min()
print(f"{len(t)} keypoint warps, span {(t[:, 6].max() - t0) / 1000:.2f} us, last entry {(t[:, 0].max() - t0) / 1000:.2f} us")
names = ["pdl wait", "offsets", "patch", "moments+V", "brief", "tail"]
d = np.diff(t[:, :7], axis=1) / 1000
for j, n in enumerate(names):
    print(f"  {n:10s} median {np.median(d[:, j]):.2f}  p90 {np.percentile(d[:, j], 90):.2f}  max {d[:, j].max():.2f} us")
tot = (t[:, 6] - t[:, 0]) / 1000
print(f"  warp total median {np.median(tot):.2f} max {tot.max():.2f} us")
path = t[:, 7] & 0xFF
lev = (t[:, 7] >> 8) & 0xFF
for pv, pn in [(0, "bytes"), (1, "tma"), (2, "chunks"), (3, "border")]:
    m = path == pv
    if m.any():
        print(f"  path {pn:7s}: {int(m.sum())} warps, patch median {np.median(d[m, 2]):.2f} max {d[m, 2].max():.2f} us, "
              f"levels {sorted(set(lev[m].tolist()))}")
post = (t[:, 6] - t[:, 1]) / 1000
slow = np.argsort(post)[-8:]
print("  slowest (post-wait us, path, level, phases):", [(round(post[k], 1), int(path[k]), int(lev[k]), [round(x, 1) for x in d[k, 1:]]) for k in slow])
