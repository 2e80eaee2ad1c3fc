"""Phase timeline of lastframe_kernel per frame CTA (instrumented build: -DSS_LF_PHASES), from the
last O13 launch of a short bench run: entry -> PDL wait -> P0 -> P1 (+ per-warp P1 ends) -> P2
-> P3 -> exit.  Usage: python scripts/lf_phases.py [config]"""
import os
import subprocess
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
os.environ["SS_NVCC_EXTRA"] = os.environ.get("SS_NVCC_EXTRA", "") + " -DSS_LF_PHASES"
from paper_conf_conext_dhakalrwcr22_b200 import build as b  # noqa: E402

b.build(force=True)
r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--steps", "5", "--warmup", "3", "--no-cpu-baseline",
                    "--config", sys.argv[1] if len(sys.argv) > 1 else "c2", "--dump-lf-ts", "/tmp/lf_ts.npy"],
                   capture_output=True, text=True, env=os.environ)
if r.returncode != 0:
    print(r.stderr[-3000:])
buf = np.load("/tmp/lf_ts.npy").astype(np.int64)
t = buf[:64 * 8].reshape(64, 8)
w = buf[64 * 8:64 * 8 + 64 * 32].reshape(64, 32)
w2 = buf[64 * 8 + 64 * 32:].reshape(64, 32, 2)
n = int((t[:, 0] > 0).sum())
for i in range(n):
    d = (t[i, 1:6] - t[i, 0]) / 1000
    we = (w[i][w[i] > 0] - t[i, 2]) / 1000  # warp P1 ends after the P0 barrier
    print(f"CTA {i}: wait {d[0]:.2f}  P0 {d[1] - d[0]:.2f}  P1 {d[2] - d[1]:.2f} (warp ends: median {np.median(we):.2f} "
          f"min {we.min():.2f} max {we.max():.2f})  P2+P3 {d[3] - d[2]:.2f}  tail {d[4] - d[3]:.2f}  total {d[4]:.2f} us")
    ok = (w2[i, :, 0] > 0) & (w2[i, :, 1] > 0)
    proj = (w2[i, ok, 0] - t[i, 2]) / 1000
    scan = (w2[i, ok, 1] - w2[i, ok, 0]) / 1000
    print(f"   first point per warp: projection done at {np.median(proj):.2f} (max {proj.max():.2f}) us, "
          f"window scan {np.median(scan):.2f} (max {scan.max():.2f}) us over {int(ok.sum())} warps")
