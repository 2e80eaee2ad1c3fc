"""Small extract + window match for compute-sanitizer runs (memcheck / racecheck / synccheck).

usage: compute-sanitizer --tool racecheck python scripts/sanitize_extract.py
"""
import os
import sys

import numpy as np
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import synth  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200 import ss  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline, match_out, to_device_records  # noqa: E402


def main():
    w, h, B = 320, 240, 2
    frames = synth.make_frames(w, h, B, cfg=7)
    noise = np.random.default_rng(1).integers(0, 256, size=(h, w), dtype=np.uint8)
    frames[1] = noise  # the overflow / fallback paths too
    pipe = OrbPipeline(w, h, 300, 4, max_frames=B, max_queries=512)
    pipe.extract(torch.from_numpy(frames).cuda())
    kps, desc, counts = pipe.results(B)
    q = np.zeros(512, ss.QUERY_DTYPE)
    rng = np.random.default_rng(2)
    q["frame"] = rng.integers(0, B, 512)
    q["u"], q["v"] = rng.uniform(0, w, 512), rng.uniform(0, h, 512)
    q["pred_level"] = rng.integers(0, 4, 512)
    q["radius"] = 12.0
    qd = rng.integers(0, 256, (512, 32), dtype=np.uint8)
    out = match_out(512, "cuda")
    pipe.match_window(B, to_device_records(q, "cuda"), torch.from_numpy(qd).cuda(), out)
    torch.cuda.synchronize()
    print("sanitize run ok", int(counts[:, -1].sum()), "keypoints")


if __name__ == "__main__":
    main()
