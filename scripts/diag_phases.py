"""Print the distribution kernel's phase timeline (ns since its start) per (frame 0, level)."""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import synth  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200 import ss  # noqa: E402
from paper_conf_conext_dhakalrwcr22_b200.pipeline import OrbPipeline  # noqa: E402

w, h = synth.SHAPES[sys.argv[1] if len(sys.argv) > 1 else "euroc"]
pipe = OrbPipeline(w, h, 1000, 8, max_frames=4)
fr = torch.from_numpy(synth.make_frames(w, h, 4, cfg=2)).cuda()
for _ in range(5):
    pipe.extract(fr)
torch.cuda.synchronize()
names = ["start", "n", "gather", "zeroed", "keys+hist", "rules", "partial", "best", "kept", "written", "entry", "setup"]
for l in range(8):
    t = ss.ss_debug_phase_times(pipe.ctx, 0, l, 12)
    rel = [(names[i], int(t[i] - t[0])) for i in range(len(t)) if t[i] >= t[0] or i >= 10]
    n = len(ss.ss_debug_candidates(pipe.ctx, 0, l)[0])
    print(f"level {l} n={n}", rel)
