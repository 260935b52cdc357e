"""Kernel times of compress_async alone (no header read-back): for timing experiments whose
streams are not valid (SZX_EXP_* builds).  FIELD / EDGE / STEPS env as prof_nyx.py."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth

field = int(os.environ.get("FIELD", "1"))
x = synth.nyx_like(field, n=int(os.environ.get("EDGE", "512")), device="cuda").reshape(-1).contiguous()
c = szx.Codec(x.numel(), torch.float32, 128)
for _ in range(5):
    c.compress_async(x, 1e-3, "rel")
torch.cuda.synchronize()
szx.timing_enable(True)
szx.timing_reset()
for _ in range(int(os.environ.get("STEPS", "30"))):
    c.compress_async(x, 1e-3, "rel")
torch.cuda.synchronize()
t = szx.timing_read()
print(os.environ.get("SZX_LIB", "default").split("/")[-1], {k: round(v[0] / v[1] * 1000, 1) for k, v in t.items()})
