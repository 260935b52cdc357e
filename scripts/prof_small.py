"""Small driver for ncu on a small config (CESM-ATM-shaped T-like field, REL 1e-3, b = 128)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth

cfg = os.environ.get("CFG", "cesm")
x = (synth.cesm_like(0, device="cuda") if cfg == "cesm" else synth.hurricane_like(0, device="cuda")).reshape(-1).contiguous()
c = szx.Codec(x.numel(), torch.float32, 128)
y = torch.empty_like(x)
c.compress_async(x, 1e-3, "rel")
h = c.header()
for _ in range(3):
    c.compress_async(x, 1e-3, "rel")
    c.decompress_async(c.out, h, y)
torch.cuda.synchronize()
print("ok", c.stream_bytes())
