"""Small driver for ncu: NYX-shaped 512^3 f32 REL 1e-3, a few compress+decompress steps."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth

field = int(os.environ.get("FIELD", "0"))
n = int(os.environ.get("EDGE", "512"))
steps = int(os.environ.get("STEPS", "3"))
x = synth.nyx_like(field, n=n, device="cuda").reshape(-1).contiguous()
c = szx.Codec(x.numel(), torch.float32, 128)
y = torch.empty_like(x)
c.compress_async(x, 1e-3, "rel")
h = c.header()
for _ in range(steps):
    c.compress_async(x, 1e-3, "rel")
    c.decompress_async(c.out, h, y)
torch.cuda.synchronize()
print("ok", c.stream_bytes(), int(c.d_status.item()))
