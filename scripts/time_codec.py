"""Kernel times of compress + decompress (library CUDA events per launch) on one NYX-shaped
512^3 float32 field (FIELD 0 density, 1 velocity, 2 temperature; EDGE, STEPS env)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth

cfg = os.environ.get("CFG", "nyx")  # nyx | miranda | qmcpack | cesm | hurricane
field = int(os.environ.get("FIELD", "1"))
eb = 1e-3
if cfg == "miranda":
    x, eb = synth.miranda_like(device="cuda").reshape(-1).contiguous(), 1e-4
elif cfg == "qmcpack":
    x, eb = synth.qmcpack_like(device="cuda").reshape(-1).contiguous(), 1e-4
elif cfg == "cesm":
    x = synth.cesm_like(field, device="cuda").reshape(-1).contiguous()
elif cfg == "hacc":
    x = synth.hacc_like(field, device="cuda").reshape(-1).contiguous()
elif cfg == "hurricane":
    x = synth.hurricane_like(field, device="cuda").reshape(-1).contiguous()
else:
    x = synth.nyx_like(field, n=int(os.environ.get("EDGE", "512")), device="cuda").reshape(-1).contiguous()
c = szx.Codec(x.numel(), x.dtype, 128)
y = torch.empty_like(x)
c.compress_async(x, eb, "rel")
h = c.header()
for _ in range(3):
    c.compress_async(x, eb, "rel")
    c.decompress_async(c.out, h, y)
torch.cuda.synchronize()
szx.timing_enable(True)
szx.timing_reset()
for _ in range(int(os.environ.get("STEPS", "30"))):
    c.compress_async(x, eb, "rel")
    c.decompress_async(c.out, h, y)
torch.cuda.synchronize()
t = szx.timing_read()
ok = int(c.d_status.item()) == 0
# bound check (the parity tests compare bytes with the oracle)
err = (x.double() - y.double()).abs().max().item()
print(os.environ.get("SZX_LIB", "default").split("/")[-1], f"{cfg} field {field}",
      {k: round(v[0] / v[1] * 1000, 1) for k, v in t.items()}, "status ok" if ok else "STATUS ERR",
      f"maxerr {err:.6g} <= eb {h.eb_abs:.6g}: {err <= h.eb_abs}")
