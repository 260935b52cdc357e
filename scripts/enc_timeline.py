"""Per-tile timeline of the fused encoder (diagnostic; needs a -DSZX_ETIMELINE=1 build):
publish -> prefix written by the scanner -> retire start -> copy-out done.
    SZX_LIB=$PWD/build_exp/lib__DSZX_ETIMELINE_1.so FIELD=1 python scripts/enc_timeline.py"""
import ctypes
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
from paper_conf_hpdc_yudztt0c22_b200 import szx as api
import synth

field = int(os.environ.get("FIELD", "1"))
x = synth.nyx_like(field, n=512, device="cuda").reshape(-1).contiguous()
c = szx.Codec(x.numel(), torch.float32, 128)
for _ in range(4):
    c.compress_async(x, 1e-3, "rel")
torch.cuda.synchronize()
h = c.header()
ntiles = (int(h.n_nonconst) + 15) // 16
L = api.lib()
f = L.szx_debug_enc_timeline
f.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
buf = np.zeros(ntiles * 4, dtype=np.uint64)
assert f(buf.ctypes.data, buf.size) == 0
tl = buf.reshape(ntiles, 4).astype(np.int64)
t0 = tl[:, 0].min()
us = (tl - t0) / 1000.0


def q(a):
    a = np.sort(a.reshape(-1))
    return {"p10": round(float(a[len(a) // 10]), 2), "p50": round(float(a[len(a) // 2]), 2),
            "p90": round(float(a[int(len(a) * 0.9)]), 2), "max": round(float(a[-1]), 2)}


print("tiles", ntiles, "span us", round(float(us[:, 3].max()), 1))
print("publish -> prefix (scanner lag)", q(us[:, 1] - us[:, 0]))
print("retire start - prefix (>0: no wait)", q(us[:, 2] - us[:, 1]))
print("retire wait", q(np.maximum(0, us[:, 1] - us[:, 2])), "sum over tiles us", round(float(np.maximum(0, us[:, 1] - us[:, 2]).sum()), 1))
print("copy-out", q(us[:, 3] - np.maximum(us[:, 1], us[:, 2])))
# frontier: at time T, how many tiles published in order vs prefixed
for T in np.linspace(0, us[:, 3].max(), 11)[1:]:
    pub = us[:, 0] <= T
    inorder = int(np.argmin(pub)) if not pub.all() else ntiles
    print(f"t={T:7.1f} published {int(pub.sum()):6d} in-order {inorder:6d} prefixed {int((us[:, 1] <= T).sum()):6d} retired {int((us[:, 3] <= T).sum()):6d}")
