"""Per-warp phase timeline of the decoder (diagnostic; needs a -DSZX_TIMELINE=1 build).

    bash scripts/build_variants.sh "-DSZX_TIMELINE=1"
    SZX_LIB=$PWD/build_exp/lib__DSZX_TIMELINE_1.so FIELD=0 python scripts/timeline.py

Runs compress + decompress of the NYX-shaped field a few times, then reads the
last decode's %globaltimer stamps (per warp: entry, index ready, fill done,
all done) and prints phase times in microseconds from the earliest entry.
"""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
from paper_conf_hpdc_yudztt0c22_b200 import szx as api
import synth

field = int(os.environ.get("FIELD", "0"))
fillw = int(os.environ.get("FILLW", "2"))
cfg = os.environ.get("CFG", "nyx")  # nyx | cesm | hurricane
if cfg == "cesm":
    x = synth.cesm_like(0, device="cuda").reshape(-1).contiguous()
elif cfg == "hurricane":
    x = synth.hurricane_like(0, device="cuda").reshape(-1).contiguous()
else:
    x = synth.nyx_like(field, n=512, device="cuda").reshape(-1).contiguous()
c = szx.Codec(x.numel(), torch.float32, 128)
y = torch.empty_like(x)
c.compress_async(x, 1e-3, "rel")
h = c.header()
for _ in range(5):
    c.compress_async(x, 1e-3, "rel")
    c.decompress_async(c.out, h, y)
torch.cuda.synchronize()

L = api.lib()
f = L.szx_debug_timeline
f.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
n = 2048 * 8 * 4
buf = np.zeros(n, dtype=np.uint64)
assert f(buf.ctypes.data, n) == 0
tl = buf.reshape(2048, 8, 4).astype(np.int64)
ctas = int((tl[:, 0, 0] != 0).sum())
tl = tl[:ctas]
t0 = tl[:, :, 0].min()
us = (tl - t0) / 1000.0
fill = us[:, :fillw, :]
dec = us[:, fillw:, :]


def q(a):
    a = np.sort(a.reshape(-1))
    return {"min": round(float(a[0]), 1), "p50": round(float(a[len(a) // 2]), 1),
            "p90": round(float(a[int(len(a) * 0.9)]), 1), "max": round(float(a[-1]), 1)}


print(json.dumps({
    "cfg": cfg, "field": field, "ctas": ctas,
    "entry": q(us[:, :, 0]),
    # warp 0 only: its stamp follows the barrier's polling loop; the other
    # warps' stamp may be scheduled before the barrier's second bar.sync
    "index_ready_warp0": q(us[:, 0, 1]),
    "fill_warps_fill_done": q(fill[:, :, 2]),
    "fill_warps_done": q(fill[:, :, 3]),
    "decode_warps_done": q(dec[:, :, 3]),
    "kernel_span_us": round(float(us[:, :, 3].max()), 1),
}))
fi = L.szx_debug_timeline_index
fi.argtypes = [ctypes.c_void_p, ctypes.c_uint64]
bi = np.zeros(2048 * 8, dtype=np.uint64)
assert fi(bi.ctypes.data, bi.size) == 0
tall = bi.reshape(2048, 8).astype(np.int64)
ti = tall[tall[:, 0] != 0]
if ti.size:
    ui = (ti - t0) / 1000.0
    print(json.dumps({"index_ctas": int(ti.shape[0]), "local_counts_done": q(ui[:, 0]), "prefix1_done": q(ui[:, 1]),
                      "zsize_sums_done": q(ui[:, 2]), "prefix2_done": q(ui[:, 3]), "per_tile_pass_done": q(ui[:, 4])}))
tb = tall[:ctas, 5]
tb = tb[tb != 0]
if tb.size:
    print(json.dumps({"barrier_passed_all_ctas": q((tb - t0) / 1000.0)}))
if os.environ.get("DETAIL"):
    # index-ready time of warp 0 by CTA range (index CTAs first)
    for a in range(0, ctas, 37):
        print(a, [round(float(v), 1) for v in us[a:a + 37, 0, 1]])

