import ctypes, os, sys
sys.path.insert(0, '/root/repo')
import numpy as np, torch
import paper_conf_hpdc_yudztt0c22_b200 as szx
from paper_conf_hpdc_yudztt0c22_b200 import szx as api
import synth
for field in (1, 2, 0):
    x = synth.nyx_like(field, n=512, device="cuda").reshape(-1).contiguous()
    c = szx.Codec(x.numel(), torch.float32, 128)
    f = api.lib().szx_debug_guardstat; f.argtypes = [ctypes.c_void_p]
    b0 = np.zeros(2, dtype=np.uint64); f(b0.ctypes.data)
    c.compress_async(x, 1e-3, "rel"); torch.cuda.synchronize()
    b1 = np.zeros(2, dtype=np.uint64); f(b1.ctypes.data)
    d = b1 - b0
    h = c.header()
    print(field, "guarded blocks", int(d[0]), "of", h.n_nonconst, f"({d[0]/max(1,h.n_nonconst):.4f})", "warp-tiles", int(d[1]))
