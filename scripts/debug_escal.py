"""Compare GPU vs oracle streams section by section for an R2-escalation case (debug aid)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth

for rb, n, off, eb in ((-3, 50_000, 3e3, 1e-4), (-6, 300_000, None, 1e-3), (-3, 300_000, None, 1e-3), (-2, 50_000, 3e3, 1e-4)):
    xs = synth.offset_field(n, 7, off) if off else synth.random_mix(n, 77)
    szx.set_r_bias(rb)
    g = szx.compress(xs.cuda(), eb, "rel", 128).cpu().numpy()
    szx.set_r_bias(0)
    r, tr = oracle.compress(xs.numpy(), eb, oracle.REL, 128, trace=True, r_bias=rb)
    nB = (n + 127) // 128
    al = lambda v: (v + 15) // 16 * 16
    h = oracle.read_header(r)
    off_mu = 64 + al((nB + 7) // 8)
    off_zs = off_mu + al(4 * nB)
    off_pl = off_zs + al(2 * h["nnc"])
    same = g.size == r.size and np.array_equal(g, r)
    print(f"rb={rb} n={n} off={off}: sizes {g.size} {r.size} identical={same} escal={int(tr.escal.sum())} "
          f"raw={int((tr.R == 32).sum())}")
    if not same:
        m = min(g.size, r.size)
        d = np.flatnonzero(g[:m] != r[:m])
        i = int(d[0]) if d.size else m
        sec = "header" if i < 64 else "bitmap" if i < off_mu else "mu" if i < off_zs else "zsize" if i < off_pl else "payload"
        print("  first diff at", i, sec, "ndiff", d.size)
        if sec == "mu":
            k = (i - off_mu) // 4
            print("  block", k, "gpu mu", g[off_mu + 4 * k: off_mu + 4 * k + 4].view(np.float32), "oracle", r[off_mu + 4 * k: off_mu + 4 * k + 4].view(np.float32), "R", tr.R[k], "escal", tr.escal[k])
        if sec == "zsize":
            j = (i - off_zs) // 2
            ncidx = np.flatnonzero(tr.type)
            k = ncidx[j]
            print("  nc", j, "block", k, "gpu z", g[off_zs + 2 * j: off_zs + 2 * j + 2].view(np.uint16), "oracle z", tr.z[k], "R", tr.R[k], "escal", tr.escal[k])

# detail of the first failing case: per nonconstant block z and R on both sides
xs = synth.offset_field(50_000, 7, 3e3)
szx.set_r_bias(-3)
g = szx.compress(xs.cuda(), 1e-4, "rel", 128).cpu().numpy()
szx.set_r_bias(0)
r, tr = oracle.compress(xs.numpy(), 1e-4, oracle.REL, 128, trace=True, r_bias=-3)
n = xs.numel(); nB = (n + 127) // 128
al = lambda v: (v + 15) // 16 * 16
off_mu = 64 + al((nB + 7) // 8); off_zs = off_mu + al(4 * nB)
hg = oracle.read_header(r)
nnc = hg["nnc"]
zg = g[off_zs:off_zs + 2 * nnc].view(np.uint16).astype(int)
zr = r[off_zs:off_zs + 2 * nnc].view(np.uint16).astype(int)
ncidx = np.flatnonzero(tr.type)
bad = np.flatnonzero(zg != zr)
print("nnc", nnc, "blocks with different z:", bad.size, bad[:20])
pl_g = off_zs + al(2 * nnc); pg = np.concatenate([[0], np.cumsum(zg)]); pr = np.concatenate([[0], np.cumsum(zr)])
for j in bad[:12]:
    k = ncidx[j]
    print(f"  nc {j} block {k} tile {j//16} slot {j%16}: z gpu {zg[j]} oracle {zr[j]}  R gpu {g[pl_g + pg[j]]} oracle {tr.R[k]} escal {tr.escal[k]}")
