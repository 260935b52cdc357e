import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_hpdc_yudztt0c22_b200 as szx
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
from fig10_decoder import decode as fdec
x = synth.special_values(123_457, 9).numpy().astype(np.float64)
ref, tr = oracle.compress(x, 1e-2, oracle.REL, 128, trace=True)
got = szx.compress(torch.from_numpy(x).cuda(), 1e-2, "rel", 128).cpu().numpy()
_, ir = fdec(ref.tobytes())
try:
    _, ig = fdec(got.tobytes())
except AssertionError as e:
    print("gpu stream fails the Fig.10 decoder:", e); ig = None
nB = len(ir)
if ig:
    for k in range(nB):
        if ir[k] != ig[k]:
            blk = x[128*k:128*k+128]
            print("block", k, "oracle", ir[k], "gpu", ig[k], "escal", tr.escal[k])
            print("   ", blk[:8], "min/max", np.nanmin(blk), np.nanmax(blk), "nan", np.isnan(blk).sum(), "inf", np.isinf(blk).sum())
            break
d = np.nonzero(got[:min(got.size, ref.size)] != ref[:min(got.size, ref.size)])[0]
print("sizes", got.size, ref.size, "ndiff", d.size, "first", d[:5])
h = oracle.read_header(ref)
W = 8; nB = (x.size + 127)//128
al = lambda v: (v+15)//16*16
off_mu = 64 + al((nB+7)//8); off_zs = off_mu + al(W*nB); off_pl = off_zs + al(2*h["nnc"])
print("sections", off_mu, off_zs, off_pl)
if d.size:
    i = d[0]
    print("ref", ref[i-8:i+8], "\ngot", got[i-8:i+8])
    # which block payload?
    zs = ref[off_zs:off_zs+2*h["nnc"]].view(np.uint16).astype(np.int64)
    ends = off_pl + np.cumsum(zs)
    j = np.searchsorted(ends, i, side="right")
    print("payload block (nc index)", j, "z", zs[j], "start", ends[j]-zs[j], "offset in block", i-(ends[j]-zs[j]))
    yk = fdec(got.tobytes())[0]; yr = oracle.decompress(ref)
    dd = np.nonzero(yk.view(np.uint64) != yr.view(np.uint64))[0]
    print("decoded diffs", dd.size, dd[:5], yk[dd[:3]], yr[dd[:3]], x[dd[:3]])
