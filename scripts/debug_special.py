import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import oracle, synth
import paper_conf_hpdc_yudztt0c22_b200 as szx
x = synth.special_values(123_457, 9).numpy()
ref, tr = oracle.compress(x, 1e-2, oracle.REL, 128, trace=True)
got = szx.compress(torch.from_numpy(x).cuda(), 1e-2, "rel", 128).cpu().numpy()
nB = (x.size + 127) // 128
bm_r = np.unpackbits(ref[64:64 + (nB + 7) // 8], bitorder="little")[:nB]
bm_g = np.unpackbits(got[64:64 + (nB + 7) // 8], bitorder="little")[:nB]
d = np.nonzero(bm_r != bm_g)[0]
print("differing blocks:", d.size, d[:10])
for k in d[:3]:
    blk = x[128 * k:128 * k + 128]
    print(k, "oracle", bm_r[k], "gpu", bm_g[k], "R", tr.R[k])
    print("  finite min/max", np.nanmin(blk[np.isfinite(blk)]), np.nanmax(blk[np.isfinite(blk)]),
          "nan", np.isnan(blk).sum(), "inf", np.isinf(blk).sum())
    print("  specials:", blk[~np.isfinite(blk) | (np.abs(blk) > 1e20) | ((blk != 0) & (np.abs(blk) < 1e-30))])
