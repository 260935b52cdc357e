"""Small compress + decompress workload for compute-sanitizer (memcheck / racecheck / synccheck /
initcheck): every kernel of the library on small inputs, float32 and float64, block sizes
32..256, REL and ABS, special values, a tail block, a forced R2 escalation, the sharded
entry points and a block-range decode.  Exits non-zero on any parity failure against the oracle."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import oracle
import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth

ok = True
cases = []
for dt in (torch.float32, torch.float64):
    cases.append(("special", synth.special_values(20_011, 3, dtype=dt), 1e-2, "rel"))
    cases.append(("mix", synth.random_mix(30_007, 4, dtype=dt), 1e-3, "abs"))
    cases.append(("nyx", synth.nyx_like(1, n=24).reshape(-1).to(dt), 1e-3, "rel"))
for tag, x, eb, mode in cases:
    for b in (32, 64, 128, 256):
        xd = x.cuda()
        s = szx.compress(xd, eb, mode, b)
        ref = oracle.compress(x.numpy(), eb, oracle.REL if mode == "rel" else oracle.ABS, b)
        if s.cpu().numpy().tobytes() != ref.tobytes():
            print("stream mismatch", tag, x.dtype, b)
            ok = False
        y = szx.decompress(s)
        ui = np.uint32 if x.dtype == torch.float32 else np.uint64
        if not np.array_equal(y.cpu().numpy().view(ui), oracle.decompress(ref).view(ui)):
            print("reconstruction mismatch", tag, x.dtype, b)
            ok = False
        yb = szx.decompress_blocks(s, 3, 17)
        q = szx.decompress_quality(s, xd)
# forced escalation (r_bias test hook) on the float32 b = 128 path
szx.set_r_bias(-3)
xs = synth.offset_field(50_000, 7, 3e3)
s = szx.compress(xs.cuda(), 1e-4, "rel", 128)
oracle_s = oracle.compress(xs.numpy(), 1e-4, oracle.REL, 128, r_bias=-3)
szx.set_r_bias(0)
if s.cpu().numpy().tobytes() != oracle_s.tobytes():
    print("escalation mismatch")
    ok = False
# sharded entry points
from paper_conf_hpdc_yudztt0c22_b200 import dist as sdist
x = synth.nyx_like(0, n=32).reshape(-1).cuda()
mm = szx.local_minmax(x)
e = (1e-3 * (mm[1] - mm[0])).reshape(1).contiguous()
s = szx.compress_shard(x, 1e-3, e, "rel", 128)
# the dense float32 decoder loop (thread-serial tiles; >= ~58 M values): mixed tile shapes,
# a raw block and an all-constant tile, decoded once (SANITIZE_TS=0 skips it)
if os.environ.get("SANITIZE_TS", "1") == "1":
    xt = synth.nyx_like(1, n=400).reshape(-1).numpy().copy()[:-77]
    nW = xt.size // 4096
    blk = xt[: nW * 4096].reshape(nW, 32, 128)
    blk[3::7, :6, :] = 1.5e6
    blk[5::11, :20, :] = -2.0e6
    blk[8::17, :, :] = 0.25
    blk[1::13, 5, 17] = np.nan
    s = szx.compress(torch.from_numpy(xt).cuda(), 1e-3, "rel", 128)
    ref = oracle.compress(xt, 1e-3, oracle.REL, 128)
    if s.cpu().numpy().tobytes() != ref.tobytes():
        print("stream mismatch (dense)")
        ok = False
    y = szx.decompress(s)
    if not np.array_equal(y.cpu().numpy().view(np.uint32), oracle.decompress(ref).view(np.uint32)):
        print("reconstruction mismatch (dense)")
        ok = False
torch.cuda.synchronize()
print("sanitize driver:", "ok" if ok else "MISMATCH")
sys.exit(0 if ok else 1)
