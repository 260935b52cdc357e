"""GPU parity of the thread-serial tile decoder (lane-per-block Fig. 10,
P:L2321-2336), the path dense float32 b = 128 streams of >= ~58 M values take
(`DPlan::ts`, szx_api.cu).  The input mixes every tile shape that path meets:
all-nonconstant tiles, tiles with 24-31 nonconstant blocks (thread-serial +
constant fill), tiles with fewer (segment decoder inside the dense loop),
all-constant tiles,
raw blocks (a NaN forces R = 32, reading R14/R15) among thread-serial tiles,
and a partial last block.  Stream bytes and reconstruction bits are compared
with the oracle, the decoder is also run on the oracle's own bytes, and
corrupted lead codes inside a dense tile must be rejected."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_hpdc_yudztt0c22_b200 as szx  # noqa: E402

B, TB = 128, 32


def _mixed_dense(seed_field: int = 1, n_edge: int = 400, tail: int = 77) -> np.ndarray:
    x = synth.nyx_like(seed_field, n=n_edge).reshape(-1).numpy().copy()
    x = x[: x.size - tail]
    nW = x.size // (B * TB)
    blk = x[: nW * TB * B].reshape(nW, TB, B)
    t = np.arange(nW)
    blk[t % 7 == 3, :6, :] = 1.5e6           # 26 nonconstant blocks: thread-serial + constant fill
    blk[t % 11 == 5, :20, :] = -2.0e6        # 12 nonconstant blocks: segment decoder
    blk[t % 17 == 8, :, :] = 0.25            # all-constant tiles (skipped by the dense loop, filled after)
    sel = np.nonzero(t % 13 == 1)[0]
    blk[sel, 5, 17] = np.nan                 # a raw block in an otherwise dense tile
    blk[sel[::3], 9, :] = np.inf             # an all-Inf block (raw: Inf radius, R14)
    return x


def test_thread_serial_tiles_match_oracle():
    x = _mixed_dense()
    assert x.size >= 4 * 444 * 8 * TB * B  # >= 4 tiles per warp of B200's decode grid: the dense loop
    ref = oracle.compress(x, 1e-3, oracle.REL, B)
    xd = torch.from_numpy(x).cuda()
    s = szx.compress(xd, 1e-3, "rel", B)
    got = s.cpu().numpy()
    assert got.tobytes() == ref.tobytes()
    h = szx.read_header(got[:64].tobytes())
    assert 4 * h.n_nonconst >= 3 * ((x.size + B - 1) // B)  # dense: the thread-serial loop runs
    yr = oracle.decompress(ref)
    y = szx.decompress(s).cpu().numpy()
    assert np.array_equal(y.view(np.uint32), yr.view(np.uint32))
    y2 = szx.decompress(torch.from_numpy(ref).cuda()).cpu().numpy()  # the oracle's own bytes
    assert np.array_equal(y2.view(np.uint32), yr.view(np.uint32))
    fin = np.isfinite(x)
    e = oracle.eb_abs(x, 1e-3, oracle.REL)
    assert np.abs(x[fin].astype(np.float64) - y[fin].astype(np.float64)).max() <= e
    assert np.array_equal(x[~fin].view(np.uint32), y[~fin].view(np.uint32))


def test_thread_serial_rejects_corrupt_codes():
    x = synth.nyx_like(2, n=400).reshape(-1).contiguous()  # 64 M values, all blocks nonconstant
    s = szx.compress(x.cuda(), 1e-3, "rel", B)
    h = szx.read_header(s[:64].cpu().numpy().tobytes())
    assert h.n_nonconst == (x.numel() + B - 1) // B
    st = s.cpu().numpy()
    off_pl = st.size - h.payload_bytes
    nB = (x.numel() + B - 1) // B
    off_zs = 64 + ((nB + 7) // 8 + 15) // 16 * 16 + (4 * nB + 15) // 16 * 16
    zs = st[off_zs:off_zs + 2 * nB].view(np.uint16).astype(np.int64)
    k = 1000 * TB + 7                                   # a block in a dense (thread-serial) tile
    pk = off_pl + int(zs[:k].sum())
    cb = pk + 1 + int(np.nonzero(st[pk + 1:pk + 33])[0][0])  # a lead-code byte with a nonzero code
    bad = st.copy()
    bad[cb] = 0                                         # codes 0: more mid-bytes than z holds
    with pytest.raises(szx.SZxError) as ei:
        szx.decompress(torch.from_numpy(bad).cuda())
    assert ei.value.code == -3
    bad = st.copy()
    bad[pk] = 40                                        # R byte out of range
    with pytest.raises(szx.SZxError) as ei:
        szx.decompress(torch.from_numpy(bad).cuda())
    assert ei.value.code == -3
    y = szx.decompress(s)                               # the intact stream still decodes
    yr = oracle.decompress(oracle.compress(x.numpy(), 1e-3, oracle.REL, B))
    assert np.array_equal(y.cpu().numpy().view(np.uint32), yr.view(np.uint32))
