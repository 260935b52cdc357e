"""GPU parity: the sm_100a path (through the C ABI) against the CPU oracle.

Bar (BASELINE.json north_star): byte-identical compressed streams and
bit-identical reconstructions, and max |x - x'| <= eb with zero slack.
Inputs come from synth/ (seeded); both sides get the same bytes.
"""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

cuda = pytest.importorskip("torch").cuda
if not cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_hpdc_yudztt0c22_b200 as szx  # noqa: E402


def _ui(dt):
    return np.uint32 if dt == np.float32 else np.uint64


def _parity(x: np.ndarray, eb: float, mode: str, b: int = 128, tag: str = ""):
    """Compress on GPU and oracle, compare bytes; decompress on GPU, compare bits."""
    mcode = oracle.REL if mode == "rel" else oracle.ABS
    ref = oracle.compress(x, eb, mcode, b)
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    s = szx.compress(xd, eb, mode, b)
    got = s.cpu().numpy()
    if got.tobytes() != ref.tobytes():
        n = min(got.size, ref.size)
        diff = np.nonzero(got[:n] != ref[:n])[0]
        first = int(diff[0]) if diff.size else n
        raise AssertionError(f"{tag}: stream mismatch: gpu {got.size} B vs oracle {ref.size} B, "
                             f"first differing byte {first}")
    y = szx.decompress(s).cpu().numpy()
    yr = oracle.decompress(ref)
    ui = _ui(x.dtype)
    assert np.array_equal(y.view(ui), yr.view(ui)), f"{tag}: reconstruction mismatch"
    # GPU decoder on the oracle's bytes (independent of the GPU encoder)
    y2 = szx.decompress(torch.from_numpy(ref).cuda()).cpu().numpy()
    assert np.array_equal(y2.view(ui), yr.view(ui))
    e = oracle.eb_abs(x, eb, mcode)
    fin = np.isfinite(x)
    if fin.any():
        err = np.abs(x[fin].astype(np.float64) - y[fin].astype(np.float64)).max()
        assert err <= e, (tag, err, e)
    assert np.array_equal(x[~fin].view(ui), y[~fin].view(ui))
    return got.size


SMALL = {
    "grf2d": lambda: synth.grf((96, 130), 5.0, 7).numpy().reshape(-1),
    "cesm_clip": lambda: synth.cesm_like(1, shape=(180, 360)).numpy().reshape(-1),
    "hurricane_u": lambda: synth.hurricane_like(0, shape=(10, 100, 100)).numpy().reshape(-1),
    "hurricane_q": lambda: synth.hurricane_like(1, shape=(10, 100, 100)).numpy().reshape(-1),
    "nyx_dens": lambda: synth.nyx_like(0, n=64).numpy().reshape(-1),
    "nyx_vel": lambda: synth.nyx_like(1, n=40).numpy().reshape(-1),
    "hacc_vel": lambda: synth.hacc_like(0, n=200_011).numpy(),
    "hacc_pos": lambda: synth.hacc_like(1, n=200_011).numpy(),
    "special": lambda: synth.special_values(123_457, 9).numpy(),
    "offset": lambda: synth.offset_field(300_000, 4, 1000.0).numpy(),
    "mix": lambda: synth.random_mix(250_013, 8).numpy(),
}


@pytest.mark.parametrize("name", sorted(SMALL))
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_parity_small_fields(name, dt):
    x = SMALL[name]().astype(dt)
    for mode, eb in (("rel", 1e-2), ("rel", 1e-3), ("rel", 1e-4), ("abs", 1e-3)):
        for b in (32, 64, 128, 256):
            _parity(x, eb, mode, b, f"{name}/{dt.__name__}/{mode}{eb}/b{b}")


@pytest.mark.parametrize("n", [0, 1, 3, 4, 5, 31, 127, 128, 129, 255, 256, 4095, 4096, 4097,
                               32 * 128, 32 * 128 + 1, 257 * 128 - 1, 33 * 256 * 128 + 77])
def test_parity_sizes_and_tails(n):
    x = synth.random_mix(max(n, 1), 100 + n).numpy()[:n]
    for dt in (np.float32, np.float64):
        for b in (32, 64, 128, 256):
            _parity(x.astype(dt), 1e-3, "rel", b, f"n={n}/{dt.__name__}/b{b}")


def test_parity_zero_error_bound_and_all_constant():
    x = synth.special_values(70_000, 5).numpy()
    _parity(x, 0.0, "abs", 128, "eb0")
    _parity(np.zeros(100_000, np.float32), 1e-3, "rel", 128, "zeros")
    _parity(np.full(100_003, 7.25, np.float64), 0.0, "abs", 256, "const64")
    z = np.zeros(1000, np.float32)
    z[::3] = -0.0
    _parity(z, 1e-3, "rel", 128, "signed zeros")


def test_parity_closed_form_golden_cases():
    # B3 single spike, with the spike inside / first / last (tests/golden/b2_b3_closed_forms.txt)
    for pos, S in ((64, 154), (0, 150), (127, 151)):
        x = np.zeros(256, np.float32)
        x[pos] = 1.0
        assert _parity(x, 1e-3, "abs", 128, f"spike@{pos}") == S


def test_parity_escalation_path():
    """R2 escalation through the test hook (both sides start r_bias bits low)."""
    x = synth.random_mix(300_000, 77).numpy()
    try:
        szx.set_r_bias(-6)
        for dt in (np.float32, np.float64):
            xx = x.astype(dt)
            ref, tr = oracle.compress(xx, 1e-3, oracle.REL, 128, trace=True, r_bias=-6)
            assert tr.escal.sum() > 0
            got = szx.compress(torch.from_numpy(xx).cuda(), 1e-3, "rel", 128).cpu().numpy()
            assert got.tobytes() == ref.tobytes()
            y = szx.decompress(torch.from_numpy(got).cuda()).cpu().numpy()
            assert np.array_equal(y.view(_ui(dt)), oracle.decompress(ref).view(_ui(dt)))
    finally:
        szx.set_r_bias(0)


@pytest.mark.parametrize("rb,n,dt", [(-3, 50_000, np.float32), (-2, 50_000, np.float32), (-3, 50_048, np.float32),
                                     (-3, 128 * 16 * 5 + 77, np.float32), (-3, 50_000, np.float64),
                                     (-5, 128 * 16 * 3 + 5, np.float64)])
def test_parity_escalation_in_partial_last_block(rb, n, dt):
    """The R2 guard / escalation must also run on the partial last block (a large offset makes
    the per-block proof fail, so every block is checked value by value; Formula 1)."""
    x = synth.offset_field(n, 7, 3e3, dtype=torch.float32 if dt == np.float32 else torch.float64).numpy()
    try:
        szx.set_r_bias(rb)
        got = szx.compress(torch.from_numpy(x).cuda(), 1e-4, "rel", 128).cpu().numpy()
    finally:
        szx.set_r_bias(0)
    ref, tr = oracle.compress(x, 1e-4, oracle.REL, 128, trace=True, r_bias=rb)
    assert tr.escal.sum() > 0
    assert got.tobytes() == ref.tobytes()


def test_corrupt_streams_are_rejected():
    x = synth.random_mix(50_000, 3).numpy()
    s = szx.compress(torch.from_numpy(x).cuda(), 1e-3, "rel", 128)
    h = s.cpu().numpy()
    n = x.size
    nB = (n + 127) // 128
    off_zs = 64 + ((nB + 7) // 8 + 15) // 16 * 16 + (4 * nB + 15) // 16 * 16
    cases = []
    b = h.copy(); b[0] = 0; cases.append(b)                      # magic
    b = h.copy(); b[off_zs] ^= 0x40; cases.append(b)              # zsize no longer sums to payload
    b = h.copy(); b[64] ^= 0x01; cases.append(b)                  # bitmap popcount != nNC
    cases.append(h[:-5].copy())                                   # truncated
    hdr = szx.read_header(h[:64].tobytes())
    off_pl = h.size - hdr.payload_bytes
    b = h.copy(); b[off_pl] = 200; cases.append(b)               # R byte out of range
    for c in cases:
        with pytest.raises(szx.SZxError) as ei:
            szx.decompress(torch.from_numpy(c).cuda())
        assert ei.value.code == -3
    # the intact stream still decodes
    szx.decompress(s)


def test_host_entry_points_round_trip():
    x = synth.nyx_like(2, n=32).reshape(-1)
    xp = x.pin_memory()
    s = szx.compress_host(xp, 1e-3, "rel", 128)
    ref = oracle.compress(x.numpy(), 1e-3, oracle.REL, 128)
    assert s.numpy().tobytes() == ref.tobytes()
    y = szx.decompress_host(s)
    assert np.array_equal(y.numpy().view(np.uint32), oracle.decompress(ref).view(np.uint32))


def test_async_codec_matches_sync():
    x = synth.nyx_like(0, n=64).reshape(-1).cuda()
    c = szx.Codec(x.numel(), torch.float32, 128)
    c.compress_async(x, 1e-3, "rel")
    nbytes = c.stream_bytes()
    s = szx.compress(x, 1e-3, "rel", 128)
    assert nbytes == s.numel() and torch.equal(c.out[:nbytes], s)
    h = c.header()
    y = torch.empty_like(x)
    c.decompress_async(c.out[:nbytes], h, y)
    assert int(c.d_status.item()) == 0
    assert torch.equal(y, szx.decompress(s))
