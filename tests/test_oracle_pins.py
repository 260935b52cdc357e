"""Pins for the CPU oracle (oracle/szx_oracle.c) against what the paper and the
mathematics fix -- never against the oracle itself.  CPU only.

  * hand-worked streams (tests/golden/b1_three_blocks.txt, b4_guard.txt)
  * closed-form stream sizes (tests/golden/b2_b3_closed_forms.txt)
  * Fig. 4 printed bit patterns and lead codes (tests/golden/fig4_bits.txt)
  * Formula 5 purpose (R+s multiple of 8), Formula 4 truncation bound
  * Formula 1 error-bound invariant on seeded fields, f32 and f64
  * an independent Fig. 10 decoder (tests/fig10_decoder.py)
  * brute force over tiny blocks built from special values
"""
from __future__ import annotations

import itertools
import os

import numpy as np
import pytest
import torch

import oracle
import synth
from fig10_decoder import decode as fig10_decode

GOLD = os.path.join(os.path.dirname(__file__), "golden")


def _kv(path):
    d = {}
    for line in open(path):
        line = line.strip()
        if not line or line.startswith("#") or ":" not in line:
            continue
        k, v = line.split(":", 1)
        d[k.strip()] = v.strip()
    return d


def _bits_to_f32(words):
    return np.array([int(w, 16) for w in words.split()], dtype=np.uint32).view(np.float32)


def _same_bits(a: np.ndarray, b: np.ndarray) -> bool:
    ui = np.uint32 if a.dtype == np.float32 else np.uint64
    return np.array_equal(a.view(ui), b.view(ui))


def _check_bound(x: np.ndarray, y: np.ndarray, eb_abs: float):
    """Formula 1: |x - x'| <= e for every finite element (double arithmetic);
    non-finite elements must round-trip bit-exactly (R14/R15)."""
    xd = x.astype(np.float64)
    yd = y.astype(np.float64)
    fin = np.isfinite(xd)
    err = np.abs(xd[fin] - yd[fin])
    assert err.size == 0 or err.max() <= eb_abs, (err.max(), eb_abs)
    ui = np.uint32 if x.dtype == np.float32 else np.uint64
    assert np.array_equal(x[~fin].view(ui), y[~fin].view(ui))


# ---------------------------------------------------------------- golden
def test_b1_three_block_stream_hand_derived():
    g = _kv(os.path.join(GOLD, "b1_three_blocks.txt"))
    x = _bits_to_f32(g["input_bits"])
    s, tr = oracle.compress(x, float(g["eb"]), oracle.ABS, int(g["block"]), trace=True)
    want = bytes.fromhex(g["stream_hex"].replace(" ", ""))
    assert s.tobytes() == want
    assert list(tr.type) == [0, 1, 1] and list(tr.R) == [0, 12, 15] and list(tr.z) == [0, 8, 6]
    y = oracle.decompress(s)
    assert _same_bits(y, _bits_to_f32(g["decoded_bits"]))
    y2, _ = fig10_decode(s.tobytes())
    assert _same_bits(y2, y)


def test_b4_guard_forces_nonconstant():
    g = _kv(os.path.join(GOLD, "b4_guard.txt"))
    x = _bits_to_f32(g["input_bits"])
    s, tr = oracle.compress(x, float(g["eb"]), oracle.ABS, int(g["block"]), trace=True)
    assert s.size == int(g["stream_size"])
    assert s[-3:].tobytes() == bytes.fromhex(g["payload_hex"])
    assert list(tr.type) == [1] and list(tr.R) == [9]
    assert _same_bits(oracle.decompress(s), _bits_to_f32(g["decoded_bits"]))


def test_closed_form_sizes_b2_b3():
    rows = [l.split() for l in open(os.path.join(GOLD, "b2_b3_closed_forms.txt"))
            if l.strip() and not l.startswith("#")]
    for name, n, b, mode, eb, spike, S in rows:
        x = np.zeros(int(n), np.float32)
        if int(spike) >= 0:
            x[int(spike)] = 1.0
        s = oracle.compress(x, float(eb), oracle.ABS if mode == "abs" else oracle.REL, int(b))
        assert s.size == int(S), name
        y = oracle.decompress(s)
        assert _same_bits(y, x), name  # exact: r = 0.5 keeps every bit of 0 and 1


def test_all_constant_closed_form_f32_f64():
    for dt, W in ((np.float32, 4), (np.float64, 8)):
        for n, b in ((1, 128), (127, 128), (128 * 37 + 5, 128), (64 * 9, 64), (999, 4)):
            nB = (n + b - 1) // b
            x = np.repeat(np.arange(nB, dtype=dt) * 1.5 - 7.0, b)[:n]
            s = oracle.compress(x, 1e-3, oracle.ABS, b)
            al = lambda v: (v + 15) // 16 * 16
            assert s.size == 64 + al((nB + 7) // 8) + al(W * nB)
            assert _same_bits(oracle.decompress(s), x)


# ---------------------------------------------------------------- Fig. 4
def test_fig4_bit_patterns_and_codes():
    rows = [l.split() for l in open(os.path.join(GOLD, "fig4_bits.txt"))
            if l.strip() and not l.startswith("#") and ":" not in l]
    words = []
    for val, req, insig in rows:
        w = int(np.float32(float(val)).view(np.uint32))
        assert format(w, "032b") == req + insig  # the paper's printed IEEE-754 layout
        words.append(w)
    g = _kv(os.path.join(GOLD, "fig4_bits.txt"))
    # xor_leadingzero_array[i] = 2, [i+1] = 1 (unshifted, as drawn)
    got = [oracle.identical_leading_bytes(words[0], words[1], 4),
           oracle.identical_leading_bytes(words[1], words[2], 4)]
    assert got == [int(c) for c in g["codes_unshifted"].split()]
    # R = 27 -> s = 5 (Formula 5); after the shift the codes are 2, 2
    s = oracle.shift_for(27)
    assert s == 5
    got = [oracle.identical_leading_bytes(words[0] >> s, words[1] >> s, 4),
           oracle.identical_leading_bytes(words[1] >> s, words[2] >> s, 4)]
    assert got == [int(c) for c in g["codes_shift5"].split()]


def test_identical_leading_bytes_cap_and_order():
    # 2-bit code: 0..3 identical bytes; counted from the most significant byte
    assert oracle.identical_leading_bytes(0x12345678, 0x12345678, 4) == 3
    assert oracle.identical_leading_bytes(0x12345678, 0x92345678, 4) == 0
    assert oracle.identical_leading_bytes(0x12345678, 0x12345679, 4) == 3
    assert oracle.identical_leading_bytes(0x12345678, 0x12355678, 4) == 1
    assert oracle.identical_leading_bytes(0x1234567800000000, 0x1234567900000000, 8) == 3
    assert oracle.identical_leading_bytes(0x1234567800000000, 0x1233567800000000, 8) == 1
    assert oracle.identical_leading_bytes(0, 0x00FC0000, 4) == 1


# ---------------------------------------------------------------- Formulas 4/5
def test_formula5_makes_whole_bytes():
    for R in range(1, 65):
        s = oracle.shift_for(R)
        assert 0 <= s < 8 and (R + s) % 8 == 0  # "always a multiple of 8"
        if R % 8 == 0:
            assert s == 0


def test_exponent_function_matches_frexp():
    rng = np.random.default_rng(5)
    for v in np.concatenate([rng.standard_normal(200) * 10.0 ** rng.integers(-30, 30, 200),
                             [1.0, 0.5, 2.0, 3.9999, 1e-3, 0.05]]):
        m, e = np.frexp(v)          # v = m * 2^e, 0.5 <= |m| < 1  -> IEEE exponent e-1
        assert oracle.p_f64(float(v)) == e - 1
        v32 = np.float32(v)
        if np.isfinite(v32) and abs(v32) >= np.finfo(np.float32).tiny:
            assert oracle.p_f32(float(v32)) == np.frexp(v32)[1] - 1


def _trunc_keep_top(bits: int, R: int, W: int) -> int:
    mask = ((1 << (8 * W)) - 1) ^ ((1 << (8 * W - R)) - 1)
    return bits & mask


def test_formula4_truncation_error_below_error_bound():
    """With R from Formula 4 (R3 reading), keeping the top R bits of any v whose
    exponent does not exceed p(r) errs by < 2^p(e) <= e."""
    rng = np.random.default_rng(11)
    for _ in range(3000):
        e = float(10.0 ** rng.uniform(-8, 1))
        r = np.float32(e * 2.0 ** rng.uniform(0.0, 20.0))
        R = oracle.required_bits_f32(float(r), e)
        if R >= 32:
            continue
        pr = oracle.p_f32(float(r))
        v = np.float32(rng.uniform(-1, 1) * 2.0 ** (pr + 1))
        if v == 0 or np.frexp(v)[1] - 1 > pr:
            continue
        vb = int(v.view(np.uint32))
        vt = np.uint32(_trunc_keep_top(vb, R, 4)).view(np.float32)
        assert abs(float(v) - float(vt)) < 2.0 ** oracle.p_f64(e) <= e
    for _ in range(2000):
        e = float(10.0 ** rng.uniform(-12, 1))
        r = e * 2.0 ** rng.uniform(0.0, 40.0)
        R = oracle.required_bits_f64(r, e)
        if R >= 64:
            continue
        pr = oracle.p_f64(r)
        v = rng.uniform(-1, 1) * 2.0 ** (pr + 1)
        if v == 0 or np.frexp(v)[1] - 1 > pr:
            continue
        vb = int(np.float64(v).view(np.uint64))
        vt = np.uint64(_trunc_keep_top(vb, R, 8)).view(np.float64)
        assert abs(v - float(vt)) < 2.0 ** oracle.p_f64(e) <= e


def test_formula4_branches():
    # p(r)-p(e) <= 0 -> no mantissa bits (R = sign+exponent); > fullbits -> raw
    assert oracle.required_bits_f32(0.01, 0.1) == 9
    assert oracle.required_bits_f32(1e30, 1e-30) == 32
    assert oracle.required_bits_f64(1e300, 1e-300) == 64
    assert oracle.required_bits_f64(0.01, 0.1) == 12
    assert oracle.required_bits_f32(1.0, 2.0 ** -10) == 19
    assert oracle.required_bits_f64(1.0, 2.0 ** -10) == 22


# ---------------------------------------------------------------- REL definition
def test_rel_error_bound_is_value_range_relative():
    x = synth.special_values(5000, 3).numpy()
    fin = x[np.isfinite(x)].astype(np.float64)
    want = 1e-3 * (fin.max() - fin.min())  # footnote 1
    assert oracle.eb_abs(x, 1e-3, oracle.REL) == want
    assert oracle.eb_abs(x, 0.25, oracle.ABS) == 0.25
    assert oracle.eb_abs(np.full(10, np.nan, np.float32), 1e-3, oracle.REL) == 0.0
    z = np.array([0.0, -0.0], np.float32)
    assert np.signbit(oracle.eb_abs(z, 1e-3, oracle.REL)) == False


# ---------------------------------------------------------------- invariants
FIELDS = {
    "grf2d": lambda: synth.grf((96, 130), 5.0, 7).numpy().reshape(-1),
    "cesm_clip": lambda: synth.cesm_like(1, shape=(90, 180)).numpy().reshape(-1),
    "hurricane_u": lambda: synth.hurricane_like(0, shape=(10, 50, 50)).numpy().reshape(-1),
    "hurricane_q": lambda: synth.hurricane_like(1, shape=(10, 50, 50)).numpy().reshape(-1),
    "nyx_dens": lambda: synth.nyx_like(0, n=32).numpy().reshape(-1),
    "hacc_vel": lambda: synth.hacc_like(0, n=20011).numpy(),
    "hacc_pos": lambda: synth.hacc_like(1, n=20011).numpy(),
    "special": lambda: synth.special_values(12345, 9).numpy(),
    "offset1000": lambda: synth.offset_field(40000, 4, 1000.0).numpy(),
    "mix": lambda: synth.random_mix(30011, 8).numpy(),
}


@pytest.mark.parametrize("name", sorted(FIELDS))
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_error_bound_and_independent_decoder(name, dt):
    x = FIELDS[name]().astype(dt)
    for mode, eb, b in ((oracle.REL, 1e-2, 128), (oracle.REL, 1e-4, 128), (oracle.ABS, 1e-3, 64),
                        (oracle.REL, 1e-3, 4)):
        s, tr = oracle.compress(x, eb, mode, b, trace=True)
        e = oracle.eb_abs(x, eb, mode)
        assert oracle.read_header(s)["eb_abs"] == e
        y = oracle.decompress(s)
        _check_bound(x, y, e)
        if x.size <= 20000 or b == 128:
            y2, info = fig10_decode(s.tobytes())
            assert _same_bits(y2, y)
        assert s.size <= oracle.compress_bound(x.size, 0 if dt == np.float32 else 1, b)


def test_offset_fields_hold_bound():
    """Large offset relative to the range: the R2 constant guard
    matters here; Formula 1 must hold for every element."""
    for off in (1000.0, 4000.0, 12345.678):
        x = synth.offset_field(200000, 12, off).numpy()
        for eb in (1e-2, 1e-3, 1e-4):
            s, tr = oracle.compress(x, eb, oracle.REL, 128, trace=True)
            _check_bound(x, oracle.decompress(s), oracle.eb_abs(x, eb, oracle.REL))


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_guard_escalation_path(dt):
    """Start R below Formula 4 (test hook): the per-element R2 check must escalate
    R one bit at a time until Formula 1 holds, i.e. it lands at or below R4."""
    x = synth.random_mix(20000, 77).numpy().astype(dt)
    s0, t0 = oracle.compress(x, 1e-3, oracle.REL, 128, trace=True)
    s, tr = oracle.compress(x, 1e-3, oracle.REL, 128, trace=True, r_bias=-6)
    e = oracle.eb_abs(x, 1e-3, oracle.REL)
    _check_bound(x, oracle.decompress(s), e)
    nc = t0.type == 1
    assert tr.escal.sum() > 0
    assert np.all(tr.R[nc] <= t0.R[nc])
    y2, _ = fig10_decode(s.tobytes())
    assert _same_bits(y2, oracle.decompress(s))


def test_lossless_at_zero_error_bound():
    for dt in (np.float32, np.float64):
        x = synth.special_values(3000, 21, dtype=torch.float32 if dt == np.float32 else torch.float64).numpy()
        s = oracle.compress(x, 0.0, oracle.ABS, 128)
        y = oracle.decompress(s)
        ui = np.uint32 if dt == np.float32 else np.uint64
        same = x.view(ui) == y.view(ui)
        # only all-zero constant blocks may turn -0 into +0 (R1: mu = mn + r)
        assert np.all(same | ((x == 0) & (y == 0)))


def test_nonfinite_blocks_are_raw_and_exact():
    x = np.array([1.0, np.nan, 2.0, 3.0, np.inf, 5.0, 6.0, 7.0, -np.inf, -np.inf, 1.0, 1.0], np.float32)
    s, tr = oracle.compress(x, 0.5, oracle.ABS, 4, trace=True)
    assert list(tr.type) == [1, 1, 1] and list(tr.R) == [32, 32, 32]
    assert list(tr.mu) == [0, 0, 0]
    assert _same_bits(oracle.decompress(s), x)


# ---------------------------------------------------------------- brute force
def test_brute_force_tiny_blocks():
    vals = np.array([0.0, -0.0, 1.0, 1.0000001, -3.5, 1e-40, 65504.0, np.inf], np.float32)
    combos = np.array(list(itertools.product(range(len(vals)), repeat=4)))
    x = vals[combos].reshape(-1)
    for eb in (0.0, 1e-7, 0.01, 1.0, 100.0):
        s, tr = oracle.compress(x, eb, oracle.ABS, 4, trace=True)
        y = oracle.decompress(s)
        _check_bound(x, y, eb)
        y2, _ = fig10_decode(s.tobytes())
        assert _same_bits(y, y2)
        assert np.all(tr.escal <= 23)


# ---------------------------------------------------------------- container
def test_container_shards_match_standalone_streams():
    x = synth.random_mix(50000, 31).numpy()
    nB = (x.size + 127) // 128
    for P in (1, 2, 3, 8):
        c = oracle.container_compress(x, 1e-3, oracle.REL, 128, P)
        assert c[:4].tobytes() == b"SZXC"
        e = oracle.eb_abs(x, 1e-3, oracle.REL)
        y = oracle.decompress(c)
        _check_bound(x, y, e)
        # each shard = a standalone stream of its block range with the global eb_abs
        for p in range(P):
            ent = c[32 + 32 * p: 64 + 32 * p].view(np.uint64)
            first, cnt, off, nbytes = (int(v) for v in ent)
            b0, b1 = nB * p // P, nB * (p + 1) // P
            assert first == b0 * 128 and cnt == min(x.size, b1 * 128) - first and off % 16 == 0
            shard = c[off:off + nbytes]
            ref = oracle.compress(x[first:first + cnt], e, oracle.ABS, 128)
            h = oracle.read_header(shard)
            assert h["mode"] == oracle.REL and h["eb_user"] == 1e-3 and h["eb_abs"] == e
            a, b = shard.copy(), ref.copy()
            a[6] = b[6] = 0
            a[24:32] = b[24:32] = 0
            assert a.tobytes() == b.tobytes()
        if P == 1:
            assert np.array_equal(y, oracle.decompress(oracle.compress(x, 1e-3, oracle.REL, 128)))


# ---------------------------------------------------------------- errors
def test_argument_and_corruption_errors():
    x = np.linspace(0, 1, 1000, dtype=np.float32)
    assert oracle.compress_rc(x, -1.0) == oracle.EINVAL
    assert oracle.compress_rc(x, float("nan")) == oracle.EINVAL
    assert oracle.compress_rc(x, 1e-3, b=6) == oracle.EINVAL
    s = oracle.compress(x, 1e-3, oracle.REL, 128)
    assert oracle.decompress_rc(s[:-1], x.size, np.float32) == oracle.ECORRUPT
    bad = s.copy(); bad[0] = ord("X")
    assert oracle.decompress_rc(bad, x.size, np.float32) == oracle.ECORRUPT
    h = oracle.read_header(s)
    nB = (x.size + 127) // 128
    zoff = 64 + 16 + (4 * nB + 15) // 16 * 16
    bad = s.copy(); bad[zoff] ^= 1      # zsize no longer sums to payload_bytes
    assert oracle.decompress_rc(bad, x.size, np.float32) == oracle.ECORRUPT
    assert oracle.decompress_rc(s, x.size - 1, np.float32) == oracle.ENOSPC
    e = oracle.compress(np.zeros(0, np.float32), 1e-3, oracle.REL, 128)
    assert e.size == 64 and oracle.decompress(e).size == 0 and h["nnc"] >= 1
