"""Pins for the oracle's quality and overhead analytics:
max abs error / MSE / PSNR (Formula 7) and the Solution C vs
Solution A/B bit accounting of Formula 6.  CPU only; every
expected value comes from a closed form or an independent numpy computation,
never from the oracle itself.
"""
from __future__ import annotations

import math

import numpy as np
import pytest

import oracle


def test_quality_closed_form_constant_offset():
    # x' = x + 1/4 exactly (integers up to 999 and their quarter offsets are
    # exact in float64): max error 1/4, MSE 1/16, PSNR = 20 log10(999 / (1/4)).
    x = np.arange(1000, dtype=np.float64)
    q = oracle.quality(x, x + 0.25)
    assert q["max_abs_err"] == 0.25
    assert q["sse"] == 1000 * 0.0625
    assert q["mse"] == 0.0625
    assert (q["dmin"], q["dmax"]) == (0.0, 999.0)
    assert q["psnr"] == pytest.approx(20 * math.log10(999 / 0.25), rel=1e-15)


def test_quality_lossless_and_nonfinite():
    x = np.array([1.0, np.nan, np.inf, -0.0, 3.0], np.float32)
    q = oracle.quality(x, x.copy())
    assert q["max_abs_err"] == 0.0 and q["sse"] == 0.0 and q["psnr"] == math.inf
    # finite range ignores NaN and Inf (Formula 7's d_min, d_max over the data)
    assert (q["dmin"], q["dmax"]) == (-0.0, 3.0)
    y = x.copy()
    y.view(np.uint32)[1] ^= 1  # another NaN payload: not a faithful round trip
    assert oracle.quality(x, y)["max_abs_err"] == math.inf


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_quality_matches_numpy(dt):
    rng = np.random.default_rng(7)
    x = rng.standard_normal(20000).astype(dt) * 100
    xr = (x + rng.uniform(-1e-2, 1e-2, x.size)).astype(dt)
    q = oracle.quality(x, xr)
    d = np.abs(x.astype(np.float64) - xr.astype(np.float64))
    assert q["max_abs_err"] == d.max()
    assert q["sse"] == pytest.approx(math.fsum(d * d), rel=1e-12)
    assert (q["dmin"], q["dmax"]) == (float(x.min()), float(x.max()))


def _nc_blocks(tr, n, b):
    nB = (n + b - 1) // b
    lens = np.full(nB, b)
    if n % b:
        lens[-1] = n % b
    nc = tr.type.astype(bool)
    return nc, lens


def test_formula6_solution_c_bits_are_the_stored_mid_bytes():
    # Sum of Solution C bits / 8 = the mid-bytes in the stream, a closed form
    # of the header: payload - sum over nonconstant blocks of (1 + ceil(len/4)).
    rng = np.random.default_rng(3)
    x = np.cumsum(rng.standard_normal(50_003)).astype(np.float32)
    s, tr = oracle.compress(x, 1e-3, oracle.REL, 128, trace=True)
    h = oracle.read_header(s)
    nc, lens = _nc_blocks(tr, x.size, 128)
    mid = h["payload_bytes"] - int(np.sum(1 + (lens[nc] + 3) // 4))
    ov = oracle.shift_overhead(s, x)
    assert ov["bits_C"] == 8 * mid


def test_formula6_no_overhead_when_R_is_whole_bytes():
    # Formula 5: R % 8 == 0 -> s = 0, the shifted and unshifted words are the
    # same, so Solution C stores exactly what Solution B needs.  R = 16 for
    # every block: p(r) - p(e) = 7 (R3) with e = 1.5 * 2^-10, r in [1/8, 1/4).
    rng = np.random.default_rng(5)
    nb, b = 64, 128
    base = rng.uniform(-100, 100, nb).astype(np.float32)
    ramp = np.linspace(0.0, 0.3, b, dtype=np.float32)
    x = (base[:, None] + rng.permuted(np.tile(ramp, (nb, 1)), axis=1)).astype(np.float32).reshape(-1)
    s, tr = oracle.compress(x, 1.5 * 2.0 ** -10, oracle.ABS, b, trace=True)
    assert tr.type.all() and (tr.R == 16).all()
    ov = oracle.shift_overhead(s, x)
    assert ov["bits_C"] == ov["bits_B"] and ov["overhead"] == 0.0


def test_formula6_alternating_signs_cost_exactly_s_per_value():
    # Values alternate sign around mu ~ 0, so both the unshifted and the
    # shifted words differ in their top byte (the sign bit sits in bit 31 - s,
    # s <= 7): no identical leading bytes on either side, and each value costs
    # R + s bits under Solution C and R bits under Solution B.
    rng = np.random.default_rng(11)
    nb, b = 40, 128
    mag = (1.0 + rng.uniform(0, 0.5, nb * b)).astype(np.float32)
    sign = np.where(np.arange(nb * b) % 2 == 0, 1.0, -1.0).astype(np.float32)
    x = (mag * sign).astype(np.float32)
    s, tr = oracle.compress(x, 1.5e-3, oracle.ABS, b, trace=True)
    assert tr.type.all() and (tr.R < 32).all() and (tr.R % 8 != 0).all()
    shifts = np.array([(8 - R % 8) % 8 for R in tr.R.astype(int)])
    ov = oracle.shift_overhead(s, x)
    assert ov["bits_C"] - ov["bits_B"] == int(np.sum(shifts * b))
    assert ov["bits_B"] == int(np.sum(tr.R.astype(int) * b))
