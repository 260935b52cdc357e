"""Pins for the oracle-side analytics of SURVEY 8(f) rows 1-2 (CPU):
  * Fig. 2's block relative value range against closed forms;
  * Formula 6's Solution C / Solution B bit sums: the oracle's C accounting
    (orc_shift_overhead) against an independent numpy restatement (oracle/analytics.py) on
    seeded fields, float32 and float64, every block size including the oracle-only 8 and 16."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import synth
from oracle import analytics as A


def test_block_relative_range_ramp_closed_form():
    # a linear ramp 0..n-1: every full block spans b-1, the tail block len-1; global range n-1
    n, b = 1000, 16
    x = np.arange(n, dtype=np.float64)
    r = A.block_relative_range(x, b)
    full = n // b
    assert r.size == (n + b - 1) // b
    assert np.all(r[:full] == (b - 1) / (n - 1))
    assert r[-1] == (n - full * b - 1) / (n - 1)
    # a constant field: range 0 -> relative ranges 0; CDF at 0 is 1
    c = A.block_relative_range(np.full(100, 3.5), 8)
    assert np.all(c == 0) and A.cdf_points(c, [0.0]) == [1.0]


def test_block_relative_range_ignores_nonfinite_and_matches_bruteforce():
    rng = np.random.default_rng(3)
    x = rng.standard_normal(777)
    x[[5, 100, 300]] = [np.nan, np.inf, -np.inf]
    b = 8
    r = A.block_relative_range(x, b)
    f = x[np.isfinite(x)]
    g = f.max() - f.min()
    want = []
    for k in range(0, x.size, b):
        blk = x[k:k + b]
        blk = blk[np.isfinite(blk)]
        if blk.size:
            want.append((blk.max() - blk.min()) / g)
    assert np.array_equal(r, np.array(want))
    # CDF points are monotone and end at 1
    pts = A.cdf_points(r, [0.001, 0.01, 0.1, 1.0])
    assert pts == sorted(pts) and pts[-1] == 1.0


@pytest.mark.parametrize("b", [8, 16, 32, 128])
def test_formula6_bits_numpy_cross_check(b):
    cases = [(synth.nyx_like(1, n=24).numpy().reshape(-1), 1e-3),
             (synth.nyx_like(0, n=24).numpy().reshape(-1), 1e-3),
             (synth.special_values(9_999, 5).numpy(), 1e-2),
             (synth.offset_field(8_001, 2, 50.0, dtype=torch.float64).numpy(), 1e-5)]
    for x, eb in cases:
        s = oracle.compress(x, eb, oracle.REL, b)
        ov = oracle.shift_overhead(s, x)
        c, bb = A.shift_bits(s, x)
        assert (ov["bits_C"], ov["bits_B"]) == (c, bb), (x.dtype, b, eb)
