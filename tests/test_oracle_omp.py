"""The paper's OpenMP design as a host baseline (Sec. 6.1 "Parallelization",
P:L2338-2377): Loop 1 broken over threads, a zsize_array and prefix sums.  It must produce ONE
stream byte-identical to the serial oracle's for every thread count, and its parallel decoder
must reproduce the serial decoder's values bit for bit."""
from __future__ import annotations

import numpy as np
import pytest
import torch

import oracle
import synth


def _cases():
    yield "nyx-velocity", synth.nyx_like(1, n=48).numpy().reshape(-1), 1e-3, oracle.REL, 128
    yield "nyx-density", synth.nyx_like(0, n=48).numpy().reshape(-1), 1e-3, oracle.REL, 128
    yield "special-f32", synth.special_values(30_011, 3).numpy(), 1e-2, oracle.REL, 64
    yield "special-f64", synth.special_values(20_007, 4, dtype=torch.float64).numpy(), 1e-4, oracle.REL, 128
    yield "mix-abs", synth.random_mix(50_001, 5).numpy(), 1e-3, oracle.ABS, 32
    yield "offset-f64", synth.offset_field(9_999, 6, 1e4, dtype=torch.float64).numpy(), 1e-6, oracle.ABS, 256
    yield "tiny", np.array([1.0, 2.0, 3.0], dtype=np.float32), 0.1, oracle.ABS, 128
    yield "empty", np.zeros(0, dtype=np.float32), 1e-3, oracle.REL, 128


@pytest.mark.parametrize("threads", [1, 2, 5, 16])
def test_omp_stream_identical_to_serial_oracle(threads):
    for tag, x, eb, mode, b in _cases():
        ref = oracle.compress(x, eb, mode, b)
        got = oracle.omp_compress(x, eb, mode, b, threads=threads)
        assert got.size == ref.size and np.array_equal(got, ref), (tag, threads)
        if x.size:
            ui = np.uint32 if x.dtype == np.float32 else np.uint64
            y = oracle.omp_decompress(got, threads=threads)
            assert np.array_equal(y.view(ui), oracle.decompress(ref).view(ui)), (tag, threads)


def test_omp_decoder_rejects_corrupt_zsize():
    x = synth.nyx_like(1, n=32).numpy().reshape(-1)
    s = oracle.compress(x, 1e-3, oracle.REL, 128)
    h = oracle.read_header(s)
    nB = (x.size + 127) // 128
    al = lambda v: (v + 15) // 16 * 16
    off_zs = 64 + al((nB + 7) // 8) + al(4 * nB)
    bad = s.copy()
    bad[off_zs] ^= 0x01  # payload sum no longer matches the header
    with pytest.raises(ValueError):
        oracle.omp_decompress(bad, threads=4)
    assert h["nnc"] > 0
