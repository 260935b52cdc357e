"""GPU parity of the fused reconstruction-quality path:
szx_decompress_quality decodes and, in the same kernel, measures the
reconstruction against the original -- Formula 1's max |x - x'|
and Formula 7's MSE / value range / PSNR -- compared with the
oracle's orc_quality on the same bytes.

Bar: values bit-identical to szx_decompress; max error, d_min and d_max
exact (max and min are order-free); the sum of squared errors to 1e-12
relative (the GPU sums in a different order than the oracle's index order;
each term is exact in double for float32 data, so only the summation
rounding differs: <= n * 2^-53 relative).
"""
from __future__ import annotations

import math

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_hpdc_yudztt0c22_b200 as szx  # noqa: E402


def _check(x: np.ndarray, eb: float, mode: str, b: int = 128, tag: str = ""):
    xd = torch.from_numpy(np.ascontiguousarray(x)).cuda()
    s = szx.compress(xd, eb, mode, b)
    y, q = szx.decompress_quality(s, xd)
    ui = np.uint32 if x.dtype == np.float32 else np.uint64
    y0 = szx.decompress(s).cpu().numpy()
    assert np.array_equal(y.cpu().numpy().view(ui), y0.view(ui)), tag
    qo = oracle.quality(x, y0)
    assert q["max_abs_err"] == qo["max_abs_err"], (tag, q, qo)
    assert q["dmin"] == qo["dmin"] and q["dmax"] == qo["dmax"], (tag, q, qo)
    assert q["sse"] == pytest.approx(qo["sse"], rel=1e-12, abs=0.0), tag
    if math.isfinite(qo["psnr"]):
        assert q["psnr"] == pytest.approx(qo["psnr"], rel=1e-12), tag
    else:
        assert q["psnr"] == qo["psnr"], tag
    # Formula 1 through the fused path: the max error never exceeds the bound
    e = oracle.eb_abs(x, eb, oracle.REL if mode == "rel" else oracle.ABS)
    if np.isfinite(x).all():
        assert q["max_abs_err"] <= e, tag
    return q


FIELDS = {
    "nyx_dens": lambda: synth.nyx_like(0, n=64).numpy().reshape(-1),
    "nyx_vel": lambda: synth.nyx_like(1, n=40).numpy().reshape(-1),
    "hurricane_q": lambda: synth.hurricane_like(1, shape=(10, 100, 100)).numpy().reshape(-1),
    "hacc_vel": lambda: synth.hacc_like(0, n=200_011).numpy(),
    "mix": lambda: synth.random_mix(250_013, 8).numpy(),
}


@pytest.mark.parametrize("name", sorted(FIELDS))
@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_quality_matches_oracle(name, dt):
    x = FIELDS[name]().astype(dt)
    for mode, eb in (("rel", 1e-3), ("abs", 1e-2)):
        for b in (32, 64, 128, 256):
            _check(x, eb, mode, b, f"{name}/{dt.__name__}/{mode}{eb}/b{b}")


def test_quality_special_values_and_lossless():
    x = synth.special_values(123_457, 9).numpy()
    q = _check(x, 1e-3, "rel", 128, "special")
    assert q["max_abs_err"] < math.inf  # NaN / Inf go through raw blocks bit-exactly
    q0 = _check(x, 0.0, "abs", 128, "eb0")
    assert q0["max_abs_err"] == 0.0 and q0["sse"] == 0.0 and q0["psnr"] == math.inf


@pytest.mark.parametrize("n", [1, 127, 4097, 33 * 256 * 128 + 77])
def test_quality_tails(n):
    x = synth.random_mix(n, 300 + n).numpy()
    _check(x, 1e-3, "rel", 128, f"n={n}")


def test_quality_container_and_async_codec():
    x = synth.nyx_like(0, n=64).reshape(-1)
    # a 3-shard container, decoded and measured in one call
    cont = oracle.container_compress(x.numpy(), 1e-3, oracle.REL, 128, 3)
    xd = x.cuda()
    y, q = szx.decompress_quality(torch.from_numpy(cont).cuda(), xd)
    qo = oracle.quality(x.numpy(), oracle.decompress(cont))
    assert q["max_abs_err"] == qo["max_abs_err"] and q["sse"] == pytest.approx(qo["sse"], rel=1e-12)
    # the non-blocking codec path
    c = szx.Codec(xd.numel(), torch.float32, 128)
    c.compress_async(xd, 1e-3, "rel")
    h = c.header()
    yy = torch.empty_like(xd)
    c.decompress_quality_async(c.out, h, yy, xd)
    qa = c.quality()
    assert int(c.d_status.item()) == 0
    assert torch.equal(yy, szx.decompress(c.out[:c.stream_bytes()]))
    qo = oracle.quality(x.numpy(), yy.cpu().numpy())
    assert qa["max_abs_err"] == qo["max_abs_err"] and qa["dmin"] == qo["dmin"] and qa["dmax"] == qo["dmax"]
