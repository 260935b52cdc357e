"""Parity at BASELINE.json's full sizes, in the configuration bench.py times
(block 128, REL bounds of each config).  Configs 1-4 and the float64 fields of
config 5: the whole GPU stream must be byte-identical to the oracle's and the
reconstruction bit-identical.  Config 5's float32 box: one 4.3 GB shard of
the 8-GPU array compared whole, and one stream of more than 2^32 values (17.6 GB)
compared whole at b = 128 and b = 32."""
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


def _full_parity(xd: torch.Tensor, eb: float, tag: str, b: int = 128):
    s = szx.compress(xd, eb, "rel", b)
    x = xd.cpu().numpy().reshape(-1)
    ref = oracle.compress(x, eb, oracle.REL, b)
    got = s.cpu().numpy()
    assert got.size == ref.size and got.tobytes() == ref.tobytes(), tag
    y = szx.decompress(s)
    ui = np.uint32 if x.dtype == np.float32 else np.uint64
    yr = oracle.decompress(ref)
    assert np.array_equal(y.cpu().numpy().view(ui), yr.view(ui)), tag
    e = oracle.read_header(ref)["eb_abs"]
    err = (y.double() - xd.reshape(-1).double()).abs().max().item()
    assert err <= e, (tag, err, e)
    return x.nbytes / got.size


def test_config1_cesm():
    for f in (0, 1):
        _full_parity(synth.cesm_like(f, device="cuda"), 1e-3, f"cesm{f}")


def test_config2_hurricane():
    for f in (0, 1):
        x = synth.hurricane_like(f, device="cuda")
        for eb in (1e-2, 1e-3, 1e-4):
            _full_parity(x, eb, f"hurricane{f}/{eb}")


def test_config3_nyx():
    for f in (0, 1, 2):
        _full_parity(synth.nyx_like(f, n=512, device="cuda"), 1e-3, f"nyx{f}")


@pytest.mark.parametrize("b", [32, 64, 256])
def test_config3_nyx_other_block_sizes(b):
    # the block-size study at full size: dense velocity, sparse density
    for f in (0, 1):
        _full_parity(synth.nyx_like(f, n=512, device="cuda"), 1e-3, f"nyx{f}/b{b}", b)


def test_config4_hacc():
    for f in (0, 1):
        _full_parity(synth.hacc_like(f, device="cuda"), 1e-3, f"hacc{f}")


def test_config5_float64_fields():
    _full_parity(synth.miranda_like(device="cuda"), 1e-4, "miranda64")
    _full_parity(synth.qmcpack_like(device="cuda"), 1e-4, "qmcpack64")


def test_config5_box_shard_whole():
    # one GPU's shard of the 4096x4096x512 box (8 shards along the slowest axis): 1.07 G values,
    # the whole stream byte-compared with the oracle and the reconstruction bit-compared
    x = synth.box_like(shape=(64, 4096, 4096), device="cuda").reshape(-1)
    _full_parity(x, 1e-4, "box-shard")


def _parity_chunked(xd: torch.Tensor, eb: float, b: int, tag: str):
    """_full_parity for arrays too large to hold several host copies of: the streams are compared
    with np.array_equal (no byte copies), the reconstructions 2^28 values at a time."""
    n = xd.numel()
    s = szx.compress(xd, eb, "rel", b)
    x = xd.cpu().numpy()
    ref = oracle.compress(x, eb, oracle.REL, b)
    del x
    got = s.cpu().numpy()
    assert got.size == ref.size, (tag, got.size, ref.size)
    assert np.array_equal(got, ref), tag
    del got
    y = szx.decompress(s)
    del s
    yr = oracle.decompress(ref)
    e = oracle.read_header(ref)["eb_abs"]
    del ref
    CH = 1 << 28
    worst = 0.0
    for c in range(0, n, CH):
        yc = y[c:c + CH]
        assert np.array_equal(yc.cpu().numpy().view(np.uint32), yr[c:c + CH].view(np.uint32)), (tag, c)
        worst = max(worst, (yc.double() - xd[c:c + CH].double()).abs().max().item())
    assert worst <= e, (tag, worst, e)
    return n


@pytest.mark.parametrize("b", [128, 32])
def test_stream_above_2p32_values(b):
    """One stream of more than 2^32 values (4,395,630,515 float32 = 17.6 GB; needs ~55 GB of
    device memory and ~60 GB of host RAM), byte-identical to the oracle's stream: covers the 64-bit
    element / offset paths, the 32-bit nonconstant list and the decoder's packed 32|32 counts above
    2^32 values (Formula 1 + byte identity).  A ragged tail of 51 values (b = 128)."""
    x = synth.box_like(shape=(262, 4096, 4096), device="cuda").reshape(-1)
    n = x.numel() - 77
    assert n > (1 << 32)
    xs = x[:n]
    _parity_chunked(xs, 1e-4, b, f"2^32+ b{b}")
