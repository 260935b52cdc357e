"""Parity at BASELINE.json's full sizes, in the configuration bench.py times
(block 128, REL bounds of each config).  Configs 1-4 and the float64 fields of
config 5: the whole GPU stream must be byte-identical to the oracle's and the
reconstruction bit-identical.  Config 5's float32 box (one 4.3 GB shard of the
8-GPU array): sampled block ranges are re-encoded by the oracle with the
stream's global bound and compared payload-by-payload, and Formula 1 is
checked for every element on the GPU."""
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


def test_config5_box_shard_sampled():
    # one GPU's shard of the 4096x4096x512 box (8 shards along the slowest axis)
    x = synth.box_like(shape=(64, 4096, 4096), device="cuda").reshape(-1)
    n = x.numel()
    s = szx.compress(x, 1e-4, "rel", 128)
    h = szx.read_header(s[:64].cpu().numpy().tobytes())
    nB = (n + 127) // 128
    al = lambda v: (v + 15) // 16 * 16
    off_mu = 64 + al((nB + 7) // 8)
    off_zs = off_mu + al(4 * nB)
    off_pl = off_zs + al(2 * h.n_nonconst)
    bm = s[64:64 + (nB + 7) // 8].cpu().numpy()
    nc_flags = np.unpackbits(bm, bitorder="little")[:nB].astype(np.int64)
    ncidx = np.cumsum(nc_flags) - nc_flags
    zs = s[off_zs:off_zs + 2 * h.n_nonconst].cpu().numpy().view(np.uint16).astype(np.int64)
    zpre = np.concatenate([[0], np.cumsum(zs)])
    rng = np.random.default_rng(5)
    for k0 in rng.integers(0, nB - 64, 12):
        k1 = k0 + 64
        xs = x[k0 * 128:k1 * 128].cpu().numpy()
        ref = oracle.compress_shard(xs, 1e-4, h.eb_abs, oracle.REL, 128)
        rh = oracle.read_header(ref)
        r_nnc = rh["nnc"]
        # bitmap bits, mu values and payload bytes of the block range must agree
        assert int(nc_flags[k0:k1].sum()) == r_nnc
        mu_gpu = s[off_mu + 4 * k0: off_mu + 4 * k1].cpu().numpy()
        r_off_mu = 64 + al((64 + 7) // 8)
        assert mu_gpu.tobytes() == ref[r_off_mu:r_off_mu + 256].tobytes()
        a, b = zpre[ncidx[k0]], zpre[ncidx[k0] + r_nnc]
        pay = s[off_pl + a:off_pl + b].cpu().numpy()
        assert pay.tobytes() == ref[ref.size - rh["payload_bytes"]:].tobytes()
    y = szx.decompress(s)
    err = (y.double() - x.double()).abs().max().item()
    assert err <= h.eb_abs
