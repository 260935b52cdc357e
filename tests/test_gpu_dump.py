"""GPU parity of the dump / load pipeline (the single-box
analogue of the paper's dumping / loading experiment, Fig. 16):
szx_dump_host writes a device array to host memory as an SZXC container of P
block-range shards, overlapping the compression of shard p+1 with the copy-out
of shard p; szx_load_host reverses it.  Bar: the container is byte-identical
to the oracle's P-shard container (the shard rule and the global REL bound are
fixed, DESIGN.md s.8), and the loaded values are bit-identical to the
oracle's reconstruction."""
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


def _ui(dt):
    return np.uint32 if dt == np.float32 else np.uint64


@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("P", [1, 3, 8])
@pytest.mark.parametrize("n", [1, 1000, 250_013, 32 * 128 * 7 + 5])
def test_dump_matches_oracle_container(dt, P, n):
    x = synth.random_mix(n, 500 + n).numpy().astype(dt)
    nB = (n + 127) // 128
    for mode, mc, eb in (("rel", oracle.REL, 1e-3), ("abs", oracle.ABS, 1e-2)):
        c = szx.dump_host(torch.from_numpy(x).cuda(), eb, mode, 128, P)
        ref = oracle.container_compress(x, eb, mc, 128, min(P, nB))
        assert c.numpy().tobytes() == ref.tobytes(), (dt, P, n, mode)
        y = szx.load_host(c).cpu().numpy()
        assert np.array_equal(y.view(_ui(dt)), oracle.decompress(ref).view(_ui(dt)))


def test_dump_load_nyx_and_streams():
    x = synth.nyx_like(1, n=128).reshape(-1)
    xd = x.cuda()
    c = szx.dump_host(xd, 1e-3, "rel", 128, 16)
    ref = oracle.container_compress(x.numpy(), 1e-3, oracle.REL, 128, 16)
    assert c.numpy().tobytes() == ref.tobytes()
    y = szx.load_host(c)
    assert torch.equal(y, szx.decompress(torch.from_numpy(ref).cuda()))
    # a bare SZX1 stream loads too, and 256-blocks
    for b in (32, 64, 256):
        s = oracle.compress(x.numpy(), 1e-3, oracle.REL, b)
        y2 = szx.load_host(torch.from_numpy(s).pin_memory())
        assert np.array_equal(y2.cpu().numpy().view(np.uint32), oracle.decompress(s).view(np.uint32))
        c = szx.dump_host(xd, 1e-3, "rel", b, 5)
        assert c.numpy().tobytes() == oracle.container_compress(x.numpy(), 1e-3, oracle.REL, b, 5).tobytes()


def test_load_rejects_corrupt_and_dump_checks_capacity():
    x = synth.random_mix(100_000, 9).numpy()
    c = szx.dump_host(torch.from_numpy(x).cuda(), 1e-3, "rel", 128, 4).numpy().copy()
    bad = c.copy()
    bad[32 + 16] ^= 1  # first shard offset no longer 16-aligned
    with pytest.raises(szx.SZxError) as ei:
        szx.load_host(torch.from_numpy(bad))
    assert ei.value.code == -3
    small = torch.empty(100, dtype=torch.uint8, pin_memory=True)
    with pytest.raises(szx.SZxError) as ei:
        szx.dump_host(torch.from_numpy(x).cuda(), 1e-3, "rel", 128, 4, out=small)
    assert ei.value.code == -2
