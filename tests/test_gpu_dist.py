"""GPU tests of the sharded path through the C ABI (szx_local_range +
szx_compress_shard_async), emulating P ranks in one process: the range keys
are MIN-reduced exactly as the NCCL all-reduce does, and the P shard streams
are assembled into an SZXC container that must be byte-identical to the
oracle's P-shard container and decode on one GPU (8 -> 1 cross-decode)."""
from __future__ import annotations

import ctypes

import numpy as np
import pytest
import torch

import oracle
import synth

pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("needs a CUDA device", allow_module_level=True)

import paper_conf_hpdc_yudztt0c22_b200 as szx  # noqa: E402
from paper_conf_hpdc_yudztt0c22_b200 import dist as sdist  # noqa: E402
from paper_conf_hpdc_yudztt0c22_b200 import szx as S  # noqa: E402


def _compress_sharded(x: torch.Tensor, P: int, eb: float, mode: str, b: int):
    L = S.lib()
    m = S._mode_code(mode)
    dt = S.F32 if x.dtype == torch.float32 else S.F64
    n = x.numel()
    st = torch.cuda.current_stream().cuda_stream
    shards = [sdist.shard_elems(n, b, P, p) for p in range(P)]
    wss, keys = [], []
    for first, cnt in shards:
        ws = torch.empty(max(S.workspace_bytes(cnt, dt, b), 16), dtype=torch.uint8, device="cuda")
        k = torch.empty(2, dtype=torch.int64, device="cuda")
        xs = x[first:first + cnt]
        S._check(L.szx_local_range(xs.data_ptr() if cnt else None, dt, cnt, b, k.data_ptr(), ws.data_ptr(),
                                   ws.numel(), st), "local_range")
        wss.append(ws)
        keys.append(k)
    # the NCCL all-reduce MIN over ranks (signed order after flipping bit 63)
    flip = torch.tensor(-(1 << 63), dtype=torch.int64, device="cuda")
    g = torch.stack([torch.bitwise_xor(k, flip) for k in keys]).min(dim=0).values
    g = torch.bitwise_xor(g, flip)
    streams = []
    for (first, cnt), ws in zip(shards, wss):
        cap = S.compress_bound(cnt, dt, b)
        out = torch.empty(cap, dtype=torch.uint8, device="cuda")
        tot = torch.zeros(1, dtype=torch.int64, device="cuda")
        xs = x[first:first + cnt]
        S._check(L.szx_compress_shard_async(xs.data_ptr() if cnt else None, dt, cnt, m, float(eb),
                                            ctypes.c_void_p(g.data_ptr()), b, out.data_ptr(), cap, ws.data_ptr(),
                                            ws.numel(), tot.data_ptr(), st), "compress_shard")
        streams.append(out[: int(tot.item())])
    return sdist.build_container(streams, [c for _, c in shards])


@pytest.mark.parametrize("P", [1, 2, 3, 8])
@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("mode", ["rel", "abs"])
def test_sharded_container_matches_oracle(P, dt, mode):
    x = synth.random_mix(300_007, 99).numpy().astype(dt)
    eb = 1e-3
    c = _compress_sharded(torch.from_numpy(x).cuda(), P, eb, mode, 128).cpu().numpy()
    ref = oracle.container_compress(x, eb, oracle.REL if mode == "rel" else oracle.ABS, 128, P)
    assert c.tobytes() == ref.tobytes()
    # P -> 1 cross-decode on one GPU
    y = szx.decompress(torch.from_numpy(c).cuda()).cpu().numpy()
    ui = np.uint32 if dt == np.float32 else np.uint64
    assert np.array_equal(y.view(ui), oracle.decompress(ref).view(ui))


def test_sharded_special_values_and_empty_shards():
    x = synth.special_values(1000, 3).numpy()  # 8 blocks, 16 shards -> empty shards
    c = _compress_sharded(torch.from_numpy(x).cuda(), 16, 1e-2, "rel", 128).cpu().numpy()
    ref = oracle.container_compress(x, 1e-2, oracle.REL, 128, 16)
    assert c.tobytes() == ref.tobytes()
    y = szx.decompress(torch.from_numpy(c).cuda()).cpu().numpy()
    assert np.array_equal(y.view(np.uint32), oracle.decompress(ref).view(np.uint32))


def test_sharded_compressor_single_rank_matches_plain_stream():
    x = synth.nyx_like(1, n=64).reshape(-1).cuda()
    sc = sdist.ShardedCompressor(x.numel(), torch.float32, 128)
    sc.compress(x, 1e-3, "rel")
    s = sc.stream()
    assert torch.equal(s, szx.compress(x, 1e-3, "rel", 128))
    c = sdist.gather_container(sc)
    ref = oracle.container_compress(x.cpu().numpy(), 1e-3, oracle.REL, 128, 1)
    assert c.cpu().numpy().tobytes() == ref.tobytes()
