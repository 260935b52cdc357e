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


@pytest.mark.parametrize("b", [32, 64, 256])
def test_sharded_container_small_and_large_blocks(b):
    x = synth.random_mix(300_007, 41).numpy()
    c = _compress_sharded(torch.from_numpy(x).cuda(), 5, 1e-3, "rel", b).cpu().numpy()
    ref = oracle.container_compress(x, 1e-3, oracle.REL, b, 5)
    assert c.tobytes() == ref.tobytes()


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


def _blocks_ref(yref: np.ndarray, b: int, k0: int, nb: int) -> np.ndarray:
    n = yref.size
    nB = (n + b - 1) // b
    e0 = min(k0, nB) * b
    e1 = min(n, min(nB, k0 + nb) * b)
    return yref[e0:max(e0, e1)]


@pytest.mark.parametrize("dt", [np.float32, np.float64])
@pytest.mark.parametrize("b", [32, 64, 128, 256])
def test_decompress_blocks_matches_oracle_slices(dt, b):
    """1 stream -> Q GPUs: any block range of a stream decodes to the same slice of the oracle's
    reconstruction, bit for bit (ranges inside one tile, across tiles, unaligned, the tail, empty,
    clipped at the end)."""
    x = synth.random_mix(300_007, 7).numpy().astype(dt)  # ragged tail block
    ref = oracle.compress(x, 1e-3, oracle.REL, b)
    yref = oracle.decompress(ref)
    s = torch.from_numpy(ref).cuda()
    nB = (x.size + b - 1) // b
    ui = np.uint32 if dt == np.float32 else np.uint64
    ranges = [(0, nB), (0, 1), (5, 3), (31, 2), (32, 32), (33, 100), (nB - 1, 1), (nB - 40, 1000),
              (100, 0), (nB, 5), (nB + 3, 1), (7, nB)]
    for k0, nb in ranges:
        got = szx.decompress_blocks(s, k0, nb).cpu().numpy()
        exp = _blocks_ref(yref, b, k0, nb)
        assert got.size == exp.size, (k0, nb)
        assert np.array_equal(got.view(ui), exp.view(ui)), (k0, nb)


@pytest.mark.parametrize("Q", [2, 3, 8])
def test_one_stream_to_q_ranks(Q):
    """A stream written on 1 GPU, decoded by Q ranks (emulated): each rank's block range
    (shard_blocks) concatenates to the full reconstruction."""
    x = synth.nyx_like(0, n=96).reshape(-1).contiguous()
    ref = oracle.compress(x.numpy(), 1e-3, oracle.REL, 128)
    yref = oracle.decompress(ref)
    s = torch.from_numpy(ref).cuda()
    nB = (x.numel() + 127) // 128
    parts = []
    for q in range(Q):
        b0, b1 = sdist.shard_blocks(nB, Q, q)
        parts.append(szx.decompress_blocks(s, b0, b1 - b0).cpu().numpy())
    assert np.array_equal(np.concatenate(parts).view(np.uint32), yref.view(np.uint32))


@pytest.mark.parametrize("P,Q", [(8, 1), (8, 3), (3, 8), (2, 2)])
def test_container_block_ranges(P, Q):
    """A P-shard container decoded as Q block ranges with global block numbering
    (ranges straddle shard boundaries)."""
    x = synth.random_mix(200_003, 11).numpy()
    ref = oracle.container_compress(x, 1e-3, oracle.REL, 128, P)
    yref = oracle.decompress(ref)
    c = torch.from_numpy(ref).cuda()
    nB = (x.size + 127) // 128
    parts = []
    for q in range(Q):
        b0, b1 = sdist.shard_blocks(nB, Q, q)
        parts.append(szx.decompress_blocks(c, b0, b1 - b0).cpu().numpy())
    assert np.array_equal(np.concatenate(parts).view(np.uint32), yref.view(np.uint32))
    got = szx.decompress_blocks(c, 17, 777).cpu().numpy()
    assert np.array_equal(got.view(np.uint32), _blocks_ref(yref, 128, 17, 777).view(np.uint32))


def test_decompress_blocks_errors():
    x = synth.random_mix(10_000, 5).numpy()
    ref = oracle.compress(x, 1e-3, oracle.REL, 128)
    s = torch.from_numpy(ref).cuda()
    small = torch.empty(10, dtype=torch.float32, device="cuda")
    with pytest.raises(S.SZxError) as e:
        szx.decompress_blocks(s, 0, 5, out=small)
    assert e.value.code == -2  # ENOSPC
    bad = s.clone()
    bad[0] = 0
    with pytest.raises(S.SZxError) as e:
        szx.decompress_blocks(bad, 0, 5)
    assert e.value.code == -3  # ECORRUPT


@pytest.mark.parametrize("dt", [np.float32, np.float64])
def test_minmax_and_compress_shard_double_forms(dt):
    """SURVEY 8(b)'s double-valued boundary: szx_local_minmax of every shard, the MIN/MAX combine an
    all-reduce would do, eb_abs = REL x (max - min) in double (footnote 1), then the
    blocking szx_compress_shard with that device-held bound: each shard stream is byte-identical to
    the oracle's shard stream with the oracle's global bound."""
    x = synth.special_values(200_003, 17, dtype=torch.float32 if dt == np.float32 else torch.float64).cuda()
    n, P, b, rel = x.numel(), 3, 128, 1e-3
    parts = [sdist.shard_elems(n, b, P, p) for p in range(P)]
    mms = [szx.local_minmax(x[f:f + c]) for f, c in parts]
    gmin = torch.stack([m[0] for m in mms]).min()
    gmax = torch.stack([m[1] for m in mms]).max()
    xn = x.cpu().numpy()
    fin = xn[np.isfinite(xn)]
    assert gmin.item() == float(fin.min()) and gmax.item() == float(fin.max())
    e_ref = oracle.eb_abs(xn, rel, oracle.REL)
    eb_abs = (rel * (gmax - gmin)).reshape(1).contiguous()
    assert eb_abs.item() == e_ref
    for f, c in parts:
        got = szx.compress_shard(x[f:f + c], rel, eb_abs, "rel", b).cpu().numpy()
        ref = oracle.compress_shard(xn[f:f + c], rel, e_ref, oracle.REL, b)
        assert got.tobytes() == ref.tobytes(), (f, c)
    # a shard without finite values
    nan = torch.full((300,), float("nan"), dtype=x.dtype, device="cuda")
    mm = szx.local_minmax(nan).cpu().tolist()
    assert mm[0] == float("inf") and mm[1] == float("-inf")
