"""Multi-process (world_size 2, gloo, CPU) tests of the sharding plumbing in
paper_conf_hpdc_yudztt0c22_b200/dist.py: block-range partition, the all-reduce of
the REL range keys, the all-gather of shard records and the SZXC container.
The per-shard codec here is the CPU oracle (test infrastructure); on GPUs the
same functions run over NCCL with the CUDA codec (tests/test_gpu_dist.py)."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_hpdc_yudztt0c22_b200 import dist as sdist


def _free_port() -> int:
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _dkey(d: float) -> int:
    """Order-preserving uint64 key of a double (total order) -- the C ABI's szx_local_range."""
    b = int(np.float64(d).view(np.uint64))
    return (~b & 0xFFFFFFFFFFFFFFFF) if b >> 63 else (b | (1 << 63))


def _dkey_inv(k: int) -> float:
    b = (k & 0x7FFFFFFFFFFFFFFF) if k >> 63 else (~k & 0xFFFFFFFFFFFFFFFF)
    return float(np.uint64(b).view(np.float64))


def _as_i64(u: int) -> int:
    return u - (1 << 64) if u >= (1 << 63) else u


def _local_keys(x: np.ndarray) -> torch.Tensor:
    fin = x[np.isfinite(x)].astype(np.float64)
    if fin.size == 0:
        return torch.tensor([-1, -1], dtype=torch.int64)  # 0xFF..FF
    return torch.tensor([_as_i64(_dkey(fin.min())), _as_i64(~_dkey(fin.max()) & 0xFFFFFFFFFFFFFFFF)],
                        dtype=torch.int64)


def _worker(rank, world, port, n, b, rel, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        x = synth.random_mix(n, 4242).numpy()
        first, cnt = sdist.shard_elems(n, b, world, rank)
        xs = x[first:first + cnt]
        keys = sdist.allreduce_range_keys(_local_keys(xs))
        k0, k1 = (int(v) & 0xFFFFFFFFFFFFFFFF for v in keys.tolist())
        if k0 == 0xFFFFFFFFFFFFFFFF:
            e = 0.0
        else:
            e = rel * (_dkey_inv(~k1 & 0xFFFFFFFFFFFFFFFF) - _dkey_inv(k0))
        e = e + 0.0
        s = torch.from_numpy(oracle.compress_shard(xs, rel, e, oracle.REL, b))
        recs = sdist.allgather_records(cnt, torch.tensor([s.numel()], dtype=torch.int64))
        c = sdist.gather_streams(s, recs, dst=0)
        if rank == 0:
            q.put(("container", c.numpy().tobytes(), e))
        else:
            q.put(("ok", None, e))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("n,b", [(100_003, 128), (64 * 256 * 3 + 7, 256), (300, 128)])
def test_two_rank_container_matches_oracle(n, b):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, n, b, 1e-3, q)) for r in range(2)]
    for p in procs:
        p.start()
    try:
        res = [q.get(timeout=120) for _ in procs]
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    assert all(p.exitcode == 0 for p in procs)
    c = [r for r in res if r[0] == "container"][0][1]
    x = synth.random_mix(n, 4242).numpy()
    ref = oracle.container_compress(x, 1e-3, oracle.REL, b, 2)
    assert c == ref.tobytes()
    # both ranks agreed on the global bound, equal to the whole array's REL bound
    assert all(r[2] == oracle.eb_abs(x, 1e-3, oracle.REL) for r in res)
    y = oracle.decompress(np.frombuffer(c, np.uint8))
    assert np.array_equal(y.view(np.uint32), oracle.decompress(oracle.container_compress(x, 1e-3, oracle.REL, b, 2)).view(np.uint32))


def test_shard_partition_is_block_aligned_and_complete():
    for n in (0, 1, 127, 128, 129, 10_000, 1_234_567):
        for b in (128, 256):
            nB = (n + b - 1) // b
            for P in (1, 2, 3, 8):
                prev = 0
                for p in range(P):
                    f, c = sdist.shard_elems(n, b, P, p)
                    assert f == prev and f % b == 0
                    prev = f + c
                    b0, b1 = sdist.shard_blocks(nB, P, p)
                    assert f == b0 * b
                assert prev == n


def test_container_layout_closed_form():
    n_elems = [10, 0, 7, 5]
    nbytes = [101, 64, 90, 77]
    firsts, offs, total = sdist.container_layout(n_elems, nbytes)
    assert firsts == [0, 10, 10, 17]
    assert all(o % 16 == 0 for o in offs)
    assert offs[0] == 32 + 32 * 4
    # container bytes = 32 + 32P + sum_{p<P-1} al16(S_p) + S_{P-1}  (DESIGN.md s.4)
    assert total == 32 + 32 * 4 + sum((s + 15) // 16 * 16 for s in nbytes[:-1]) + nbytes[-1]


class _OracleShardCodec:
    """The CPU oracle as the per-shard codec of dist.dump / dist.load (test infrastructure)."""

    def local_minmax(self, x):
        f = x[np.isfinite(x)].astype(np.float64)
        return (float(f.min()), float(f.max())) if f.size else (float("inf"), float("-inf"))

    def compress(self, x, eb, eb_abs, mode, b):
        return oracle.compress_shard(x, eb, eb_abs, oracle.REL if mode == "rel" else oracle.ABS, b)

    def read(self, fd, off, nb):
        return np.frombuffer(os.pread(fd, nb, off), np.uint8)

    def decompress(self, s):
        return oracle.decompress(s)


def _dump_worker(rank, world, port, n, b, rel, path, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        x = synth.random_mix(n, 777).numpy()
        first, cnt = sdist.shard_elems(n, b, world, rank)
        total = sdist.dump(x[first:first + cnt], rel, path, "rel", b, codec=_OracleShardCodec())
        f2, y = sdist.load(path, codec=_OracleShardCodec())
        fo, yo = sdist.load(path, part=world - 1 - rank, codec=_OracleShardCodec())
        q.put((rank, total, f2, y.tobytes(), fo, yo.tobytes()))
    finally:
        dist.destroy_process_group()


def test_two_rank_dump_load_container_file(tmp_path):
    """two ranks dump their shards into one SZXC file (global REL bound by
    all-reduce, offsets by all-gather); the file is byte-identical to the oracle's 2-shard
    container, and each rank loads its own and the other rank's shard bit-exactly."""
    n, b, rel = 70_001, 128, 1e-3
    path = str(tmp_path / "dump.szxc")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_dump_worker, args=(r, 2, port, n, b, rel, path, q)) for r in range(2)]
    for p in procs:
        p.start()
    try:
        res = sorted(q.get(timeout=120) for _ in procs)
    finally:
        for p in procs:
            p.join(timeout=30)
            if p.is_alive():
                p.kill()
    assert all(p.exitcode == 0 for p in procs)
    x = synth.random_mix(n, 777).numpy()
    ref = oracle.container_compress(x, rel, oracle.REL, b, 2)
    data = open(path, "rb").read()
    assert data == ref.tobytes() and all(r[1] == len(data) for r in res)
    y = oracle.decompress(ref)
    for rank, _, f2, yb, fo, yob in res:
        first, cnt = sdist.shard_elems(n, b, 2, rank)
        assert f2 == first and yb == y[first:first + cnt].tobytes()
        fo_, co = sdist.shard_elems(n, b, 2, 1 - rank)
        assert fo == fo_ and yob == y[fo_:fo_ + co].tobytes()
