"""Multi-GPU SZx: one process per GPU, the array sharded by contiguous block ranges.

The paper's compressor has no collective (blocks are independent, P:L2340-2342,
P:L2393-2396); the only couplings of a sharded array are
  (i)  the value-range-relative bound, which is GLOBAL (footnote 1):
       an all-reduce MIN of two 8-byte order-preserving keys;
  (ii) the container header: an all-gather of each shard's (n_elem, bytes) so
       every rank knows every shard's offset in the SZXC container.
Shard p of P owns blocks [floor(p nB / P), floor((p+1) nB / P)) (DESIGN.md s.8),
so a container written on P GPUs decodes on one GPU and vice versa.

torch.distributed (NCCL on GPUs, gloo in the CPU tests) is the plumbing; the
codec itself is the C ABI (szx_local_range + szx_compress_shard_async).
"""
from __future__ import annotations

import ctypes
import os
import struct

import torch
import torch.distributed as dist

CONTAINER_HEAD = 32
CONTAINER_ENTRY = 32
_FLIP = -(1 << 63)  # bit 63 as int64: maps unsigned key order to signed order


def al16(x: int) -> int:
    return (x + 15) // 16 * 16


def shard_blocks(nB: int, P: int, p: int) -> tuple[int, int]:
    return nB * p // P, nB * (p + 1) // P


def shard_elems(n: int, b: int, P: int, p: int) -> tuple[int, int]:
    """(first element, element count) of shard p."""
    nB = (n + b - 1) // b
    b0, b1 = shard_blocks(nB, P, p)
    e0, e1 = b0 * b, min(n, b1 * b)
    return e0, max(0, e1 - e0)


def allreduce_range_keys(keys: torch.Tensor, group=None, force: bool = False) -> torch.Tensor:
    """Element-wise MIN of [key(min), ~key(max)] (uint64 bit patterns held in int64) over ranks."""
    if group is None and not (dist.is_available() and dist.is_initialized()):
        return keys
    if dist.get_world_size(group) == 1 and not force:
        return keys
    k = torch.bitwise_xor(keys, torch.full_like(keys, _FLIP))
    dist.all_reduce(k, op=dist.ReduceOp.MIN, group=group)
    return torch.bitwise_xor(k, torch.full_like(k, _FLIP))


def container_layout(n_elems: list[int], nbytes: list[int]):
    """Offsets (16-aligned) of each shard stream inside the SZXC container and its total size."""
    P = len(n_elems)
    pos = CONTAINER_HEAD + CONTAINER_ENTRY * P
    offs, firsts = [], []
    first = 0
    for p in range(P):
        pos = al16(pos)
        offs.append(pos)
        firsts.append(first)
        pos += nbytes[p]
        first += n_elems[p]
    return firsts, offs, pos


def container_header(n_elems: list[int], nbytes: list[int]) -> bytes:
    P = len(n_elems)
    firsts, offs, _ = container_layout(n_elems, nbytes)
    head = bytearray(CONTAINER_HEAD + CONTAINER_ENTRY * P)
    head[0:4] = b"SZXC"
    struct.pack_into("<IIIQQ", head, 4, 1, P, 0, sum(n_elems), 0)
    for p in range(P):
        struct.pack_into("<QQQQ", head, CONTAINER_HEAD + CONTAINER_ENTRY * p, firsts[p], n_elems[p], offs[p],
                         nbytes[p])
    return bytes(head)


def build_container(streams: list[torch.Tensor], n_elems: list[int]) -> torch.Tensor:
    """Concatenate P shard streams (uint8 tensors, any device) into one SZXC container."""
    nbytes = [int(s.numel()) for s in streams]
    _, offs, total = container_layout(n_elems, nbytes)
    dev = streams[0].device if streams else torch.device("cpu")
    out = torch.zeros(total, dtype=torch.uint8, device=dev)
    head = torch.frombuffer(bytearray(container_header(n_elems, nbytes)), dtype=torch.uint8)
    out[:head.numel()] = head.to(dev)
    for s, o in zip(streams, offs):
        out[o:o + s.numel()] = s.to(dev)
    return out


class ShardedCompressor:
    """Compress this rank's shard of a global array into a standalone SZX1 stream.

    compress() enqueues, without host synchronisation:
      szx_local_range (block statistics + local finite range, one read of the shard)
      -> all-reduce MIN of the 16-byte range keys (REL only)
      -> szx_compress_shard_async (classify + encode with the GLOBAL bound)
      -> all-gather of (n_elem, stream bytes) so every rank knows the container offsets.
    """

    def __init__(self, n_local: int, dtype=torch.float32, block_size: int = 128, device="cuda", group=None,
                 force_collectives: bool = False):
        from . import szx as _szx
        self._szx = _szx
        self.n, self.b, self.group = n_local, block_size, group
        self.dtype = dtype
        self.dt = _szx.F32 if dtype == torch.float32 else _szx.F64
        self.cap = _szx.compress_bound(n_local, self.dt, block_size)
        self.out = torch.empty(self.cap, dtype=torch.uint8, device=device)
        self.ws = torch.empty(max(_szx.workspace_bytes(n_local, self.dt, block_size), 16), dtype=torch.uint8,
                              device=device)
        self.keys = torch.empty(2, dtype=torch.int64, device=device)
        self.total = torch.zeros(1, dtype=torch.int64, device=device)
        self.rec = torch.zeros(2, dtype=torch.int64, device=device)
        self.rec[0] = n_local  # (constant: set once, so the compress sequence has no host-to-device copy)
        ws = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
        self.world = ws
        # run the collectives even on a 1-rank group (the bench's torchrun --nproc-per-node 1 path
        # exercises the same NCCL calls, captured in the step's CUDA graph, as N > 1)
        self.collectives = ws > 1 or (force_collectives and dist.is_available() and dist.is_initialized())
        self.records = torch.zeros(ws * 2, dtype=torch.int64, device=device)

    def compress(self, x: torch.Tensor, eb: float, mode="rel", stream=None):
        """Enqueue the shard's compression on `stream` (default: the current stream).

        Every step -- the two C-ABI calls, the key and record copies and both
        collectives -- is issued on that one stream (torch's collectives run on
        the current stream's order for NCCL), so the all-reduce reads the local
        keys after szx_local_range wrote them, the encoder reads the global keys
        after the all-reduce, and the record all-gather reads the stream length
        after the encoder wrote it."""
        if stream is not None and x.is_cuda:
            with torch.cuda.stream(stream):
                return self._compress(x, eb, mode)
        return self._compress(x, eb, mode)

    def _compress(self, x: torch.Tensor, eb: float, mode):
        L = self._szx.lib()
        m = self._szx._mode_code(mode)
        st = self._szx._stream(None)
        assert x.is_contiguous() and x.numel() == self.n and x.dtype == self.dtype
        xp = x.data_ptr() if self.n else None
        self._szx._check(L.szx_local_range(xp, self.dt, self.n, self.b, self.keys.data_ptr(), self.ws.data_ptr(),
                                           self.ws.numel(), st), "szx_local_range")
        if m == self._szx.REL and self.collectives:
            self.keys.copy_(allreduce_range_keys(self.keys, self.group, force=True))
        self._szx._check(L.szx_compress_shard_async(xp, self.dt, self.n, m, float(eb),
                                                    ctypes.c_void_p(self.keys.data_ptr()), self.b,
                                                    self.out.data_ptr(), self.cap, self.ws.data_ptr(),
                                                    self.ws.numel(), self.total.data_ptr(), st),
                         "szx_compress_shard_async")
        self.rec[1:2].copy_(self.total)
        if self.collectives:
            dist.all_gather_into_tensor(self.records, self.rec, group=self.group)
        else:
            self.records.copy_(self.rec)

    def stream(self) -> torch.Tensor:
        """This rank's stream (synchronises to read its length)."""
        return self.out[: int(self.total.item())]

    def container_offsets(self):
        """(firsts, offsets, total container bytes) from the all-gathered records (host sync)."""
        r = self.records.view(-1, 2).cpu().tolist()
        return container_layout([int(a) for a, _ in r], [int(bb) for _, bb in r])


def allgather_records(n_elem: int, nbytes: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather of each rank's (n_elem, stream bytes) record -> [P, 2] int64 (same device)."""
    rec = torch.stack([torch.full_like(nbytes.view(-1)[:1], n_elem).view(()), nbytes.view(-1)[0]]).to(torch.int64)
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size(group) == 1:
        return rec.view(1, 2)
    out = torch.empty(dist.get_world_size(group) * 2, dtype=torch.int64, device=rec.device)
    dist.all_gather_into_tensor(out, rec.contiguous(), group=group)
    return out.view(-1, 2)


def gather_streams(stream: torch.Tensor, records: torch.Tensor, dst: int = 0, group=None) -> torch.Tensor | None:
    """Collect every rank's stream on rank dst and build the SZXC container there
    (records = allgather_records output).  Works for NCCL (CUDA) and gloo (CPU)."""
    r = records.cpu().tolist()
    n_elems = [int(a) for a, _ in r]
    nbytes = [int(bb) for _, bb in r]
    world = len(r)
    if world == 1:
        return build_container([stream], n_elems)
    mx = max(nbytes)
    pad = torch.zeros(mx, dtype=torch.uint8, device=stream.device)
    pad[: stream.numel()] = stream
    rank = dist.get_rank(group)
    bufs = [torch.empty(mx, dtype=torch.uint8, device=stream.device) for _ in range(world)] if rank == dst else None
    dist.gather(pad, bufs, dst=dst, group=group)
    if rank != dst:
        return None
    return build_container([b[:nb] for b, nb in zip(bufs, nbytes)], n_elems)


def gather_container(sc: ShardedCompressor, dst: int = 0, group=None) -> torch.Tensor | None:
    """Collect every rank's stream on rank dst and build the SZXC container there."""
    return gather_streams(sc.stream(), sc.records.view(-1, 2), dst, group)


def decompress_local(stream: torch.Tensor, n: int, block_size: int, group=None) -> tuple[int, torch.Tensor]:
    """1 stream -> Q GPUs: this rank reconstructs the block range it would own as
    shard `rank` of `world` (shard_blocks), from a stream or container held on its device.
    No collective: each rank reads the bitmap/zsize prefix it needs and decodes its tiles.
    Returns (first element, values)."""
    from . import szx as _szx
    world = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
    rank = dist.get_rank(group) if world > 1 else 0
    nB = (n + block_size - 1) // block_size
    b0, b1 = shard_blocks(nB, world, rank)
    return b0 * block_size, _szx.decompress_blocks(stream, b0, b1 - b0)


# --------------------------------------------------------------------------- dump / load
# SURVEY 8(f) row 3 (the paper's data dumping / loading experiment, Fig. 16) on one
# box: every rank compresses its block-range shard of a global array with the GLOBAL REL bound and
# writes its stream into ONE SZXC container file at the offset the all-gathered stream sizes give
# (rank 0 writes the header and shard table); loading reads a rank's shard (or any shard) back.
# The per-shard codec is pluggable: CudaShardCodec (this library, the product path) or any object
# with the same three methods (the CPU oracle in the gloo tests).

class CudaShardCodec:
    """Per-shard codec over the C ABI: szx_local_minmax, szx_compress_shard (device-held global
    bound) and szx_decompress; streams are copied to pinned host memory in chunks so the D2H
    copy of chunk i+1 overlaps the file write of chunk i."""

    def __init__(self, device="cuda"):
        from . import szx as _szx
        self._szx = _szx
        self.device = torch.device(device)

    def local_minmax(self, x: torch.Tensor):
        return self._szx.local_minmax(x).cpu().tolist() if x.numel() else [float("inf"), float("-inf")]

    def compress(self, x: torch.Tensor, eb: float, eb_abs: float, mode: str, block_size: int) -> torch.Tensor:
        e = torch.tensor([eb_abs], dtype=torch.float64, device=x.device)
        return self._szx.compress_shard(x, eb, e, mode, block_size)

    def write(self, fd: int, stream: torch.Tensor, offset: int, chunk: int = 64 << 20) -> None:
        n = stream.numel()
        if n == 0:
            return
        bufs = [torch.empty(min(chunk, n), dtype=torch.uint8, pin_memory=True) for _ in range(2)]
        evs = [torch.cuda.Event() for _ in range(2)]
        cs = torch.cuda.Stream(device=stream.device)
        cs.wait_stream(torch.cuda.current_stream(stream.device))
        pos, i = 0, 0
        pend = None
        while pos < n or pend is not None:
            if pos < n:
                m = min(chunk, n - pos)
                with torch.cuda.stream(cs):
                    bufs[i % 2][:m].copy_(stream[pos:pos + m], non_blocking=True)
                    evs[i % 2].record(cs)
                cur = (i % 2, pos, m)
                pos += m
                i += 1
            else:
                cur = None
            if pend is not None:  # write the previous chunk while this one copies
                j, p0, m0 = pend
                evs[j].synchronize()
                os.pwrite(fd, memoryview(bufs[j][:m0].numpy()), offset + p0)
            pend = cur

    def read(self, fd: int, offset: int, nbytes: int) -> torch.Tensor:
        host = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
        got = os.preadv(fd, [memoryview(host.numpy())], offset) if nbytes else 0
        if got != nbytes:
            raise IOError(f"short read {got} of {nbytes}")
        return host.to(self.device, non_blocking=True)

    def decompress(self, stream: torch.Tensor) -> torch.Tensor:
        return self._szx.decompress(stream)


def _rel_bound(rel: float, gmin: float, gmax: float) -> float:
    """REL x (gmax - gmin) in double over the finite values (reading R13); canonical +0."""
    if not (gmin <= gmax):  # no finite value anywhere
        return 0.0
    e = rel * (gmax - gmin)
    return e if e != 0.0 else 0.0


def dump(x_local, eb: float, path: str, mode: str = "rel", block_size: int = 128, codec=None, group=None):
    """Write this rank's shard into the SZXC container at `path` (all ranks call it collectively;
    x_local is shard `rank` of `world`, shard_elems layout).  Returns the container bytes."""
    import numpy as np
    codec = codec or CudaShardCodec()
    world = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
    rank = dist.get_rank(group) if world > 1 else 0
    n_local = int(x_local.numel() if hasattr(x_local, "numel") else len(x_local))
    # (i) the global finite range (REL): MIN of the minima, MAX of the maxima
    mn, mx = codec.local_minmax(x_local)
    if world > 1:
        t = torch.tensor([mn, -mx], dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MIN, group=group)
        mn, mx = float(t[0]), -float(t[1])
    eb_abs = _rel_bound(eb, mn, mx) if mode in ("rel", "REL") else float(eb)
    s = codec.compress(x_local, eb, eb_abs, mode, block_size)
    nbytes = int(s.numel() if hasattr(s, "numel") else len(s))
    # (ii) the container offsets: all-gather of (n_elem, stream bytes)
    rec = torch.tensor([n_local, nbytes], dtype=torch.int64)
    if world > 1:
        recs = [torch.zeros(2, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(recs, rec, group=group)
    else:
        recs = [rec]
    n_elems = [int(r[0]) for r in recs]
    sizes = [int(r[1]) for r in recs]
    _, offs, total = container_layout(n_elems, sizes)
    if rank == 0:
        fd = os.open(path, os.O_CREAT | os.O_RDWR | os.O_TRUNC, 0o644)
        os.ftruncate(fd, total)
        head = container_header(n_elems, sizes)
        os.pwrite(fd, head, 0)
        os.close(fd)
    if world > 1:
        dist.barrier(group=group)
    fd = os.open(path, os.O_RDWR)
    try:
        if isinstance(s, torch.Tensor) and s.is_cuda:
            codec.write(fd, s, offs[rank])
        else:
            os.pwrite(fd, np.ascontiguousarray(s, np.uint8).tobytes(), offs[rank])
        os.fsync(fd) if os.environ.get("SZX_DUMP_FSYNC") else None
    finally:
        os.close(fd)
    if world > 1:
        dist.barrier(group=group)
    return total


def load(path: str, part: int | None = None, codec=None, group=None):
    """Read shard `part` (default: this rank's) of the SZXC container at `path` and decode it.
    Returns (first element, values)."""
    codec = codec or CudaShardCodec()
    world = dist.get_world_size(group) if dist.is_available() and dist.is_initialized() else 1
    rank = dist.get_rank(group) if world > 1 else 0
    p = rank if part is None else part
    fd = os.open(path, os.O_RDONLY)
    try:
        head = os.pread(fd, CONTAINER_HEAD, 0)
        if head[:4] != b"SZXC":
            raise ValueError("not an SZXC container")
        ver, P = struct.unpack_from("<II", head, 4)
        if ver != 1 or not (0 <= p < P):
            raise ValueError("bad container header or shard index")
        first, n_el, off, nb = struct.unpack("<QQQQ", os.pread(fd, CONTAINER_ENTRY, CONTAINER_HEAD + CONTAINER_ENTRY * p))
        s = codec.read(fd, off, nb)
    finally:
        os.close(fd)
    return first, codec.decompress(s)
