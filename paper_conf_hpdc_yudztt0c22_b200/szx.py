"""Thin ctypes binding of libszx_b200.so (include/szx.h).

Argument marshalling only: every step of compression and decompression runs
in the sm_100a kernels behind the C ABI.  torch provides device memory
(``data_ptr``) and streams (``cuda_stream``).  There is no CPU fallback: if
the library or a CUDA device is missing, every call raises.
"""
from __future__ import annotations

import ctypes
import math
import os
import struct
from dataclasses import dataclass

import torch

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("SZX_LIB", os.path.join(_PKG, "libszx_b200.so"))  # SZX_LIB: experiment builds

F32, F64 = 0, 1
ABS, REL = 0, 1
_ERR = {0: "ok", -1: "EINVAL", -2: "ENOSPC", -3: "ECORRUPT", -4: "ECUDA", -5: "ENOMEM"}


class SZxError(RuntimeError):
    def __init__(self, code: int, what: str):
        super().__init__(f"{what}: {_ERR.get(code, code)} ({code})")
        self.code = code


class _Header(ctypes.Structure):
    _fields_ = [("version", ctypes.c_uint32), ("dtype", ctypes.c_uint32), ("eb_mode", ctypes.c_uint32),
                ("block_size", ctypes.c_uint32), ("n", ctypes.c_uint64), ("eb_user", ctypes.c_double),
                ("eb_abs", ctypes.c_double), ("n_nonconst", ctypes.c_uint64),
                ("payload_bytes", ctypes.c_uint64), ("stream_bytes", ctypes.c_uint64)]


_lib = None


def lib() -> ctypes.CDLL:
    """Load the in-tree CUDA library (fails loudly if it was not built)."""
    global _lib
    if _lib is not None:
        return _lib
    if not os.path.exists(LIB_PATH):
        raise RuntimeError(f"{LIB_PATH} missing: run `python -c 'import __graft_entry__ as g; g.build()'`")
    L = ctypes.CDLL(LIB_PATH)
    u64, i64, i32, vp, dbl, u32 = (ctypes.c_uint64, ctypes.c_int64, ctypes.c_int, ctypes.c_void_p,
                                   ctypes.c_double, ctypes.c_uint32)
    sig = {
        "szx_compress_bound": (u64, [u64, i32, u32]),
        "szx_compress_workspace_bytes": (u64, [u64, i32, u32]),
        "szx_decompress_workspace_bytes": (u64, [ctypes.POINTER(_Header)]),
        "szx_compress": (i64, [vp, i32, u64, i32, dbl, u32, vp, u64, vp]),
        "szx_compress_ws": (i64, [vp, i32, u64, i32, dbl, u32, vp, u64, vp, u64, vp]),
        "szx_compress_async": (i32, [vp, i32, u64, i32, dbl, u32, vp, u64, vp, u64, vp, vp]),
        "szx_read_header": (i32, [vp, u64, ctypes.POINTER(_Header)]),
        "szx_decompress": (i64, [vp, u64, vp, u64, vp]),
        "szx_decompress_blocks": (i64, [vp, u64, u64, u64, vp, u64, vp]),
        "szx_decompress_ws": (i64, [vp, u64, vp, u64, vp, u64, vp]),
        "szx_decompress_async": (i32, [vp, u64, ctypes.POINTER(_Header), vp, u64, vp, u64, vp, vp]),
        "szx_compress_host": (i64, [vp, i32, u64, i32, dbl, u32, vp, u64, vp]),
        "szx_decompress_host": (i64, [vp, u64, vp, u64, vp]),
        "szx_decompress_quality": (i64, [vp, u64, vp, vp, u64, vp, vp]),
        "szx_decompress_quality_async": (i32, [vp, u64, ctypes.POINTER(_Header), vp, vp, u64, vp, u64, vp, vp,
                                               vp]),
        "szx_quality_finish": (None, [vp, vp]),
        "szx_dump_host": (i64, [vp, i32, u64, i32, dbl, u32, u32, vp, u64, vp]),
        "szx_load_host": (i64, [vp, u64, vp, u64, vp]),
        "szx_local_range": (i32, [vp, i32, u64, u32, vp, vp, u64, vp]),
        "szx_compress_shard_async": (i32, [vp, i32, u64, i32, dbl, vp, u32, vp, u64, vp, u64, vp, vp]),
        "szx_local_minmax": (i32, [vp, i32, u64, vp, vp]),
        "szx_compress_shard": (i64, [vp, i32, u64, i32, dbl, vp, u32, vp, u64, vp]),
        "szx_timing_enable": (None, [i32]),
        "szx_timing_reset": (None, []),
        "szx_timing_read": (i32, [ctypes.POINTER(ctypes.c_char_p), ctypes.POINTER(dbl),
                                  ctypes.POINTER(u64), i32]),
        "szx_launch_count": (u64, []),
        "szx_debug_set_r_bias": (None, [i32]),
        "szx_strerror": (ctypes.c_char_p, [i32]),
    }
    for name, (res, args) in sig.items():
        if "SZX_LIB" in os.environ and not hasattr(L, name):
            continue  # an older experiment build (scripts/run_variants.sh) without this entry point
        f = getattr(L, name)
        f.restype = res
        f.argtypes = args
    _lib = L
    return L


EXPORTED = ["szx_compress_bound", "szx_compress_workspace_bytes", "szx_decompress_workspace_bytes",
            "szx_compress", "szx_compress_ws", "szx_compress_async", "szx_read_header",
            "szx_decompress", "szx_decompress_blocks", "szx_decompress_ws", "szx_decompress_async", "szx_compress_host",
            "szx_decompress_host", "szx_decompress_quality", "szx_decompress_quality_async",
            "szx_quality_finish", "szx_dump_host", "szx_load_host", "szx_local_range", "szx_compress_shard_async",
            "szx_local_minmax", "szx_compress_shard",
            "szx_timing_enable", "szx_timing_reset", "szx_timing_read", "szx_launch_count",
            "szx_debug_set_r_bias", "szx_strerror"]


def _check(rc: int, what: str) -> int:
    if rc < 0:
        raise SZxError(int(rc), what)
    return rc


def _dtype_code(t: torch.Tensor) -> int:
    if t.dtype == torch.float32:
        return F32
    if t.dtype == torch.float64:
        return F64
    raise TypeError(f"SZx compresses float32/float64 tensors, got {t.dtype}")


def _mode_code(mode) -> int:
    if mode in (REL, "rel", "REL"):
        return REL
    if mode in (ABS, "abs", "ABS"):
        return ABS
    raise ValueError(f"mode must be 'abs' or 'rel', got {mode!r}")


def _stream(stream=None) -> int:
    s = stream if stream is not None else torch.cuda.current_stream()
    return s.cuda_stream


def _require_cuda(t: torch.Tensor):
    if not t.is_cuda:
        raise ValueError("device tensor required (use compress_host for host buffers)")


def compress_bound(n: int, dtype_code: int, block_size: int = 128) -> int:
    return int(lib().szx_compress_bound(n, dtype_code, block_size))


def workspace_bytes(n: int, dtype_code: int, block_size: int = 128) -> int:
    return int(lib().szx_compress_workspace_bytes(n, dtype_code, block_size))


def compress(x: torch.Tensor, eb: float, mode="rel", block_size: int = 128, out: torch.Tensor | None = None,
             workspace: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Compress a CUDA float32/float64 tensor; returns the stream as a uint8 CUDA tensor."""
    _require_cuda(x)
    x = x.contiguous().view(-1)
    dt = _dtype_code(x)
    n = x.numel()
    cap = compress_bound(n, dt, block_size)
    if out is None:
        out = torch.empty(cap, dtype=torch.uint8, device=x.device)
    if workspace is None:
        workspace = torch.empty(max(workspace_bytes(n, dt, block_size), 16), dtype=torch.uint8, device=x.device)
    r = lib().szx_compress_ws(x.data_ptr() if n else None, dt, n, _mode_code(mode), float(eb), block_size,
                              out.data_ptr(), out.numel(), workspace.data_ptr(), workspace.numel(),
                              _stream(stream))
    _check(r, "szx_compress")
    return out[:r]


@dataclass
class Header:
    version: int
    dtype: int
    eb_mode: int
    block_size: int
    n: int
    eb_user: float
    eb_abs: float
    n_nonconst: int
    payload_bytes: int
    stream_bytes: int
    _c: _Header

    @property
    def torch_dtype(self):
        return torch.float32 if self.dtype == F32 else torch.float64


def read_header(b: bytes) -> Header:
    h = _Header()
    buf = ctypes.create_string_buffer(bytes(b[:64]), 64)
    _check(lib().szx_read_header(buf, len(b), ctypes.byref(h)), "szx_read_header")
    return Header(h.version, h.dtype, h.eb_mode, h.block_size, h.n, h.eb_user, h.eb_abs, h.n_nonconst,
                  h.payload_bytes, h.stream_bytes, h)


def _container_info(stream_t: torch.Tensor):
    head = stream_t[:64].cpu().numpy().tobytes()
    if head[:4] == b"SZXC":
        P = struct.unpack_from("<I", head, 8)[0]
        n = struct.unpack_from("<Q", head, 16)[0]
        off0 = struct.unpack_from("<Q", stream_t[32 + 16:32 + 24].cpu().numpy().tobytes())[0]
        dt = int(stream_t[off0 + 5].item())
        return n, dt
    h = read_header(head)
    return h.n, h.dtype


def _block_size(stream_t: torch.Tensor) -> int:
    head = stream_t[:4].cpu().numpy().tobytes()
    off = 0
    if head == b"SZXC":
        off = struct.unpack_from("<Q", stream_t[48:56].cpu().numpy().tobytes())[0]
    return struct.unpack_from("<I", stream_t[off + 8:off + 12].cpu().numpy().tobytes())[0]


def decompress(s: torch.Tensor, out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """Decompress an SZX1 stream or SZXC container held in a uint8 CUDA tensor."""
    _require_cuda(s)
    n, dt = _container_info(s)
    tdt = torch.float32 if dt == F32 else torch.float64
    if out is None:
        out = torch.empty(max(n, 1), dtype=tdt, device=s.device)
    r = lib().szx_decompress(s.data_ptr(), s.numel(), out.data_ptr(), out.numel() * out.element_size(),
                             _stream(stream))
    _check(r, "szx_decompress")
    return out[:n]


def decompress_blocks(s: torch.Tensor, first_block: int, n_blocks: int, out: torch.Tensor | None = None,
                      stream=None) -> torch.Tensor:
    """Decompress blocks [first_block, first_block + n_blocks) of an SZX1 stream or SZXC container
    (global block numbering); returns values [first_block*b, min(n, (first_block+n_blocks)*b))."""
    _require_cuda(s)
    n, dt = _container_info(s)
    b = _block_size(s)
    tdt = torch.float32 if dt == F32 else torch.float64
    nB = (n + b - 1) // b
    e0 = min(first_block, nB) * b
    e1 = min(n, min(nB, first_block + n_blocks) * b)
    cnt = max(0, e1 - e0)
    if out is None:
        out = torch.empty(max(cnt, 1), dtype=tdt, device=s.device)
    r = lib().szx_decompress_blocks(s.data_ptr(), s.numel(), first_block, n_blocks, out.data_ptr(),
                                    out.numel() * out.element_size(), _stream(stream))
    _check(r, "szx_decompress_blocks")
    return out[:r]


def _quality_dict(q, n: int) -> dict:
    maxe, sse, dmin, dmax = (float(v) for v in q)
    mse = sse / n if n else 0.0
    rng = dmax - dmin
    if mse == 0.0:
        psnr = math.inf
    elif not math.isfinite(mse) or not rng > 0:
        psnr = -math.inf
    else:
        psnr = 20.0 * math.log10(rng / math.sqrt(mse))
    return dict(max_abs_err=maxe, sse=sse, mse=mse, dmin=dmin, dmax=dmax, psnr=psnr)


def decompress_quality(s: torch.Tensor, ref: torch.Tensor, out: torch.Tensor | None = None, stream=None):
    """Decompress and, fused into the decode kernel, measure the reconstruction against the
    original ``ref``: returns (values, {max_abs_err, sse, mse, dmin, dmax, psnr}) -- Formula 1's
    max error and Formula 7's PSNR."""
    _require_cuda(s)
    _require_cuda(ref)
    n, dt = _container_info(s)
    tdt = torch.float32 if dt == F32 else torch.float64
    ref = ref.contiguous().view(-1)
    if ref.numel() != n or ref.dtype != tdt:
        raise ValueError(f"reference must hold {n} {tdt} values")
    if out is None:
        out = torch.empty(max(n, 1), dtype=tdt, device=s.device)
    q = (ctypes.c_double * 4)()
    r = lib().szx_decompress_quality(s.data_ptr(), s.numel(), ref.data_ptr() if n else None, out.data_ptr(),
                                     out.numel() * out.element_size(), q, _stream(stream))
    _check(r, "szx_decompress_quality")
    return out[:n], _quality_dict(list(q), n)


def dump_host(x: torch.Tensor, eb: float, mode="rel", block_size: int = 128, parts: int = 8, out=None,
              stream=None) -> torch.Tensor:
    """Dump a CUDA tensor to host memory as an SZXC container of `parts` block-range shards,
    compression of shard p+1 overlapping the copy-out of shard p (Fig. 16 analogue).  Returns a
    uint8 CPU tensor view (pinned)."""
    _require_cuda(x)
    x = x.contiguous().view(-1)
    dt = _dtype_code(x)
    if out is None:
        nb = (x.numel() + block_size - 1) // block_size
        P = max(1, min(parts, max(nb, 1)))
        per = (nb + P - 1) // P * block_size
        out = torch.empty(32 + 32 * P + P * (compress_bound(per, dt, block_size) + 16), dtype=torch.uint8,
                          pin_memory=True)
    r = lib().szx_dump_host(x.data_ptr() if x.numel() else None, dt, x.numel(), _mode_code(mode), float(eb),
                            block_size, parts, out.data_ptr(), out.numel(), _stream(stream))
    _check(r, "szx_dump_host")
    return out[:r]


def load_host(s: torch.Tensor, out: torch.Tensor | None = None, device="cuda", stream=None) -> torch.Tensor:
    """Load a host-resident stream or container (uint8 CPU tensor, ideally pinned) into a CUDA tensor,
    the copy of shard q+1 overlapping the decode of shard q."""
    if s.is_cuda:
        raise ValueError("host tensor required")
    head = s[:64].numpy().tobytes()
    if head[:4] == b"SZXC":
        n = struct.unpack_from("<Q", head, 16)[0]
        off0 = struct.unpack_from("<Q", s[48:56].numpy().tobytes())[0]
        dt = int(s[off0 + 5])
    else:
        h = read_header(head)
        n, dt = h.n, h.dtype
    tdt = torch.float32 if dt == F32 else torch.float64
    if out is None:
        out = torch.empty(max(n, 1), dtype=tdt, device=device)
    r = lib().szx_load_host(s.data_ptr(), s.numel(), out.data_ptr(), out.numel() * out.element_size(),
                            _stream(stream))
    _check(r, "szx_load_host")
    return out[:n]


def compress_host(x, eb: float, mode="rel", block_size: int = 128, out=None, stream=None):
    """End-to-end compress of a HOST tensor (ideally pinned) through the C ABI's host entry point.
    Returns a uint8 CPU tensor view of the stream."""
    x = x.contiguous().view(-1)
    if x.is_cuda:
        raise ValueError("host tensor required")
    dt = _dtype_code(x)
    cap = compress_bound(x.numel(), dt, block_size)
    if out is None:
        out = torch.empty(cap, dtype=torch.uint8, pin_memory=True)
    r = lib().szx_compress_host(x.data_ptr() if x.numel() else None, dt, x.numel(), _mode_code(mode),
                                float(eb), block_size, out.data_ptr(), out.numel(), _stream(stream))
    _check(r, "szx_compress_host")
    return out[:r]


def decompress_host(s, out=None, stream=None):
    """End-to-end decompress of a HOST stream (uint8 CPU tensor) into a host tensor."""
    if s.is_cuda:
        raise ValueError("host tensor required")
    head = s[:64].numpy().tobytes()
    if head[:4] == b"SZXC":
        n = struct.unpack_from("<Q", head, 16)[0]
        off0 = struct.unpack_from("<Q", s[48:56].numpy().tobytes())[0]
        dt = int(s[off0 + 5])
    else:
        h = read_header(head)
        n, dt = h.n, h.dtype
    tdt = torch.float32 if dt == F32 else torch.float64
    if out is None:
        out = torch.empty(max(n, 1), dtype=tdt, pin_memory=True)
    r = lib().szx_decompress_host(s.data_ptr(), s.numel(), out.data_ptr(), out.numel() * out.element_size(),
                                  _stream(stream))
    _check(r, "szx_decompress_host")
    return out[:n]


def local_minmax(x: torch.Tensor, stream=None) -> torch.Tensor:
    """SURVEY 8(b) szx_local_minmax: (min, max) of the finite values of a CUDA tensor, as a float64
    device tensor of 2 (no finite value -> (+inf, -inf)); non-blocking."""
    _require_cuda(x)
    x = x.contiguous().view(-1)
    mm = torch.empty(2, dtype=torch.float64, device=x.device)
    _check(lib().szx_local_minmax(x.data_ptr() if x.numel() else None, _dtype_code(x), x.numel(), mm.data_ptr(),
                                  _stream(stream)), "szx_local_minmax")
    return mm


def compress_shard(x: torch.Tensor, eb: float, eb_abs: torch.Tensor, mode="rel", block_size: int = 128,
                   out: torch.Tensor | None = None, stream=None) -> torch.Tensor:
    """SURVEY 8(b) szx_compress_shard: compress a shard with the absolute bound held on the device
    (eb_abs: float64 CUDA tensor of 1); blocking, returns the stream (uint8 CUDA tensor)."""
    _require_cuda(x)
    x = x.contiguous().view(-1)
    dt = _dtype_code(x)
    cap = compress_bound(x.numel(), dt, block_size)
    if out is None:
        out = torch.empty(cap, dtype=torch.uint8, device=x.device)
    assert eb_abs.is_cuda and eb_abs.dtype == torch.float64 and eb_abs.is_contiguous()
    nb = _check(lib().szx_compress_shard(x.data_ptr() if x.numel() else None, dt, x.numel(), _mode_code(mode),
                                         float(eb), eb_abs.data_ptr(), block_size, out.data_ptr(), out.numel(),
                                         _stream(stream)), "szx_compress_shard")
    return out[:nb]


class Codec:
    """Reusable buffers for repeated compress/decompress of same-shaped arrays (bench, pipelines).

    ``compress_async`` / ``decompress_async`` never synchronise: the stream length stays on
    the device (``self.d_total``) until ``stream_bytes()`` reads it back.
    """

    def __init__(self, n: int, dtype=torch.float32, block_size: int = 128, device="cuda"):
        self.n, self.block_size = n, block_size
        self.dt = F32 if dtype == torch.float32 else F64
        self.dtype = dtype
        self.device = torch.device(device)
        self.cap = compress_bound(n, self.dt, block_size)
        self.out = torch.empty(self.cap, dtype=torch.uint8, device=device)
        self.ws = torch.empty(max(workspace_bytes(n, self.dt, block_size), 16), dtype=torch.uint8, device=device)
        self.d_total = torch.zeros(1, dtype=torch.int64, device=device)
        self.d_status = torch.zeros(1, dtype=torch.int32, device=device)
        self.dws = None

    def compress_async(self, x: torch.Tensor, eb: float, mode="rel", stream=None):
        assert x.is_cuda and x.numel() == self.n and x.dtype == self.dtype and x.is_contiguous()
        rc = lib().szx_compress_async(x.data_ptr() if self.n else None, self.dt, self.n, _mode_code(mode),
                                      float(eb), self.block_size, self.out.data_ptr(), self.cap,
                                      self.ws.data_ptr(), self.ws.numel(), self.d_total.data_ptr(),
                                      _stream(stream))
        _check(rc, "szx_compress_async")

    def stream_bytes(self) -> int:
        return int(self.d_total.item())

    def header(self) -> Header:
        return read_header(self.out[:64].cpu().numpy().tobytes())

    def decompress_async(self, s: torch.Tensor, h: Header, y: torch.Tensor, stream=None):
        need = int(lib().szx_decompress_workspace_bytes(ctypes.byref(h._c)))
        if self.dws is None or self.dws.numel() < need:
            self.dws = torch.empty(max(need, 16), dtype=torch.uint8, device=self.device)
        rc = lib().szx_decompress_async(s.data_ptr(), s.numel(), ctypes.byref(h._c), y.data_ptr(),
                                        y.numel() * y.element_size(), self.dws.data_ptr(), self.dws.numel(),
                                        self.d_status.data_ptr(), _stream(stream))
        _check(rc, "szx_decompress_async")

    def decompress_quality_async(self, s: torch.Tensor, h: Header, y: torch.Tensor, ref: torch.Tensor,
                                 stream=None):
        """decompress_async with the fused quality accumulators (read with ``quality()``)."""
        need = int(lib().szx_decompress_workspace_bytes(ctypes.byref(h._c)))
        if self.dws is None or self.dws.numel() < need:
            self.dws = torch.empty(max(need, 16), dtype=torch.uint8, device=self.device)
        if getattr(self, "d_qual", None) is None:
            self.d_qual = torch.zeros(4, dtype=torch.int64, device=self.device)
        rc = lib().szx_decompress_quality_async(s.data_ptr(), s.numel(), ctypes.byref(h._c), ref.data_ptr(),
                                                y.data_ptr(), y.numel() * y.element_size(), self.dws.data_ptr(),
                                                self.dws.numel(), self.d_qual.data_ptr(),
                                                self.d_status.data_ptr(), _stream(stream))
        _check(rc, "szx_decompress_quality_async")

    def quality(self) -> dict:
        raw = self.d_qual.cpu().numpy()
        q = (ctypes.c_double * 4)()
        lib().szx_quality_finish(raw.ctypes.data, q)
        return _quality_dict(list(q), self.n)


def timing_enable(on: bool = True):
    lib().szx_timing_enable(1 if on else 0)


def timing_reset():
    lib().szx_timing_reset()


def timing_read() -> dict:
    names = (ctypes.c_char_p * 32)()
    ms = (ctypes.c_double * 32)()
    cnt = (ctypes.c_uint64 * 32)()
    k = lib().szx_timing_read(names, ms, cnt, 32)
    return {names[i].decode(): (ms[i], int(cnt[i])) for i in range(min(k, 32))}


def launch_count() -> int:
    return int(lib().szx_launch_count())


def set_r_bias(r: int):
    """Test hook (see szx_debug_set_r_bias)."""
    lib().szx_debug_set_r_bias(int(r))
