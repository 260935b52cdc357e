"""ctypes wrapper around the serial C oracle (oracle/szx_oracle.c).

TEST INFRASTRUCTURE ONLY: tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / ``--impl reference`` legs are the only callers.  The product
package never imports this module.

Every function takes / returns numpy arrays and mirrors one exported C
function; see szx_oracle.c for the paper passages each step follows.
"""
from __future__ import annotations

import ctypes
import os
import subprocess
from dataclasses import dataclass

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "szx_oracle.c")
_LIB = os.path.join(_HERE, "libszx_oracle.so")

F32, F64 = 0, 1
ABS, REL = 0, 1
OK, EINVAL, ENOSPC, ECORRUPT, ENOMEM = 0, -1, -2, -3, -5

CFLAGS = ["-O2", "-std=c99", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]


def build(force: bool = False) -> str:
    """Compile the oracle with gcc (no FMA contraction, no fast-math)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-o", tmp, _SRC, "-lm"])
        os.replace(tmp, _LIB)
    return _LIB


_OMP_SRC = os.path.join(_HERE, "szx_omp.c")
_OMP_LIB = os.path.join(_HERE, "libszx_omp.so")


def build_omp(force: bool = False) -> str:
    """Compile the OpenMP-design host baseline (szx_omp.c includes szx_oracle.c; same FP flags)."""
    if (force or not os.path.exists(_OMP_LIB)
            or os.path.getmtime(_OMP_LIB) < max(os.path.getmtime(_OMP_SRC), os.path.getmtime(_SRC))):
        tmp = _OMP_LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *CFLAGS, "-fopenmp", "-o", tmp, _OMP_SRC, "-lm"], cwd=_HERE)
        os.replace(tmp, _OMP_LIB)
    return _OMP_LIB


_lib = None
_omp = None


def omp_lib():
    global _omp
    if _omp is None:
        build_omp()
        L = ctypes.CDLL(_OMP_LIB)
        L.omp_compress.restype = ctypes.c_int64
        L.omp_compress.argtypes = [ctypes.c_void_p, ctypes.c_int, ctypes.c_uint64, ctypes.c_int, ctypes.c_double,
                                   ctypes.c_uint32, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_int]
        L.omp_decompress.restype = ctypes.c_int64
        L.omp_decompress.argtypes = [ctypes.c_void_p, ctypes.c_uint64, ctypes.c_void_p, ctypes.c_uint64,
                                     ctypes.c_int]
        _omp = L
    return _omp


def omp_compress(x: np.ndarray, eb: float, mode: int = REL, b: int = 128, threads: int = 0) -> np.ndarray:
    """The paper's OpenMP design (Sec. 6.1): one stream, byte-identical to compress()."""
    x = np.ascontiguousarray(x).reshape(-1)
    dt = _dtype_code(x)
    out = np.empty(max(compress_bound(x.size, dt, b), 64), dtype=np.uint8)
    r = omp_lib().omp_compress(x.ctypes.data if x.size else None, dt, x.size, mode, float(eb), b,
                               out.ctypes.data, out.size, int(threads))
    if r < 0:
        raise ValueError(f"omp_compress failed: {r}")
    return out[:r].copy()


def omp_decompress(stream: np.ndarray, threads: int = 0) -> np.ndarray:
    stream = np.ascontiguousarray(stream, dtype=np.uint8)
    h = read_header(stream)
    out = np.empty(h["n"], dtype=np.float32 if h["dtype"] == F32 else np.float64)
    r = omp_lib().omp_decompress(stream.ctypes.data, stream.size, out.ctypes.data if out.size else None,
                                 out.nbytes, int(threads))
    if r < 0:
        raise ValueError(f"omp_decompress failed: {r}")
    return out


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(_LIB)
        u64, i64, c_int, vp, dbl = (ctypes.c_uint64, ctypes.c_int64, ctypes.c_int,
                                    ctypes.c_void_p, ctypes.c_double)
        L.orc_compress.restype = i64
        L.orc_compress.argtypes = [vp, c_int, u64, c_int, dbl, ctypes.c_uint32, vp, u64, vp]
        L.orc_compress_ex.restype = i64
        L.orc_compress_ex.argtypes = [vp, c_int, u64, c_int, dbl, ctypes.c_uint32, vp, u64, vp,
                                      c_int]
        L.orc_decompress.restype = i64
        L.orc_decompress.argtypes = [vp, u64, vp, u64]
        L.orc_decompress_any.restype = i64
        L.orc_decompress_any.argtypes = [vp, u64, vp, u64]
        L.orc_compress_bound.restype = u64
        L.orc_compress_bound.argtypes = [u64, c_int, ctypes.c_uint32]
        L.orc_container_bound.restype = u64
        L.orc_container_bound.argtypes = [u64, c_int, ctypes.c_uint32, ctypes.c_uint32]
        L.orc_container_compress.restype = i64
        L.orc_container_compress.argtypes = [vp, c_int, u64, c_int, dbl, ctypes.c_uint32,
                                             ctypes.c_uint32, vp, u64]
        L.orc_compress_shard.restype = i64
        L.orc_compress_shard.argtypes = [vp, c_int, u64, c_int, dbl, dbl, ctypes.c_uint32, vp, u64]
        L.orc_eb_abs.restype = dbl
        L.orc_eb_abs.argtypes = [vp, c_int, u64, c_int, dbl]
        L.orc_p_f32.restype = c_int
        L.orc_p_f32.argtypes = [ctypes.c_float]
        L.orc_p_f64.restype = c_int
        L.orc_p_f64.argtypes = [dbl]
        L.orc_required_bits_f32.restype = c_int
        L.orc_required_bits_f32.argtypes = [ctypes.c_float, dbl]
        L.orc_required_bits_f64.restype = c_int
        L.orc_required_bits_f64.argtypes = [dbl, dbl]
        L.orc_shift_for.restype = c_int
        L.orc_shift_for.argtypes = [c_int]
        L.orc_identical_leading_bytes.restype = c_int
        L.orc_identical_leading_bytes.argtypes = [u64, u64, c_int]
        L.orc_quality.restype = c_int
        L.orc_quality.argtypes = [vp, vp, c_int, u64, vp]
        L.orc_shift_overhead.restype = c_int
        L.orc_shift_overhead.argtypes = [vp, u64, vp, vp]
        _lib = L
    return _lib


class _Trace(ctypes.Structure):
    _fields_ = [("type", ctypes.c_void_p), ("mu", ctypes.c_void_p), ("R", ctypes.c_void_p),
                ("z", ctypes.c_void_p), ("escal", ctypes.c_void_p)]


@dataclass
class Trace:
    type: np.ndarray
    mu: np.ndarray
    R: np.ndarray
    z: np.ndarray
    escal: np.ndarray


def _dtype_code(x: np.ndarray) -> int:
    if x.dtype == np.float32:
        return F32
    if x.dtype == np.float64:
        return F64
    raise TypeError(f"oracle supports float32/float64, got {x.dtype}")


def compress_bound(n: int, dtype: int, b: int = 128) -> int:
    return int(lib().orc_compress_bound(n, dtype, b))


def compress(x: np.ndarray, eb: float, mode: int = REL, b: int = 128,
             trace: bool = False, r_bias: int = 0):
    """Serial SZx compress -> (stream bytes as np.uint8[, Trace]).

    r_bias != 0 is a test hook that starts the R2 escalation search r_bias
    bits away from Formula 4 (the GPU library has the same hook)."""
    x = np.ascontiguousarray(x).reshape(-1)
    dt = _dtype_code(x)
    n = x.size
    cap = compress_bound(n, dt, b) if b > 0 else 64
    out = np.empty(max(cap, 64), dtype=np.uint8)
    tr_ptr = None
    tr = None
    if trace:
        nB = (n + b - 1) // b if b > 0 else 0
        tr = Trace(np.zeros(nB, np.uint8), np.zeros(nB, np.uint64), np.zeros(nB, np.uint8),
                   np.zeros(nB, np.uint16), np.zeros(nB, np.uint32))
        ct = _Trace(tr.type.ctypes.data, tr.mu.ctypes.data, tr.R.ctypes.data,
                    tr.z.ctypes.data, tr.escal.ctypes.data)
        tr_ptr = ctypes.byref(ct)
    r = lib().orc_compress_ex(x.ctypes.data if n else None, dt, n, mode, float(eb), b,
                              out.ctypes.data, out.size, tr_ptr, int(r_bias))
    if r < 0:
        raise ValueError(f"orc_compress failed: {r}")
    s = out[:r].copy()
    return (s, tr) if trace else s


def compress_rc(x: np.ndarray, eb: float, mode: int = REL, b: int = 128) -> int:
    """Return code only (for argument-validation tests)."""
    x = np.ascontiguousarray(x).reshape(-1)
    dt = _dtype_code(x)
    out = np.empty(max(compress_bound(x.size, dt, max(b, 4)), 64) * 2, dtype=np.uint8)
    return int(lib().orc_compress(x.ctypes.data if x.size else None, dt, x.size, mode, float(eb),
                                  b, out.ctypes.data, out.size, None))


def decompress(stream: np.ndarray) -> np.ndarray:
    """Decode an SZX1 stream or an SZXC container."""
    stream = np.ascontiguousarray(stream, dtype=np.uint8)
    h = read_header_any(stream)
    out = np.empty(h["n"], dtype=np.float32 if h["dtype"] == F32 else np.float64)
    r = lib().orc_decompress_any(stream.ctypes.data, stream.size,
                                 out.ctypes.data if out.size else None, out.nbytes)
    if r < 0:
        raise ValueError(f"orc_decompress failed: {r}")
    return out


def decompress_rc(stream: np.ndarray, n: int, dtype) -> int:
    stream = np.ascontiguousarray(stream, dtype=np.uint8)
    out = np.empty(max(n, 1), dtype=dtype)
    return int(lib().orc_decompress_any(stream.ctypes.data, stream.size, out.ctypes.data,
                                        n * out.itemsize))


def container_compress(x: np.ndarray, eb: float, mode: int, b: int, P: int) -> np.ndarray:
    x = np.ascontiguousarray(x).reshape(-1)
    dt = _dtype_code(x)
    cap = int(lib().orc_container_bound(x.size, dt, b, P))
    out = np.empty(cap, dtype=np.uint8)
    r = lib().orc_container_compress(x.ctypes.data if x.size else None, dt, x.size, mode,
                                     float(eb), b, P, out.ctypes.data, cap)
    if r < 0:
        raise ValueError(f"orc_container_compress failed: {r}")
    return out[:r].copy()


def compress_shard(x: np.ndarray, eb_user: float, eb_abs: float, mode: int = REL, b: int = 128) -> np.ndarray:
    """Standalone stream of a shard compressed with the GLOBAL bound eb_abs."""
    x = np.ascontiguousarray(x).reshape(-1)
    dt = _dtype_code(x)
    out = np.empty(max(compress_bound(x.size, dt, b), 64), dtype=np.uint8)
    r = lib().orc_compress_shard(x.ctypes.data if x.size else None, dt, x.size, mode, float(eb_user),
                                 float(eb_abs), b, out.ctypes.data, out.size)
    if r < 0:
        raise ValueError(f"orc_compress_shard failed: {r}")
    return out[:r].copy()


def eb_abs(x: np.ndarray, eb: float, mode: int) -> float:
    x = np.ascontiguousarray(x).reshape(-1)
    return float(lib().orc_eb_abs(x.ctypes.data if x.size else None, _dtype_code(x), x.size,
                                  mode, float(eb)))


def read_header(s: np.ndarray) -> dict:
    s = np.asarray(s, dtype=np.uint8)
    b = s[:64].tobytes()
    assert b[:4] == b"SZX1", b[:4]
    le = int.from_bytes
    return dict(version=b[4], dtype=b[5], mode=b[6], b=le(b[8:12], "little"),
                n=le(b[16:24], "little"),
                eb_user=np.frombuffer(b[24:32], np.float64)[0],
                eb_abs=np.frombuffer(b[32:40], np.float64)[0],
                nnc=le(b[40:48], "little"), payload_bytes=le(b[48:56], "little"))


def read_header_any(s: np.ndarray) -> dict:
    s = np.asarray(s, dtype=np.uint8)
    if s[:4].tobytes() == b"SZXC":
        le = int.from_bytes
        raw = s[:48].tobytes()
        P = le(raw[8:12], "little")
        n = le(raw[16:24], "little")
        off0 = le(s[32 + 16:32 + 24].tobytes(), "little")
        h0 = read_header(s[off0:])
        return dict(n=n, dtype=h0["dtype"], P=P)
    return read_header(s)


# helpers exported for the pins
def p_f32(x: float) -> int:
    return int(lib().orc_p_f32(x))


def p_f64(x: float) -> int:
    return int(lib().orc_p_f64(x))


def required_bits_f32(r: float, e: float) -> int:
    return int(lib().orc_required_bits_f32(r, e))


def required_bits_f64(r: float, e: float) -> int:
    return int(lib().orc_required_bits_f64(r, e))


def shift_for(R: int) -> int:
    return int(lib().orc_shift_for(R))


def identical_leading_bytes(prev: int, cur: int, W: int) -> int:
    return int(lib().orc_identical_leading_bytes(prev, cur, W))


def quality(x: np.ndarray, xr: np.ndarray) -> dict:
    """Max abs error (Formula 1's quantity), SSE / MSE, finite value range and
    PSNR (Formula 7) of a reconstruction xr of x."""
    x = np.ascontiguousarray(x).reshape(-1)
    xr = np.ascontiguousarray(xr, dtype=x.dtype).reshape(-1)
    assert x.size == xr.size
    q = np.zeros(4, np.float64)
    r = lib().orc_quality(x.ctypes.data if x.size else None, xr.ctypes.data if xr.size else None,
                          _dtype_code(x), x.size, q.ctypes.data)
    if r < 0:
        raise ValueError(f"orc_quality failed: {r}")
    return _quality_dict(q, x.size)


def _quality_dict(q, n: int) -> dict:
    maxe, sse, dmin, dmax = (float(v) for v in q)
    mse = sse / n if n else 0.0
    rng = dmax - dmin
    if mse == 0.0:
        psnr = float("inf")
    elif not np.isfinite(mse) or not rng > 0:
        psnr = float("-inf")
    else:
        psnr = 20.0 * np.log10(rng / np.sqrt(mse))
    return dict(max_abs_err=maxe, sse=sse, mse=mse, dmin=dmin, dmax=dmax, psnr=float(psnr))


def shift_overhead(stream: np.ndarray, x: np.ndarray) -> dict:
    """Formula 6: necessary bits under Solution C (stored) and
    Solution A/B, and the overhead relative to the stream size."""
    stream = np.ascontiguousarray(stream, dtype=np.uint8)
    x = np.ascontiguousarray(x).reshape(-1)
    out = np.zeros(2, np.uint64)
    r = lib().orc_shift_overhead(stream.ctypes.data, stream.size, x.ctypes.data if x.size else None,
                                 out.ctypes.data)
    if r < 0:
        raise ValueError(f"orc_shift_overhead failed: {r}")
    bc, bb = int(out[0]), int(out[1])
    return dict(bits_C=bc, bits_B=bb, overhead=(bc - bb) / 8.0 / stream.size)
