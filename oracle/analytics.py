"""Oracle-side analytics of SURVEY 8(f) rows 1-2 (TEST / ANALYSIS INFRASTRUCTURE: used by
scripts/ and tests/ only, never by the product).

block_relative_range: Fig. 2's quantity (footnote 1):
    for every block of b consecutive values, (max - min) / (global max - global min), over the
    finite values (a block with no finite value is skipped), in float64.
cdf_points: the empirical CDF of those ranges at given thresholds (Fig. 2's curves).
shift_bits: an independent numpy restatement of Formula 6's two sums from a
    stream and its input -- Solution C's necessary bits R_k + s - L'_i and Solution B's R_k - L_i
    per value of every nonconstant block -- cross-checking oracle.shift_overhead.
"""
from __future__ import annotations

import numpy as np


def block_relative_range(x: np.ndarray, b: int) -> np.ndarray:
    x = np.ascontiguousarray(x).reshape(-1).astype(np.float64)
    fin = np.isfinite(x)
    if not fin.any():
        return np.zeros(0)
    gmin, gmax = x[fin].min(), x[fin].max()
    rng = gmax - gmin
    nB = (x.size + b - 1) // b
    pad = nB * b - x.size
    lo = np.where(fin, x, np.inf)
    hi = np.where(fin, x, -np.inf)
    if pad:
        lo = np.concatenate([lo, np.full(pad, np.inf)])
        hi = np.concatenate([hi, np.full(pad, -np.inf)])
    bmin = lo.reshape(nB, b).min(axis=1)
    bmax = hi.reshape(nB, b).max(axis=1)
    ok = np.isfinite(bmin)
    r = bmax[ok] - bmin[ok]
    return r / rng if rng > 0 else np.zeros_like(r)


def cdf_points(rel: np.ndarray, thresholds) -> list:
    """Fraction of blocks whose relative range is <= each threshold."""
    rel = np.sort(rel)
    return [float(np.searchsorted(rel, t, side="right") / max(rel.size, 1)) for t in thresholds]


def _lead_bytes(a: np.ndarray, b: np.ndarray, W: int) -> np.ndarray:
    """Identical leading bytes of two W-byte words (uncapped), vectorised."""
    x = (a ^ b).astype(np.uint64)
    n = np.zeros(x.shape, np.int64)
    alive = np.ones(x.shape, bool)
    for j in range(W - 1, -1, -1):
        same = ((x >> np.uint64(8 * j)) & np.uint64(0xFF)) == 0
        alive &= same
        n += alive
    return n


def shift_bits(stream: np.ndarray, x: np.ndarray) -> tuple[int, int]:
    """(bits_C, bits_B) of Formula 6 for an SZX1 stream of x (DESIGN.md s.3 reading:
    L'_i = 8 min(lead'_i, req) on the shifted words, L_i = 8 min(lead_i, floor(R / 8)) on the
    unshifted normalised words, lead capped at 3 (the 2-bit code), u_{-1} = 0 per block)."""
    s8 = np.ascontiguousarray(stream, np.uint8)
    h = np.frombuffer(s8[:64].tobytes(), dtype="<u8")
    dtype, b, n, nnc = int(s8[5]), int(h[1] & 0xFFFFFFFF), int(h[2]), int(h[5])
    W = 4 if dtype == 0 else 8
    al = lambda v: (v + 15) // 16 * 16
    nB = (n + b - 1) // b
    off_mu = 64 + al((nB + 7) // 8)
    off_zs = off_mu + al(W * nB)
    off_pl = off_zs + al(2 * nnc)
    bm = np.unpackbits(s8[64:64 + (nB + 7) // 8], bitorder="little")[:nB]
    ft, ut = (np.float32, np.uint32) if W == 4 else (np.float64, np.uint64)
    mus = s8[off_mu:off_mu + W * nB].view(ut)
    zs = s8[off_zs:off_zs + 2 * nnc].view(np.uint16).astype(np.int64)
    xf = np.ascontiguousarray(x, ft).reshape(-1)
    mask = np.uint64((1 << (8 * W)) - 1)
    bitsC = bitsB = 0
    off = off_pl
    for j, k in enumerate(np.flatnonzero(bm)):
        R = int(s8[off])
        raw = R >= 8 * W
        s = 0 if raw else (8 - R % 8) % 8
        req = W if raw else (R + s) // 8
        alpha = R // 8
        blk = xf[k * b:(k + 1) * b]
        if raw:
            v = blk.view(ut).astype(np.uint64)
        else:
            mu = mus[k:k + 1].view(ft)[0]
            v = (blk - mu).astype(ft).view(ut).astype(np.uint64)  # v_i = d_i - mu in the data type
        v &= mask
        u = v >> np.uint64(s)
        pu = np.concatenate([[np.uint64(0)], u[:-1]])
        pv = np.concatenate([[np.uint64(0)], v[:-1]])
        lc = np.minimum(np.minimum(_lead_bytes(u, pu, W), 3), req)
        lb = np.minimum(np.minimum(_lead_bytes(v, pv, W), 3), alpha)
        bitsC += int(np.sum(R + s - 8 * lc))
        bitsB += int(np.sum(R - 8 * lb))
        off += int(zs[j])
    return bitsC, bitsB
