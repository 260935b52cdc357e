"""Independent pure-Python SZx decoder, written straight from the paper.

Used only to pin the C oracle's stream and decoder: it shares nothing with
oracle/szx_oracle.c or the CUDA path.  It follows Fig. 10 / Sec. 6.1
 point by point:
  (1) read the leading number n of the current point,
  (2) copy the first n bytes of the previous point,
  (3) read the remaining (mid-)bytes,
  (4) combine and overwrite the previous point,
  (5) left shift, then add the block's mu.
Layout readings R7-R12; small inputs only.
"""
from __future__ import annotations

import struct

import numpy as np


def _al16(x: int) -> int:
    return (x + 15) // 16 * 16


def decode(stream: bytes):
    """Return (values as np array, per-block info list)."""
    s = bytes(stream)
    assert s[:4] == b"SZX1"
    dtype = s[5]
    b = struct.unpack_from("<I", s, 8)[0]
    n = struct.unpack_from("<Q", s, 16)[0]
    nnc = struct.unpack_from("<Q", s, 40)[0]
    pbytes = struct.unpack_from("<Q", s, 48)[0]
    W = 4 if dtype == 0 else 8
    npdt = np.float32 if W == 4 else np.float64
    uint = np.uint32 if W == 4 else np.uint64
    nB = (n + b - 1) // b
    off_bm = 64
    off_mu = off_bm + _al16((nB + 7) // 8)
    off_zs = off_mu + _al16(W * nB)
    off_pl = off_zs + _al16(2 * nnc)
    assert len(s) == off_pl + pbytes, (len(s), off_pl, pbytes)
    zs = [struct.unpack_from("<H", s, off_zs + 2 * j)[0] for j in range(nnc)]
    assert sum(zs) == pbytes
    out = np.zeros(n, dtype=npdt)
    info = []
    pos = off_pl
    nc = 0
    full = 8 * W
    for k in range(nB):
        first = k * b
        ln = min(b, n - first)
        state = (s[off_bm + k // 8] >> (k % 8)) & 1
        mu_bits = int.from_bytes(s[off_mu + W * k: off_mu + W * k + W], "little")
        mu = np.array([mu_bits], dtype=uint).view(npdt)[0]
        if state == 0:
            out[first:first + ln] = mu
            info.append(("const", mu_bits))
            continue
        start = pos
        R = s[pos]
        pos += 1
        ncode = (ln + 3) // 4
        codes = s[pos:pos + ncode]
        pos += ncode
        raw = R >= full
        sh = 0 if raw else (0 if R % 8 == 0 else 8 - R % 8)
        req = W if raw else (R + sh) // 8
        prev = [0] * W          # bytes, index 0 = most significant
        for i in range(ln):
            lead = (codes[i // 4] >> (2 * (i % 4))) & 3           # (1)
            cur = [0] * W
            for j in range(min(lead, req)):                          # (2)
                cur[j] = prev[j]
            # (3) mid-bytes: stored least-significant first (R7), i.e. the
            # byte at significance position req-1 comes first, lead last.
            for j in range(req - 1, lead - 1, -1):
                cur[j] = s[pos]
                pos += 1
            prev = cur                                               # (4)
            word = 0
            for j in range(W):
                word = (word << 8) | cur[j]
            word = (word << sh) & ((1 << full) - 1)                  # (5)
            v = np.array([word], dtype=uint).view(npdt)[0]
            out[first + i] = v if raw else npdt(v + mu)
        z = pos - start
        assert z == zs[nc], (k, z, zs[nc])
        info.append(("nonconst", R, z))
        nc += 1
    assert nc == nnc and pos == len(s)
    return out, info
