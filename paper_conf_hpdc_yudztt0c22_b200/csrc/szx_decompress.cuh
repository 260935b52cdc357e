// szx_decompress.cuh -- SZx decompression kernels for sm_100a.
//
//   k_index   (K5a) two single-pass decoupled-look-back scans in one launch:
//             (a) nonconstant index per bitmap word = prefix of popcounts,
//             (b) payload byte offset per group of 32 nonconstant blocks =
//                 prefix of zsize (the paper's "prefix-sum step to compute
//                 the starting location of each block").
//             Both totals are validated against the header (nNC, payload).
//   k_decode  (K5)  a CTA per tile of 32 blocks: stage the tile's payload
//             bytes in shared memory with 16-byte loads, then a warp per
//             block rebuilds each value with the five steps of Fig. 10
//             (P:L2321-2336).  The leading-byte dependence chains
//             (Challenge 2) are resolved by a warp scan of
//             byte-mask transfer functions instead of the paper's log-step
//             index propagation: lane l's values map an
//             incoming previous word c to (c & M_l) | D_l, and composing
//             those maps is associative.
#pragma once

#include "szx_device.cuh"

namespace szx {

struct DPlan {
    // host-known shape (from the caller); everything that depends on the
    // compressed content (nNC, payload size) is read from the header on the device
    uint64_t n, nB, nW, in_bytes;
    uint64_t off_mu;
    uint32_t b, dtype;
    uint32_t* ctr;             // [2] tickets, init 0
    uint64_t* status_a;        // init 0
    uint64_t* status_z;        // init 0
    uint32_t* ncpre;           // [nW]
    uint64_t* zpre;            // [ceil(nB/32) + 1]
    int32_t* err;              // 0 ok, else SZX_ECORRUPT
};

// Stream facts read from the 64-byte header in device memory, validated
// against the caller's shape.
struct DHdr {
    uint64_t nnc, payload_bytes, off_zs, off_pl, ngroups;
    bool ok;
};
template <int W>
__device__ inline DHdr read_dheader(const uint8_t* in, const DPlan& p) {
    const uint64_t* h = reinterpret_cast<const uint64_t*>(in);
    DHdr d;
    const uint64_t w0 = h[0];
    d.nnc = h[5];
    d.payload_bytes = h[6];
    const uint64_t maxz = 1 + p.b / 4 + (uint64_t)W * p.b;
    d.ok = (w0 & 0xFFFFFFFFFFull) == (0x31585A53ull | (1ull << 32)) && ((w0 >> 40) & 0xFF) == p.dtype &&
           ((w0 >> 48) & 0xFF) <= 1 && (w0 >> 56) == 0 && (uint32_t)h[1] == p.b && h[2] == p.n &&
           d.nnc <= p.nB && d.payload_bytes <= d.nnc * maxz;
    d.off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    d.off_pl = d.off_zs + al16(2 * d.nnc);
    d.ok = d.ok && d.off_pl + d.payload_bytes <= p.in_bytes;
    d.ngroups = (d.nnc + 31) / 32;
    return d;
}

__device__ inline void set_corrupt(int32_t* err) { atomicExch(err, -3); }

// 256-thread CTA exclusive scan of one value per thread; returns exclusive, sets *agg.
__device__ inline uint64_t cta_scan256(uint64_t v, uint64_t* agg, uint64_t* s_w /*[8]*/) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint64_t incl = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint64_t t = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += t;
    }
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    uint64_t wpre = 0, tot = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint64_t t = s_w[i];
        wpre += i < warp ? t : 0;
        tot += t;
    }
    *agg = tot;
    return wpre + incl - v;
}

template <int W>
__global__ void __launch_bounds__(256) k_index(DPlan p, const uint8_t* __restrict__ in) {
    __shared__ uint64_t s_tile, s_excl, s_w[8];
    const DHdr hd = read_dheader<W>(in, p);
    if (!hd.ok) {
        if (blockIdx.x == 0 && threadIdx.x == 0) set_corrupt(p.err);
        return;
    }
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[0], 1u);
    __syncthreads();
    const uint64_t t = s_tile;
    const uint64_t nTA = (p.nW + 1023) / 1024;
    const uint64_t nTZ = (hd.ngroups + 255) / 256;
    if (t >= nTA + nTZ) return;  // grid is sized for the largest possible nNC
    const int warp = threadIdx.x >> 5;
    if (t < nTA) {
        // (a) popcount prefix over bitmap words, 4 words per thread
        const uint32_t* bm = reinterpret_cast<const uint32_t*>(in + kHeaderBytes);
        const uint64_t w0 = t * 1024 + threadIdx.x * 4;
        uint32_t c[4];
        uint64_t sum = 0;
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const uint64_t w = w0 + q;
            uint32_t word = w < p.nW ? bm[w] : 0u;
            if (w == p.nW - 1 && (p.nB & 31)) word &= (1u << (p.nB & 31)) - 1u;  // ignore padding bits
            c[q] = __popc(word);
            sum += c[q];
        }
        uint64_t agg;
        uint64_t ex = cta_scan256(sum, &agg, s_w);
        if (warp == 0) {
            const uint64_t e = lookback_exclusive(p.status_a, t, agg);
            if ((threadIdx.x & 31) == 0) {
                s_excl = e;
                if (t == nTA - 1 && e + agg != hd.nnc) set_corrupt(p.err);
            }
        }
        __syncthreads();
        ex += s_excl;
#pragma unroll
        for (int q = 0; q < 4; q++) {
            if (w0 + q < p.nW) p.ncpre[w0 + q] = (uint32_t)ex;
            ex += c[q];
        }
    } else {
        // (b) zsize sums per group of 32 entries
        const uint64_t tz = t - nTA;
        const uint16_t* zs = reinterpret_cast<const uint16_t*>(in + hd.off_zs);
        const uint64_t g = tz * 256 + threadIdx.x;
        uint64_t sum = 0;
        if (g < hd.ngroups) {
            const uint64_t e0 = g * 32;
            if (e0 + 32 <= hd.nnc) {
                const uint4* q4 = reinterpret_cast<const uint4*>(zs + e0);
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    const uint4 v = q4[q];
                    const uint32_t a[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
                    for (int r = 0; r < 4; r++) sum += (a[r] & 0xFFFFu) + (a[r] >> 16);
                }
            } else {
                for (uint64_t e = e0; e < hd.nnc; e++) sum += zs[e];
            }
        }
        uint64_t agg;
        uint64_t ex = cta_scan256(sum, &agg, s_w);
        if (warp == 0) {
            const uint64_t e = lookback_exclusive(p.status_z, tz, agg);
            if ((threadIdx.x & 31) == 0) {
                s_excl = e;
                if (tz == nTZ - 1) {
                    p.zpre[hd.ngroups] = e + agg;
                    if (e + agg != hd.payload_bytes) set_corrupt(p.err);
                }
            }
        }
        __syncthreads();
        if (g < hd.ngroups) p.zpre[g] = ex + s_excl;
    }
}

template <typename T, int VPL>
struct DecodeCfg {
    static constexpr int B = 32 * VPL;
    static constexpr int BPW = VPL == 4 ? 4 : 2;
    static constexpr int NWARP = kTileBlocks / BPW;
    static constexpr int NT = NWARP * 32;
    static constexpr int MAXZ = 1 + B / 4 + Traits<T>::W * B;
    static constexpr int SMEM = 16 + kTileBlocks * MAXZ + 16;
};

template <typename T, int VPL>
__device__ inline void store_lane(T* __restrict__ y, uint64_t n, uint64_t k, int lane, const T (&v)[VPL]) {
    constexpr int B = 32 * VPL;
    const uint64_t first = k * B + (uint64_t)lane * VPL;
    if ((k + 1) * B <= n) {
        constexpr int NV = VPL * (int)sizeof(T) / 16;
        uint4* q = reinterpret_cast<uint4*>(y + first);
#pragma unroll
        for (int i = 0; i < NV; i++) q[i] = reinterpret_cast<const uint4*>(v)[i];
        return;
    }
#pragma unroll
    for (int i = 0; i < VPL; i++)
        if (first + i < n) y[first + i] = v[i];
}

// Decode one nonconstant block whose payload (z bytes) starts at src (smem).
template <typename T, int VPL>
__device__ inline bool decode_block(const uint8_t* src, uint32_t z, int len, T mu, T (&out)[VPL]) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    const int ncode = (len + 3) / 4;
    const int R = src[0];
    if (R < TR::kFloor || R > TR::kFull) return false;
    const bool raw = R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (R & 7)) & 7);
    const int req = (R + s) >> 3;
    const int first = lane * VPL;
    const int cnt = first >= len ? 0 : min(VPL, len - first);
    // (1) read the leading numbers
    uint32_t leads = 0;
#pragma unroll
    for (int q = 0; q < VPL / 4; q++) {
        const int cb = lane * (VPL / 4) + q;
        if (cb < ncode) leads |= (uint32_t)src[1 + cb] << (8 * q);
    }
    uint32_t m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const int L = (leads >> (2 * i)) & 3;
        m += (i < cnt && req > L) ? req - L : 0;
    }
    const uint32_t incl = warp_incl_scan(m);
    const uint32_t total = __shfl_sync(0xffffffffu, incl, 31);
    if (1u + (uint32_t)ncode + total != z) return false;
    // (3) mid-bytes -> own bytes, and the byte-mask transfer function of this lane
    const uint8_t* mb = src + 1 + ncode + (incl - m);
    U own[VPL];
    U M = ~U(0), D = 0;  // lane map: c -> (c & M) | D
    int pos = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        own[i] = 0;
        if (i < cnt) {
            const int L = (leads >> (2 * i)) & 3;
            for (int j = W - req; j < W - L; j++) own[i] |= (U)mb[pos++] << (8 * j);
            const int copy = L < req ? L : req;
            // bytes copied from the previous value: the top `copy` bytes (step 2)
            const U cm = copy == 0 ? U(0) : (~U(0) << (8 * (W - copy)));
            M &= cm;
            D = (D & cm) | own[i];
        }
    }
    // exclusive warp scan of lane maps -> the word carried into this lane (u_{-1} = 0)
    U cM = M, cD = D;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const U pM = __shfl_up_sync(0xffffffffu, cM, o);
        const U pD = __shfl_up_sync(0xffffffffu, cD, o);
        if (lane >= o) { cD = (pD & cM) | cD; cM = pM & cM; }
    }
    U prev = __shfl_up_sync(0xffffffffu, cD, 1);
    if (lane == 0) prev = 0;
    // (2)(4)(5) combine, overwrite previous, left shift, add mu
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        if (i < cnt) {
            const int L = (leads >> (2 * i)) & 3;
            const int copy = L < req ? L : req;
            const U cm = copy == 0 ? U(0) : (~U(0) << (8 * (W - copy)));
            const U w = (prev & cm) | own[i];
            prev = w;
            const U vb = w << s;
            out[i] = raw ? TR::from(vb) : TR::add(TR::from(vb), mu);
        } else {
            out[i] = T(0);
        }
    }
    return true;
}

template <typename T, int VPL>
__global__ void __launch_bounds__(DecodeCfg<T, VPL>::NT)
    k_decode(DPlan p, const uint8_t* __restrict__ in, T* __restrict__ y) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = DecodeCfg<T, VPL>;
    extern __shared__ __align__(16) uint8_t stg[];
    __shared__ uint32_t s_off[kTileBlocks], s_z[kTileBlocks];
    __shared__ uint64_t s_base;
    __shared__ int s_ok;
    const DHdr hd = read_dheader<TR::W>(in, p);
    if (!hd.ok) return;  // k_index has flagged it
    const uint64_t tile = blockIdx.x;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    uint32_t word = reinterpret_cast<const uint32_t*>(in + kHeaderBytes)[tile];
    if (tile == p.nW - 1 && (p.nB & 31)) word &= (1u << (p.nB & 31)) - 1u;
    const uint32_t cnt = __popc(word);

    if (warp == 0) {
        const uint64_t ncb = p.ncpre[tile];
        const uint16_t* zs = reinterpret_cast<const uint16_t*>(in + hd.off_zs);
        bool ok = ncb + cnt <= hd.nnc;
        uint64_t base = 0;
        uint32_t zl = 0;
        if (ok && cnt) {
            const uint64_t g0 = ncb & ~uint64_t(31);
            const uint64_t e = g0 + lane;
            const uint32_t part = warp_sum((e < ncb) ? zs[e] : 0u);
            base = p.zpre[ncb >> 5] + part;
            zl = (uint32_t)lane < cnt ? zs[ncb + lane] : 0u;
        }
        // the block containing bit `lane` of the word
        const uint32_t incl = warp_incl_scan(zl);
        const uint32_t tot = __shfl_sync(0xffffffffu, incl, 31);
        // each zsize must lie in [1 + ncode, MAXZ]  (ncode = b/4 except the tail block)
        bool zok = true;
        if ((uint32_t)lane < cnt) zok = zl >= 2 && zl <= (uint32_t)C::MAXZ;
        ok = ok && __all_sync(0xffffffffu, zok) && base + tot <= hd.payload_bytes;
        if ((uint32_t)lane < 32) { s_off[lane] = incl - zl; s_z[lane] = zl; }
        if (lane == 0) {
            s_base = base;
            s_ok = ok;
            if (!ok) set_corrupt(p.err);
        }
    }
    __syncthreads();
    if (!s_ok) return;
    const uint64_t base = s_base;
    const uint32_t Tb = cnt ? s_off[cnt - 1] + s_z[cnt - 1] : 0;
    // stage payload bytes [base, base + Tb) with 16-byte loads
    if (Tb) {
        const uint8_t* g0 = in + hd.off_pl + base;
        const uintptr_t A = reinterpret_cast<uintptr_t>(g0) & ~uintptr_t(15);
        const uintptr_t E = reinterpret_cast<uintptr_t>(g0) + Tb;
        const uintptr_t lim = reinterpret_cast<uintptr_t>(in) + p.in_bytes;
        const uint32_t nch = (uint32_t)((E - A + 15) >> 4);
        for (uint32_t ch = threadIdx.x; ch < nch; ch += C::NT) {
            const uintptr_t a = A + 16 * (uintptr_t)ch;
            if (a + 16 <= lim) {
                *reinterpret_cast<uint4*>(stg + 16 * ch) = ld_stream16(reinterpret_cast<const void*>(a));
            } else {
                for (int q = 0; q < 16; q++)
                    stg[16 * ch + q] = (a + q < lim) ? *reinterpret_cast<const uint8_t*>(a + q) : 0;
            }
        }
    }
    __syncthreads();
    const int sb = (int)(reinterpret_cast<uintptr_t>(in + hd.off_pl + base) & 15);
    const U* mus = reinterpret_cast<const U*>(in + p.off_mu);
#pragma unroll
    for (int j = 0; j < C::BPW; j++) {
        const int idx = warp * C::BPW + j;
        const uint64_t k = tile * kTileBlocks + idx;
        if (k >= p.nB) break;
        const int len = (int)umin64(C::B, p.n - k * C::B);
        const T mu = TR::from(mus[k]);
        T v[VPL];
        if (!((word >> idx) & 1u)) {
#pragma unroll
            for (int i = 0; i < VPL; i++) v[i] = mu;  // constant block: retrieve with mu
        } else {
            const uint32_t rank = __popc(word & ((1u << idx) - 1u));
            if (!decode_block<T, VPL>(stg + sb + s_off[rank], s_z[rank], len, mu, v)) {
                if (lane == 0) set_corrupt(p.err);
                continue;
            }
        }
        store_lane<T, VPL>(y, p.n, k, lane, v);
    }
}

}  // namespace szx
