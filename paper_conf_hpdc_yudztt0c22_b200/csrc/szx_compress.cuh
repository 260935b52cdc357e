// szx_compress.cuh -- SZx compression kernels for sm_100a.
//
//   k_block_stats  (K1)  per-block min/max with warp reductions (redux.sync
//                        for 32-bit keys) + NaN flag + global finite range
//                        for REL (footnote 1).  One pass over x.
//   k_classify     (K1b) constant-block test (Alg. 1 l.3-8, R1/R2), mu
//                        array, type bitmap via __ballot_sync, and the
//                        nonconstant-index scan (decoupled look-back).
//   k_encode       (K2+K3+K4 fused) for each nonconstant block: normalise,
//                        Formula 4 R, Formula 5 shift, lead codes with __clz
//                        on 16-byte vector loads, R2 guard, warp-scan of
//                        mid-byte counts, tile look-back for payload offsets,
//                        shared-memory staging and 16-byte packed stores.
//
// A warp owns one data block of b = 32*VPL values: lane l holds values
// [VPL*l, VPL*l + VPL) (contiguous, so one or two 16-byte loads per lane).
// This replaces the paper's thread-per-point mapping: the
// lane's VPL points are processed sequentially in registers and the warp
// communicates only the neighbour word (Solution 2) and one
// prefix scan of mid-byte counts (Solution 1).
#pragma once

#include "szx_device.cuh"

namespace szx {

struct Plan {
    uint64_t n, nB, nW;        // values, blocks, bitmap words (= tiles of 32 blocks)
    uint64_t off_mu;           // stream offset of the mu section
    uint32_t b, dtype, mode;
    int32_t r_bias;
    double eb_user;
    // workspace
    uint64_t* range_keys;      // [2] finite range keys (min, ~max), init 0xFF..
    uint32_t* ctr;             // [4] tile tickets, init 0
    uint64_t* status_b;        // classify look-back, init 0
    uint64_t* status_c;        // encode look-back, init 0
    void* stats;               // 2 words per block
    uint32_t* ncpre;           // exclusive nonconstant count per bitmap word
    double* eb_abs;            // [1]
    uint64_t* nnc;             // [1]
    uint64_t* total;           // [1] stream bytes (output of the call)
};

// Load the VPL values lane `lane` owns in block k.  Returns how many are valid.
template <typename T, int VPL>
__device__ inline int load_lane(const T* __restrict__ x, uint64_t n, uint64_t k, int lane, T (&v)[VPL]) {
    constexpr int B = 32 * VPL;
    const uint64_t first = k * B + (uint64_t)lane * VPL;
    if ((k + 1) * B <= n) {
        constexpr int NV = VPL * (int)sizeof(T) / 16;
        const uint4* p = reinterpret_cast<const uint4*>(x + first);
#pragma unroll
        for (int q = 0; q < NV; q++) {
            uint4 w = ld_stream16(p + q);
            reinterpret_cast<uint4*>(v)[q] = w;
        }
        return VPL;
    }
    int cnt = first >= n ? 0 : (int)umin64(VPL, n - first);
#pragma unroll
    for (int i = 0; i < VPL; i++) v[i] = i < cnt ? x[first + i] : T(0);
    return cnt;
}

// ------------------------------------------------------------------ K1
template <typename T, int VPL, int UNR>
__global__ void __launch_bounds__(256) k_block_stats(const T* __restrict__ x, Plan p, int want_range) {
    using TR = Traits<T>;
    using U = typename TR::U;
    const int lane = threadIdx.x & 31;
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    U* stats = reinterpret_cast<U*>(p.stats);
    uint64_t fmin = ~0ull, fmaxi = ~0ull;  // finite range as double keys: min, ~max

    for (uint64_t k0 = gw * UNR; k0 < p.nB; k0 += nw * UNR) {
        T v[UNR][VPL];
        int cnt[UNR];
#pragma unroll
        for (int u = 0; u < UNR; u++) cnt[u] = (k0 + u < p.nB) ? load_lane<T, VPL>(x, p.n, k0 + u, lane, v[u]) : 0;
#pragma unroll
        for (int u = 0; u < UNR; u++) {
            if (k0 + u >= p.nB) break;
            bool nan = false;
            U kmn = ~U(0), kmx = 0;
#pragma unroll
            for (int i = 0; i < VPL; i++) {
                if (i < cnt[u]) {
                    const T xi = v[u][i];
                    if (TR::isnan_(xi)) {
                        nan = true;
                    } else {
                        const U key = okey(TR::bits(xi));
                        kmn = key < kmn ? key : kmn;
                        kmx = key > kmx ? key : kmx;
                        if (want_range) {
                            const double d = (double)xi;
                            if (d - d == 0.0) {  // finite
                                const uint64_t dk = dkey((uint64_t)__double_as_longlong(d));
                                fmin = dk < fmin ? dk : fmin;
                                fmaxi = ~dk < fmaxi ? ~dk : fmaxi;
                            }
                        }
                    }
                }
            }
            nan = __any_sync(0xffffffffu, nan);
            kmn = warp_min(kmn);
            kmx = warp_max(kmx);
            if (lane == 0) {
                const uint64_t k = k0 + u;
                if (nan) {
                    stats[2 * k] = ~U(0);  // NaN marker (all-ones is a NaN pattern)
                    stats[2 * k + 1] = 0;
                } else {
                    stats[2 * k] = okey_inv(kmn);
                    stats[2 * k + 1] = okey_inv(kmx);
                }
            }
        }
    }
    if (want_range) {
        __shared__ uint64_t s_r[2][8];
        fmin = warp_min(fmin);
        fmaxi = warp_min(fmaxi);
        const int w = threadIdx.x >> 5;
        if (lane == 0) { s_r[0][w] = fmin; s_r[1][w] = fmaxi; }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int i = 1; i < (int)(blockDim.x >> 5); i++) {
                fmin = s_r[0][i] < fmin ? s_r[0][i] : fmin;
                fmaxi = s_r[1][i] < fmaxi ? s_r[1][i] : fmaxi;
            }
            if (fmin != ~0ull) atomicMin((unsigned long long*)&p.range_keys[0], (unsigned long long)fmin);
            if (fmaxi != ~0ull) atomicMin((unsigned long long*)&p.range_keys[1], (unsigned long long)fmaxi);
        }
    }
}

// Formula 4 under reading R3, then the test hook r_bias, clamped.
template <typename T>
__device__ inline int initial_R(T r, int pe, int r_bias) {
    using TR = Traits<T>;
    const int gap = TR::expo(r) - pe;
    int R = gap <= 0 ? TR::kFloor : (gap >= TR::kFull - TR::kFloor ? TR::kFull : TR::kFloor + gap);
    R += r_bias;
    R = R < TR::kFloor ? TR::kFloor : R;
    R = R > TR::kFull ? TR::kFull : R;
    return R;
}

// Block statistics -> (constant?, mu, r).  Alg. 1 line 3-4 with R1/R2.
template <typename T>
struct BlockClass {
    bool nan, constant;
    T mu, r;
};
template <typename T>
__device__ inline BlockClass<T> classify(typename Traits<T>::U smn, typename Traits<T>::U smx, double eb) {
    using TR = Traits<T>;
    BlockClass<T> c;
    const T mn = TR::from(smn), mx = TR::from(smx);
    c.nan = TR::isnan_(mn);
    c.constant = false;
    c.mu = T(0);
    c.r = T(0);
    if (!c.nan) {
        c.r = TR::half(TR::sub(mx, mn));   // radius r_k (R1)
        c.mu = TR::add(mn, c.r);           // mu_k = mn + r (R1)
        c.constant = ((double)c.r <= eb) && (__dsub_rn((double)mx, (double)c.mu) <= eb) &&
                     (__dsub_rn((double)c.mu, (double)mn) <= eb);  // R2 guard
    }
    return c;
}

// ------------------------------------------------------------------ K1b
// One thread per block, 256 blocks (8 bitmap words) per CTA tile.
template <typename T>
__global__ void __launch_bounds__(256) k_classify(Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    __shared__ uint64_t s_tile;
    __shared__ uint32_t s_cnt[8];
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[0], 1u);
    __syncthreads();
    const uint64_t tile = s_tile;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t k = tile * 256 + threadIdx.x;
    const double eb = eb_from_range(p.mode, p.eb_user, p.range_keys);
    const int pe = expo_f64(eb);
    const U* stats = reinterpret_cast<const U*>(p.stats);

    bool nc = false;
    if (k < p.nB) {
        BlockClass<T> c = classify<T>(stats[2 * k], stats[2 * k + 1], eb);
        T mu = c.mu;
        if (!c.constant) {
            nc = true;
            if (c.nan || initial_R<T>(c.r, pe, p.r_bias) >= TR::kFull) mu = T(0);  // raw block: mu = +0 (R15)
        }
        reinterpret_cast<U*>(out + p.off_mu)[k] = TR::bits(mu);
    }
    const uint32_t word = __ballot_sync(0xffffffffu, nc);
    const uint64_t widx = tile * 8 + warp;
    if (lane == 0) {
        if (widx < p.nW) reinterpret_cast<uint32_t*>(out + kHeaderBytes)[widx] = word;
        s_cnt[warp] = __popc(word);
    }
    __syncthreads();
    if (warp == 0) {
        const uint32_t c = lane < 8 ? s_cnt[lane] : 0;
        const uint32_t incl = warp_incl_scan(c);
        const uint32_t agg = __shfl_sync(0xffffffffu, incl, 31);
        const uint64_t excl = lookback_exclusive(p.status_b, tile, agg);
        if (lane < 8 && tile * 8 + lane < p.nW) p.ncpre[tile * 8 + lane] = (uint32_t)(excl + incl - c);
        const uint64_t ntiles = (p.nB + 255) / 256;
        if (tile == ntiles - 1 && lane == 0) {
            const uint64_t nnc = excl + agg;
            *p.nnc = nnc;
            *p.eb_abs = eb;
            // zero the padding of the bitmap, mu and zsize sections
            const uint64_t bm_end = kHeaderBytes + 4 * p.nW;
            const uint64_t bm_pad = kHeaderBytes + al16((p.nB + 7) / 8);
            for (uint64_t a = bm_end; a < bm_pad; a++) out[a] = 0;
            const uint64_t mu_end = p.off_mu + (uint64_t)TR::W * p.nB;
            const uint64_t off_zs = p.off_mu + al16((uint64_t)TR::W * p.nB);
            for (uint64_t a = mu_end; a < off_zs; a++) out[a] = 0;
            for (uint64_t a = off_zs + 2 * nnc; a < off_zs + al16(2 * nnc); a++) out[a] = 0;
        }
    }
}

// ------------------------------------------------------------------ K2
// Encode one nonconstant block held by the warp.  Returns z_k (warp-uniform)
// and leaves the shifted words, lead codes and per-lane mid-byte offsets in
// registers for the packing stage.
template <typename T, int VPL>
struct LaneCode {
    typename Traits<T>::U u[VPL];  // shifted words (Formula 5)
    uint32_t leads;                // 2 bits per value
    uint32_t mexcl;                // exclusive mid-byte offset of this lane
    int R;
    uint32_t z;
};

template <typename T, int VPL>
__device__ inline void encode_block(const T (&xv)[VPL], int cnt, int len, const BlockClass<T>& c,
                                    double eb, int pe, int r_bias, LaneCode<T, VPL>& lc) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    int R = c.nan ? TR::kFull : initial_R<T>(c.r, pe, r_bias);
    T mu = c.mu;
    int s, req;
    bool raw;
    for (;;) {
        raw = R >= TR::kFull;
        if (raw) { R = TR::kFull; mu = T(0); }
        s = raw ? 0 : ((8 - (R & 7)) & 7);
        req = (R + s) >> 3;
        const U keep = raw ? ~U(0) : ~((U(1) << (8 * W - R)) - U(1));
        bool ok = true;
#pragma unroll
        for (int i = 0; i < VPL; i++) {
            const U vb = raw ? TR::bits(xv[i]) : TR::bits(TR::sub(xv[i], mu));  // v_i = d_i - mu
            lc.u[i] = vb >> s;                                                  // Solution C shift
            if (!raw && i < cnt) {
                // R2 guard: reconstruct exactly as the decoder does, check Formula 1
                const T xp = TR::add(TR::from(vb & keep), mu);
                ok &= fabs(__dsub_rn((double)xv[i], (double)xp)) <= eb;
            }
        }
        if (raw || __all_sync(0xffffffffu, ok)) break;
        R += 1;
    }
    // identical leading bytes vs the previous value (u_{-1} = 0, R6)
    U prev = __shfl_up_sync(0xffffffffu, lc.u[VPL - 1], 1);
    if (lane == 0) prev = 0;
    uint32_t leads = 0, m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        if (i < cnt) {
            int L = TR::clz(lc.u[i] ^ prev) >> 3;
            L = L > 3 ? 3 : L;
            leads |= (uint32_t)L << (2 * i);
            m += req > L ? req - L : 0;
            prev = lc.u[i];
        }
    }
    const uint32_t incl = warp_incl_scan(m);
    lc.leads = leads;
    lc.mexcl = incl - m;
    lc.R = R;
    lc.z = 1 + (uint32_t)((len + 3) / 4) + __shfl_sync(0xffffffffu, incl, 31);
}

// Write the block payload [R][codes][mid-bytes] into shared memory at dst.
template <typename T, int VPL>
__device__ inline void pack_block(const LaneCode<T, VPL>& lc, int cnt, int len, uint8_t* dst) {
    using TR = Traits<T>;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    const int ncode = (len + 3) / 4;
    const bool raw = lc.R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (lc.R & 7)) & 7);
    const int req = (lc.R + s) >> 3;
    if (lane == 0) dst[0] = (uint8_t)lc.R;
    // code bytes: lane l owns bytes [l*VPL/4, (l+1)*VPL/4)  (R8: LSB-first)
#pragma unroll
    for (int q = 0; q < VPL / 4; q++) {
        const int cb = lane * (VPL / 4) + q;
        if (cb < ncode) dst[1 + cb] = (uint8_t)(lc.leads >> (8 * q));
    }
    // mid-bytes: bytes [W-req, W-lead) of each little-endian word (R7)
    uint8_t* mb = dst + 1 + ncode + lc.mexcl;
    int pos = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        if (i < cnt) {
            const int L = (lc.leads >> (2 * i)) & 3;
            for (int j = W - req; j < W - L; j++) mb[pos++] = (uint8_t)(lc.u[i] >> (8 * j));
        }
    }
}

// ------------------------------------------------------------------ K2+K3+K4
template <typename T, int VPL>
struct EncodeCfg {
    static constexpr int B = 32 * VPL;
    static constexpr int BPW = VPL == 4 ? 4 : 2;             // blocks per warp
    static constexpr int NWARP = kTileBlocks / BPW;
    static constexpr int NT = NWARP * 32;
    static constexpr int MAXZ = 1 + B / 4 + Traits<T>::W * B;  // max z_k
    static constexpr int SMEM = 16 + kTileBlocks * MAXZ + 16;
};

template <typename T, int VPL>
__global__ void __launch_bounds__(EncodeCfg<T, VPL>::NT)
    k_encode(const T* __restrict__ x, Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = EncodeCfg<T, VPL>;
    constexpr int W = TR::W;
    extern __shared__ __align__(16) uint8_t stg[];
    __shared__ uint32_t s_z[kTileBlocks], s_off[kTileBlocks];
    __shared__ uint64_t s_tile, s_G;
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[1], 1u);
    __syncthreads();
    const uint64_t tile = s_tile;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t word = reinterpret_cast<const uint32_t*>(out + kHeaderBytes)[tile];
    const uint32_t ncb = p.ncpre[tile];
    const double eb = *p.eb_abs;
    const int pe = expo_f64(eb);
    const uint64_t nnc = *p.nnc;
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    const uint64_t off_pl = off_zs + al16(2 * nnc);
    const U* stats = reinterpret_cast<const U*>(p.stats);

    // ---- phase 1: load + encode this warp's blocks (constant blocks are skipped: no reads)
    T xv[C::BPW][VPL];
    int cnt[C::BPW];
#pragma unroll
    for (int j = 0; j < C::BPW; j++) {
        const int idx = warp * C::BPW + j;
        const uint64_t k = tile * kTileBlocks + idx;
        cnt[j] = 0;
        if (k < p.nB && ((word >> idx) & 1u)) cnt[j] = load_lane<T, VPL>(x, p.n, k, lane, xv[j]);
    }
    LaneCode<T, VPL> lc[C::BPW];
#pragma unroll
    for (int j = 0; j < C::BPW; j++) {
        const int idx = warp * C::BPW + j;
        const uint64_t k = tile * kTileBlocks + idx;
        uint32_t z = 0;
        if (k < p.nB && ((word >> idx) & 1u)) {
            const int len = (int)umin64(C::B, p.n - k * C::B);
            BlockClass<T> c = classify<T>(stats[2 * k], stats[2 * k + 1], eb);
            encode_block<T, VPL>(xv[j], cnt[j], len, c, eb, pe, p.r_bias, lc[j]);
            z = lc[j].z;
            if (lc[j].R >= TR::kFull && lane == 0) reinterpret_cast<U*>(out + p.off_mu)[k] = 0;
        }
        if (lane == 0) s_z[idx] = z;
    }
    __syncthreads();

    // ---- phase 2: tile scan + decoupled look-back for the payload offset
    if (warp == 0) {
        const uint32_t z = s_z[lane];
        const uint32_t incl = warp_incl_scan(z);
        s_off[lane] = incl - z;
        const uint32_t agg = __shfl_sync(0xffffffffu, incl, 31);
        const uint64_t G = lookback_exclusive(p.status_c, tile, agg);
        if (lane == 0) {
            s_G = G;
            if (tile == p.nW - 1) {
                const uint64_t pbytes = G + agg;
                uint64_t* h = reinterpret_cast<uint64_t*>(out);
                h[0] = 0x31585A53ull | (1ull << 32) | ((uint64_t)p.dtype << 40) | ((uint64_t)p.mode << 48);
                h[1] = (uint64_t)p.b;
                h[2] = p.n;
                h[3] = (uint64_t)__double_as_longlong(p.eb_user);
                h[4] = (uint64_t)__double_as_longlong(eb);
                h[5] = nnc;
                h[6] = pbytes;
                h[7] = 0;
                *p.total = off_pl + pbytes;
            }
        }
    }
    __syncthreads();
    const uint64_t G = s_G;
    const int sb = (int)(G & 15);

    // ---- phase 3: pack payloads into shared memory, write zsize
#pragma unroll
    for (int j = 0; j < C::BPW; j++) {
        const int idx = warp * C::BPW + j;
        const uint64_t k = tile * kTileBlocks + idx;
        if (k < p.nB && ((word >> idx) & 1u)) {
            const int len = (int)umin64(C::B, p.n - k * C::B);
            pack_block<T, VPL>(lc[j], cnt[j], len, stg + sb + s_off[idx]);
            if (lane == 0) {
                const uint32_t rank = __popc(word & ((1u << idx) - 1u));
                reinterpret_cast<uint16_t*>(out + off_zs)[ncb + rank] = (uint16_t)lc[j].z;
            }
        }
    }
    __syncthreads();

    // ---- phase 4: copy the staged tile payload to global with 16-byte stores
    const uint32_t T_bytes = s_off[kTileBlocks - 1] + s_z[kTileBlocks - 1];
    uint8_t* g0 = out + off_pl + G;
    const uintptr_t A = reinterpret_cast<uintptr_t>(g0) & ~uintptr_t(15);
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(g0), E = a0 + T_bytes;
    const uint32_t nch = (uint32_t)((E - A + 15) >> 4);
    for (uint32_t ch = threadIdx.x; ch < nch; ch += C::NT) {
        const uintptr_t a = A + 16 * (uintptr_t)ch;
        if (a >= a0 && a + 16 <= E) {
            *reinterpret_cast<uint4*>(a) = *reinterpret_cast<const uint4*>(stg + 16 * ch);
        } else {
            for (int q = 0; q < 16; q++)
                if (a + q >= a0 && a + q < E) *reinterpret_cast<uint8_t*>(a + q) = stg[16 * ch + q];
        }
    }
}

__global__ void k_empty_header(uint8_t* out, uint32_t dtype, uint32_t mode, uint32_t b, double eb_user,
                               uint64_t* total) {
    uint64_t* h = reinterpret_cast<uint64_t*>(out);
    h[0] = 0x31585A53ull | (1ull << 32) | ((uint64_t)dtype << 40) | ((uint64_t)mode << 48);
    h[1] = b;
    h[2] = 0;
    h[3] = (uint64_t)__double_as_longlong(eb_user);
    h[4] = 0;  // eb_abs: ABS -> eb (set below); REL with no values -> 0
    if (mode == 0) { double e = eb_user; if (e == 0.0) e = 0.0; h[4] = (uint64_t)__double_as_longlong(e); }
    h[5] = 0;
    h[6] = 0;
    h[7] = 0;
    if (total) *total = 64;
}

}  // namespace szx
