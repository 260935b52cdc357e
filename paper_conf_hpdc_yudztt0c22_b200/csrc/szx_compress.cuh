// szx_compress.cuh -- SZx compression kernels for sm_100a.
//
//   k_block_stats  (K1)  one streaming read of x: per-block min/max as
//                        order-preserving integer keys (warp redux.sync), and
//                        the global finite range for REL (footnote 1,
//                        P:L929-938).  NaN needs no per-element test: a NaN
//                        key lies outside [key(-Inf), key(+Inf)].
//   k_classify     (K1b) constant-block test from the block keys alone
//                        (Alg. 1 l.3-8 with R1/R2), mu array, type bitmap via
//                        __ballot_sync, nonconstant-count scan (decoupled
//                        look-back) that also writes the compacted list of
//                        nonconstant block ids, and the stream header.
//   k_encode       (K2+K3+K4 fused, persistent, warp-specialised) a producer
//                        warp streams the nonconstant blocks of each tile
//                        into a shared-memory ring with TMA bulk copies
//                        (cp.async.bulk + mbarrier); 8 consumer warps encode
//                        them: normalise, Formula 4 R, Formula 5 shift, lead
//                        codes with __clz, R2 guard, warp scan of mid-byte
//                        counts, tile look-back for the payload offset,
//                        shared-memory packing, 16-byte stores.
//
// Constant blocks are never read twice: after k_block_stats only the
// nonconstant blocks are fetched again.  A warp owns one data block of
// b = 32*VPL values: lane l holds values [VPL*l, VPL*l + VPL), so one or two
// 16-byte accesses per lane.  This replaces the paper's thread-per-point
// mapping: a lane's VPL points are processed sequentially in
// registers and the warp exchanges only the neighbour word (Solution 2,
// P:L2687-2693) and one prefix scan of mid-byte counts (Solution 1,
// P:L2497-2632).
#pragma once

#include "szx_device.cuh"

namespace szx {

struct Plan {
    uint64_t n, nB, nW;        // values, blocks, bitmap words
    uint64_t off_mu;           // stream offset of the mu section
    uint32_t b, dtype, mode;
    int32_t r_bias;
    double eb_user;
    // workspace
    uint64_t* range_keys;      // [2] finite range keys (min, ~max), init 0xFF..
    uint32_t* ctr;             // [4] tile tickets, init 0
    uint64_t* status_b;        // classify look-back, init 0
    uint64_t* status_c;        // encode look-back, init 0
    void* stats;               // 2 keys per block (min, max)
    uint32_t* nclist;          // ids of the nonconstant blocks, in block order
    void* ncmu;                // their mu (bits), same order
    uint8_t* ncR;              // classify: R_init | proven << 7; size pass: final R
    uint64_t* gbase;           // payload offset of each write tile (+ total)
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
        for (int q = 0; q < NV; q++) reinterpret_cast<uint4*>(v)[q] = ld_stream16(p + q);
        return VPL;
    }
    int cnt = first >= n ? 0 : (int)umin64(VPL, n - first);
#pragma unroll
    for (int i = 0; i < VPL; i++) v[i] = i < cnt ? x[first + i] : T(0);
    return cnt;
}

template <typename U>
__device__ inline U umin_(U a, U b) { return a < b ? a : b; }
template <typename U>
__device__ inline U umax_(U a, U b) { return a > b ? a : b; }

// ------------------------------------------------------------------ K1
template <typename T, int VPL, int UNR>
__global__ void __launch_bounds__(256) k_block_stats(const T* __restrict__ x, Plan p, int want_range) {
    using TR = Traits<T>;
    using U = typename TR::U;
    const int lane = threadIdx.x & 31;
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    U* stats = reinterpret_cast<U*>(p.stats);
    U fmin = ~U(0), fmax = 0;  // finite range (keys), warp-uniform

    // one block's keys -> stats and the finite range (all lanes; keys exact,
    // NaN lies outside [key(-Inf), key(+Inf)] and is detected by k_classify)
    auto block = [&](const T (&v)[VPL], int cnt, uint64_t k) {
        U kmn = ~U(0), kmx = 0;
#pragma unroll
        for (int i = 0; i < VPL; i++) {
            const U key = okey(TR::bits(v[i]));
            kmn = i < cnt ? umin_(kmn, key) : kmn;
            kmx = i < cnt ? umax_(kmx, key) : kmx;
        }
        kmn = warp_min(kmn);
        kmx = warp_max(kmx);
        if (lane == 0) {
            stats[2 * k] = kmn;
            stats[2 * k + 1] = kmx;
        }
        if (want_range) {
            if (kmn > TR::kKeyNInf && kmx < TR::kKeyPInf) {
                fmin = umin_(fmin, kmn);
                fmax = umax_(fmax, kmx);
            } else {  // the block holds +-Inf or NaN: finite extremes value by value (rare)
                U a = ~U(0), b = 0;
#pragma unroll
                for (int i = 0; i < VPL; i++) {
                    const U key = okey(TR::bits(v[i]));
                    if (i < cnt && key > TR::kKeyNInf && key < TR::kKeyPInf) {
                        a = umin_(a, key);
                        b = umax_(b, key);
                    }
                }
                fmin = umin_(fmin, warp_min(a));
                fmax = umax_(fmax, warp_max(b));
            }
        }
    };
    constexpr int B = 32 * VPL;
    constexpr int NV = VPL * (int)sizeof(T) / 16;   // 16-byte loads per lane per block
    const uint64_t nBf = p.n / B;                    // full blocks
    uint64_t k0 = gw * UNR;
    // fast path: UNR full blocks per warp, all loads issued first, no bounds checks
    for (; k0 + UNR <= nBf; k0 += nw * UNR) {
        const uint4* src = reinterpret_cast<const uint4*>(x + k0 * B) + lane * NV;
        T v[UNR][VPL];
#pragma unroll
        for (int u = 0; u < UNR; u++)
#pragma unroll
            for (int q = 0; q < NV; q++) reinterpret_cast<uint4*>(v[u])[q] = ld_stream16(src + u * (B / 4 * sizeof(T) / 4) + q);
#pragma unroll
        for (int u = 0; u < UNR; u++) block(v[u], VPL, k0 + u);
    }
    // remaining blocks (partial group, tail block): one at a time
    for (; k0 < p.nB; k0 += nw * UNR) {
#pragma unroll 1
        for (int u = 0; u < UNR && k0 + u < p.nB; u++) {
            T v[VPL];
            const int cnt = load_lane<T, VPL>(x, p.n, k0 + u, lane, v);
            block(v, cnt, k0 + u);
        }
    }
    if (want_range) {
        __shared__ U s_r[2][8];
        const int w = threadIdx.x >> 5;
        if (lane == 0) { s_r[0][w] = fmin; s_r[1][w] = fmax; }
        __syncthreads();
        if (threadIdx.x == 0) {
            for (int i = 1; i < (int)(blockDim.x >> 5); i++) {
                fmin = umin_(fmin, s_r[0][i]);
                fmax = umax_(fmax, s_r[1][i]);
            }
            if (fmin != ~U(0)) {  // convert to keys of the double value (exact widening)
                const double dmn = (double)TR::from(okey_inv(fmin)), dmx = (double)TR::from(okey_inv(fmax));
                const uint64_t kmn = dkey((uint64_t)__double_as_longlong(dmn));
                const uint64_t kmx = dkey((uint64_t)__double_as_longlong(dmx));
                atomicMin((unsigned long long*)&p.range_keys[0], (unsigned long long)kmn);
                atomicMin((unsigned long long*)&p.range_keys[1], (unsigned long long)~kmx);
            }
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

// Block keys -> (NaN?, constant?, mu, r).  Alg. 1 lines 3-4 with R1/R2.
template <typename T>
struct BlockClass {
    bool nan, constant;
    T mu, r, mn, mx;
};
template <typename T>
__device__ inline BlockClass<T> classify(typename Traits<T>::U kmn, typename Traits<T>::U kmx, double eb,
                                         bool test_constant = true) {
    using TR = Traits<T>;
    BlockClass<T> c;
    c.nan = kmn < TR::kKeyNInf || kmx > TR::kKeyPInf;  // R14
    c.constant = false;
    c.mu = c.r = c.mn = c.mx = T(0);
    if (!c.nan) {
        c.mn = TR::from(okey_inv(kmn));
        c.mx = TR::from(okey_inv(kmx));
        c.r = TR::half(TR::sub(c.mx, c.mn));   // radius r_k (R1)
        c.mu = TR::add(c.mn, c.r);             // mu_k = mn + r (R1)
        if (test_constant)
            c.constant = ((double)c.r <= eb) && (__dsub_rn((double)c.mx, (double)c.mu) <= eb) &&
                         (__dsub_rn((double)c.mu, (double)c.mn) <= eb);  // R2 guard
    }
    return c;
}

// 2^n as a double for n in [-1074, 1023] (exact; subnormal below -1022)
__device__ inline double pow2d(int n) {
    if (n >= -1022) return __longlong_as_double((long long)(n + 1023) << 52);
    return n >= -1074 ? __longlong_as_double(1ll << (n + 1074)) : 0.0;
}

// Per-block proof that the R2 per-element check cannot fail for R kept bits
// (DESIGN.md s.3, R2): with E_v <= p(r) and k = R - floor kept mantissa bits,
//   |x - x'| < 2^(p(r)-k) [truncation] + 2^(E_v-P) [v = fl(x-mu)]
//            + 2^(E_x'-P) [x' = fl(v'+mu)]  <=  2^p(e) + slack = e
// when p(r)-k <= p(e) and 2*max(2nd, 3rd term) <= slack = e - 2^p(e) (exact).
// If it does not hold the kernel evaluates the check value by value, exactly
// like the oracle, so the stream never depends on this shortcut.
template <typename T>
__device__ inline bool guard_proven(const BlockClass<T>& c, double eb, int pe, int R) {
    using TR = Traits<T>;
    constexpr int P = sizeof(T) == 4 ? 24 : 53;          // significand bits
    constexpr int EMIN = sizeof(T) == 4 ? -126 : -1022;  // smallest normal exponent
    const int pr = TR::expo(c.r);
    if (c.nan || pr < EMIN || pr >= (sizeof(T) == 4 ? 128 : 1024)) return false;
    const T v1 = fabs(TR::sub(c.mx, c.mu)), v2 = fabs(TR::sub(c.mn, c.mu));
    if (TR::expo(v1 > v2 ? v1 : v2) > pr) return false;
    if (pr - (R - TR::kFloor) > pe) return false;
    const T a1 = fabs(c.mn), a2 = fabs(c.mx);
    int ex = TR::expo(a1 > a2 ? a1 : a2) + 1;
    ex = ex < EMIN ? EMIN : ex;
    const int t2 = (pr > EMIN ? pr : EMIN) - P, t3 = ex - P;
    const double slack = __dsub_rn(eb, pow2d(pe));
    return pow2d((t2 > t3 ? t2 : t3) + 1) <= slack;
}

__device__ inline void write_header(uint8_t* out, const Plan& p, double eb, uint64_t nnc, uint64_t pbytes) {
    uint64_t* h = reinterpret_cast<uint64_t*>(out);
    h[0] = 0x31585A53ull | (1ull << 32) | ((uint64_t)p.dtype << 40) | ((uint64_t)p.mode << 48);  // "SZX1" v1
    h[1] = (uint64_t)p.b;
    h[2] = p.n;
    h[3] = (uint64_t)__double_as_longlong(p.eb_user);
    h[4] = (uint64_t)__double_as_longlong(eb);
    h[5] = nnc;
    h[6] = pbytes;
    h[7] = 0;
}

// ------------------------------------------------------------------ K1b
// 256 threads x 8 blocks = 2048 blocks (64 bitmap words) per CTA tile.
constexpr int kClassifyBlocks = 2048;

template <typename T>
__global__ void __launch_bounds__(256) k_classify(Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    __shared__ uint64_t s_tile, s_base;
    __shared__ uint32_t s_cnt[64], s_pre[64];
    pdl_wait();
    pdl_trigger();
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[0], 1u);
    __syncthreads();
    const uint64_t tile = s_tile;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t base = tile * kClassifyBlocks;
    const double eb = eb_from_range(p.mode, p.eb_user, p.range_keys);
    const int pe = expo_f64(eb);
    const U* stats = reinterpret_cast<const U*>(p.stats);
    uint32_t* bitmap = reinterpret_cast<uint32_t*>(out + kHeaderBytes);
    U* mus = reinterpret_cast<U*>(out + p.off_mu);

    uint32_t ncmask = 0;
    U rmu[8];
    uint32_t rrec[2] = {0u, 0u};  // per j: R_init | guard_proven << 7 (one byte each)
#pragma unroll
    for (int j = 0; j < 8; j++) {
        const uint64_t k = base + j * 256 + threadIdx.x;
        bool nc = false;
        rmu[j] = 0;
        if (k < p.nB) {
            BlockClass<T> c = classify<T>(stats[2 * k], stats[2 * k + 1], eb);
            T mu = c.mu;
            if (!c.constant) {
                nc = true;
                // the per-block scalar work of the encoder is done here once per
                // block (one thread) instead of once per lane of the encoding warp
                const int R = c.nan ? TR::kFull : initial_R<T>(c.r, pe, p.r_bias);
                if (R >= TR::kFull) mu = T(0);  // raw: mu = +0 (R15)
                const bool proven = R < TR::kFull && guard_proven<T>(c, eb, pe, R);
                rrec[j >> 2] |= (uint32_t)(R | (proven ? 0x80 : 0)) << (8 * (j & 3));
            }
            rmu[j] = TR::bits(mu);
            mus[k] = TR::bits(mu);
        }
        const uint32_t word = __ballot_sync(0xffffffffu, nc);
        if (lane == 0) {
            const uint64_t widx = (base >> 5) + j * 8 + warp;
            if (widx < p.nW) bitmap[widx] = word;
            s_cnt[j * 8 + warp] = __popc(word);
        }
        ncmask |= (uint32_t)nc << j;
    }
    __syncthreads();
    if (warp == 0) {
        const uint32_t c0 = s_cnt[2 * lane], c1 = s_cnt[2 * lane + 1];
        const uint32_t incl = warp_incl_scan(c0 + c1);
        const uint32_t ex = incl - c0 - c1;
        s_pre[2 * lane] = ex;
        s_pre[2 * lane + 1] = ex + c0;
        const uint32_t agg = __shfl_sync(0xffffffffu, incl, 31);
        const uint64_t G = lookback_exclusive(p.status_b, tile, agg);
        if (lane == 0) {
            s_base = G;
            const uint64_t ntiles = (p.nB + kClassifyBlocks - 1) / kClassifyBlocks;
            if (tile == ntiles - 1) {
                const uint64_t nnc = G + agg;
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
                // header; k_encode's last tile fills in the payload size
                write_header(out, p, eb, nnc, 0);
                *p.total = off_zs + al16(2 * nnc);
            }
        }
    }
    __syncthreads();
    const uint64_t G = s_base;
    U* ncmu = reinterpret_cast<U*>(p.ncmu);
#pragma unroll
    for (int j = 0; j < 8; j++) {
        const bool nc = (ncmask >> j) & 1u;
        const uint32_t word = __ballot_sync(0xffffffffu, nc);
        if (nc) {
            const uint64_t k = base + j * 256 + threadIdx.x;
            const uint64_t idx = G + s_pre[j * 8 + warp] + __popc(word & ((1u << lane) - 1u));
            p.nclist[idx] = (uint32_t)k;
            ncmu[idx] = rmu[j];
            p.ncR[idx] = (uint8_t)(rrec[j >> 2] >> (8 * (j & 3)));
        }
    }
}

// ------------------------------------------------------------------ K2
// Encode one nonconstant block held by the warp.  Leaves the shifted words,
// lead codes and this lane's mid-byte offset in registers for packing.
struct LaneCode {
    uint32_t leads;                // 2 bits per value
    uint32_t mexcl;                // exclusive mid-byte offset of this lane
    int R;
    uint32_t z;
};

template <typename T, int VPL>
__device__ inline void encode_block(const T (&xv)[VPL], int cnt, int len, T mu, int R, bool proven,
                                    double eb, typename Traits<T>::U (&u)[VPL], LaneCode& lc) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    int s, req;
    bool raw;
    bool check = !proven;
    for (;;) {
        raw = R >= TR::kFull;
        if (raw) { R = TR::kFull; mu = T(0); }
        s = raw ? 0 : ((8 - (R & 7)) & 7);
        req = (R + s) >> 3;
#pragma unroll
        for (int i = 0; i < VPL; i++)  // v_i = d_i - mu, then the Solution C shift
            u[i] = (raw ? TR::bits(xv[i]) : TR::bits(TR::sub(xv[i], mu))) >> s;
        if (raw || !check) break;
        // R2 guard (warp-uniform branch): reconstruct exactly as the decoder does
        // and check Formula 1 value by value
        const U keep = ~((U(1) << (8 * W - R)) - U(1));
        bool ok = true;
#pragma unroll
        for (int i = 0; i < VPL; i++) {
            if (i < cnt) {
                const T xp = TR::add(TR::from((u[i] << s) & keep), mu);
                ok &= fabs(__dsub_rn((double)xv[i], (double)xp)) <= eb;
            }
        }
        if (__all_sync(0xffffffffu, ok)) break;
        R += 1;
    }
    // identical leading bytes vs the previous value (u_{-1} = 0, R6)
    U prev = __shfl_up_sync(0xffffffffu, u[VPL - 1], 1);
    if (lane == 0) prev = 0;
    uint32_t leads = 0, m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        if (i < cnt) {
            int L = TR::clz(u[i] ^ prev) >> 3;
            L = L > 3 ? 3 : L;
            leads |= (uint32_t)L << (2 * i);
            m += req > L ? req - L : 0;
            prev = u[i];
        }
    }
    const uint32_t incl = warp_incl_scan(m);
    lc.leads = leads;
    lc.mexcl = incl - m;
    lc.R = R;
    lc.z = 1 + (uint32_t)((len + 3) / 4) + __shfl_sync(0xffffffffu, incl, 31);
}

// Size of one FULL nonconstant block (the size pass needs z_k and the final
// R only): same R / guard / escalation as encode_block, but the mid-byte
// count is a warp sum (one REDUX) instead of a scan and no codes are kept.
template <typename T, int VPL>
__device__ inline uint32_t size_block(const T (&xv)[VPL], T mu, int& R, bool proven, double eb) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    int s, req;
    bool raw;
    bool check = !proven;
    U u[VPL];
    for (;;) {
        raw = R >= TR::kFull;
        if (raw) { R = TR::kFull; mu = T(0); }
        s = raw ? 0 : ((8 - (R & 7)) & 7);
        req = (R + s) >> 3;
#pragma unroll
        for (int i = 0; i < VPL; i++) u[i] = (raw ? TR::bits(xv[i]) : TR::bits(TR::sub(xv[i], mu))) >> s;
        if (raw || !check) break;
        const U keep = ~((U(1) << (8 * W - R)) - U(1));
        bool ok = true;
#pragma unroll
        for (int i = 0; i < VPL; i++) {
            const T xp = TR::add(TR::from((u[i] << s) & keep), mu);
            ok &= fabs(__dsub_rn((double)xv[i], (double)xp)) <= eb;
        }
        if (__all_sync(0xffffffffu, ok)) break;
        R += 1;
    }
    U prev = __shfl_up_sync(0xffffffffu, u[VPL - 1], 1);
    if (lane == 0) prev = 0;
    uint32_t m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        int L = TR::clz(u[i] ^ prev) >> 3;
        L = L > 3 ? 3 : L;
        m += req > L ? req - L : 0;
        prev = u[i];
    }
    return 1 + (uint32_t)(8 * VPL) + warp_sum(m);
}

// Write a block payload with shared-memory OR reductions into a zero-filled
// staging area: every byte of [R][codes][mid-bytes] is OR-ed into its 32-bit
// word, so neighbouring values, lanes and blocks may share boundary words
// without byte stores or run assembly.  dst is the shared-memory address of
// the block payload; values [0, cnt) of the lane are valid, len in the block.
__device__ inline void red_or_s(uint32_t a, uint32_t v) {
    asm volatile("red.shared.or.b32 [%0], %1;" ::"r"(a), "r"(v) : "memory");
}
__device__ inline void red_or_byte(uint32_t a, uint32_t v) { red_or_s(a & ~3u, (v & 0xFFu) << (8 * (a & 3u))); }

template <typename T, int VPL>
__device__ inline void pack_red(const typename Traits<T>::U (&u)[VPL], const LaneCode& lc, int cnt, int len,
                                uint32_t dst) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    const int ncode = (len + 3) / 4;
    const bool raw = lc.R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (lc.R & 7)) & 7);
    const int req = (lc.R + s) >> 3;
    if (lane == 0) red_or_byte(dst, (uint32_t)lc.R);
#pragma unroll
    for (int q = 0; q < VPL / 4; q++) {
        const int cb = lane * (VPL / 4) + q;
        if (cb < ncode) red_or_byte(dst + 1 + cb, lc.leads >> (8 * q));
    }
    uint32_t a = dst + 1 + ncode + lc.mexcl;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const int L = (lc.leads >> (2 * i)) & 3;
        const int mi = req > L ? req - L : 0;
        if (i < cnt && mi > 0) {
            // the mid-bytes: bytes [W-req, W-L) of the word, brought down to byte 0
            const U chunk = (U)(u[i] << (8 * L)) >> (8 * (W - req + L));
            const uint32_t sh = 8 * (a & 3u), wa = a & ~3u;
            const uint32_t c0 = (uint32_t)chunk;
            if (W == 4) {
                red_or_s(wa, c0 << sh);
                const uint32_t w1 = __funnelshift_l(c0, 0u, sh);
                if (w1) red_or_s(wa + 4, w1);
            } else {
                const uint32_t c1 = (uint32_t)((uint64_t)chunk >> 32);
                red_or_s(wa, c0 << sh);
                const uint32_t w1 = __funnelshift_l(c0, c1, sh), w2 = __funnelshift_l(c1, 0u, sh);
                if (w1) red_or_s(wa + 4, w1);
                if (w2) red_or_s(wa + 8, w2);
            }
            a += mi;
        }
    }
}

// ------------------------------------------------------------------ K2 size pass
// For every nonconstant block (compacted list): encode (Formula 4 R, R2
// guard / escalation), write z_k into the stream's zsize section and the
// final R into the workspace.  A warp owns a contiguous run of the list; it
// fetches the block metadata 32 blocks per round trip and stages the values
// of NB blocks at a time in shared memory with cp.async, double-buffered, so
// the loads of batch b+1 overlap the encoding of batch b.
template <typename T, int VPL>
struct SizeCfg {
    static constexpr int W = Traits<T>::W;
    static constexpr int B = 32 * VPL;
    static constexpr int BW = B * W;
    static constexpr int QV = VPL * W / 16;      // 16-byte chunks per lane per block
    static constexpr int NB = 4;                 // blocks per batch
    static constexpr int WARP_BYTES = 2 * NB * BW;
    static constexpr int SMEM = 8 * WARP_BYTES;
};

template <typename T, int VPL>
__global__ void __launch_bounds__(256) k_enc_size(const T* __restrict__ x, Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = SizeCfg<T, VPL>;
    constexpr int W = TR::W;
    constexpr int B = C::B;
    extern __shared__ __align__(16) uint8_t smem[];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    pdl_wait();
    pdl_trigger();
    const uint64_t nnc = *p.nnc;
    const double eb = *p.eb_abs;
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    uint16_t* zsize = reinterpret_cast<uint16_t*>(out + off_zs);
    U* mus = reinterpret_cast<U*>(out + p.off_mu);
    const U* ncmu = reinterpret_cast<const U*>(p.ncmu);
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t chunk = ((nnc + nw - 1) / nw + C::NB - 1) / C::NB * C::NB;
    const uint64_t c0 = gw * chunk, c1 = umin64(nnc, c0 + chunk);
    const uint32_t sbuf = smem_u32(smem) + warp * C::WARP_BYTES;
    const uint64_t nBfull = p.n / B;
    for (uint64_t g0 = c0; g0 < c1; g0 += 32) {
        // metadata of 32 blocks: lane l holds block g0 + l
        const uint64_t gi = g0 + lane;
        const bool gv = gi < c1;
        const uint32_t mk = gv ? p.nclist[gi] : 0u;
        const U mmu = gv ? ncmu[gi] : U(0);
        const uint32_t mrec = gv ? p.ncR[gi] : 0u;
        const int nbat = (int)((umin64(32, c1 - g0) + C::NB - 1) / C::NB);
        auto issue = [&](int b) {
            const uint32_t st = sbuf + (b & 1) * C::NB * C::BW;
#pragma unroll
            for (int j = 0; j < C::NB; j++) {
                const int l = b * C::NB + j;
                const uint32_t k = __shfl_sync(0xffffffffu, mk, l);
                if (g0 + l < c1 && k < nBfull) {
                    const T* src = x + (uint64_t)k * B + lane * VPL;
#pragma unroll
                    for (int q = 0; q < C::QV; q++)
                        cp_async16(st + j * C::BW + (lane * C::QV + q) * 16, src + q * (16 / W));
                }
            }
            cp_async_commit();
        };
        issue(0);
        for (int b = 0; b < nbat; b++) {
            if (b + 1 < nbat) {
                issue(b + 1);
                cp_async_wait<1>();
            } else {
                cp_async_wait<0>();
            }
            __syncwarp();
            const uint32_t st = sbuf + (b & 1) * C::NB * C::BW;
            // full blocks two at a time: independent instruction streams for ILP
#pragma unroll 1
            for (int j = 0; j < C::NB; j += 2) {
                const int l = b * C::NB + j;
                const uint64_t nc = g0 + l;
                if (nc >= c1) break;
                const bool two = nc + 1 < c1;
                const uint32_t k0 = __shfl_sync(0xffffffffu, mk, l);
                const uint32_t k1 = __shfl_sync(0xffffffffu, mk, l + 1);
                const T mu0 = TR::from(__shfl_sync(0xffffffffu, mmu, l));
                const T mu1 = TR::from(__shfl_sync(0xffffffffu, mmu, l + 1));
                const uint32_t rec0 = __shfl_sync(0xffffffffu, mrec, l);
                const uint32_t rec1 = __shfl_sync(0xffffffffu, mrec, l + 1);
                if (k0 < nBfull && (!two || k1 < nBfull)) {
                    T x0[VPL], x1[VPL];
#pragma unroll
                    for (int q = 0; q < C::QV; q++) {
                        reinterpret_cast<uint4*>(x0)[q] = lds_u128(st + j * C::BW + (lane * C::QV + q) * 16);
                        reinterpret_cast<uint4*>(x1)[q] = lds_u128(st + (j + 1) * C::BW + (lane * C::QV + q) * 16);
                    }
                    int R0 = (int)(rec0 & 0x7F), R1 = (int)(rec1 & 0x7F);
                    const uint32_t z0 = size_block<T, VPL>(x0, mu0, R0, (rec0 & 0x80) != 0, eb);
                    const uint32_t z1 = two ? size_block<T, VPL>(x1, mu1, R1, (rec1 & 0x80) != 0, eb) : 0u;
                    if (lane == 0) {
                        zsize[nc] = (uint16_t)z0;
                        p.ncR[nc] = (uint8_t)R0;
                        if (R0 >= TR::kFull) mus[k0] = 0;  // raw (NaN, Formula 4 or escalation): mu = +0 (R15)
                        if (two) {
                            zsize[nc + 1] = (uint16_t)z1;
                            p.ncR[nc + 1] = (uint8_t)R1;
                            if (R1 >= TR::kFull) mus[k1] = 0;
                        }
                    }
                    continue;
                }
                // a pair holding the partial tail block: one block at a time
                for (int h = 0; h < (two ? 2 : 1); h++) {
                    const uint32_t k = h ? k1 : k0;
                    const T mu = h ? mu1 : mu0;
                    const uint32_t rec = h ? rec1 : rec0;
                    T xv[VPL];
                    U uu[VPL];
                    LaneCode lc;
                    if (k < nBfull) {
#pragma unroll
                        for (int q = 0; q < C::QV; q++)
                            reinterpret_cast<uint4*>(xv)[q] = lds_u128(st + (j + h) * C::BW + (lane * C::QV + q) * 16);
                        encode_block<T, VPL>(xv, VPL, B, mu, (int)(rec & 0x7F), (rec & 0x80) != 0, eb, uu, lc);
                    } else {
                        const int cnt = load_lane<T, VPL>(x, p.n, k, lane, xv);
                        const int len = (int)(p.n - (uint64_t)k * B);
                        encode_block<T, VPL>(xv, cnt, len, mu, (int)(rec & 0x7F), (rec & 0x80) != 0, eb, uu, lc);
                    }
                    if (lane == 0) {
                        zsize[nc + h] = (uint16_t)lc.z;
                        p.ncR[nc + h] = (uint8_t)lc.R;
                        if (lc.R >= TR::kFull) mus[k] = 0;
                    }
                }
            }
            __syncwarp();
        }
    }
}

// ------------------------------------------------------------------ K4 offsets
// Payload offset of every write tile (kWriteTile nonconstant blocks):
// exclusive prefix of the zsize sums, decoupled look-back over CTAs of 256
// tiles.  The last CTA completes the header (payload bytes) and the total.
constexpr int kWriteTile = 32;

template <int W>
__global__ void __launch_bounds__(256) k_zscan(Plan p, uint8_t* __restrict__ out) {
    __shared__ uint64_t s_tile, s_excl, s_w[8];
    pdl_wait();
    pdl_trigger();
    const uint64_t nnc = *p.nnc;
    const uint64_t ntiles = (nnc + kWriteTile - 1) / kWriteTile;
    const uint64_t nct = (ntiles + 255) / 256;
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[2], 1u);
    __syncthreads();
    const uint64_t c = s_tile;
    if (c >= nct) return;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    const uint16_t* zs = reinterpret_cast<const uint16_t*>(out + off_zs);
    const uint64_t t = c * 256 + threadIdx.x;
    uint64_t sum = 0;
    if (t < ntiles) {
        const uint64_t e0 = t * kWriteTile;
        if (e0 + kWriteTile <= nnc) {
            const uint4* q4 = reinterpret_cast<const uint4*>(zs + e0);
#pragma unroll
            for (int q = 0; q < kWriteTile / 8; q++) {
                const uint4 v = q4[q];
                sum += (v.x & 0xFFFFu) + (v.x >> 16) + (v.y & 0xFFFFu) + (v.y >> 16) + (v.z & 0xFFFFu) +
                       (v.z >> 16) + (v.w & 0xFFFFu) + (v.w >> 16);
            }
        } else {
            for (uint64_t e = e0; e < nnc; e++) sum += zs[e];
        }
    }
    // CTA exclusive scan
    uint64_t incl = sum;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const uint64_t v = __shfl_up_sync(0xffffffffu, incl, o);
        if (lane >= o) incl += v;
    }
    if (lane == 31) s_w[warp] = incl;
    __syncthreads();
    uint64_t wpre = 0, agg = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        wpre += i < warp ? s_w[i] : 0;
        agg += s_w[i];
    }
    if (warp == 0) {
        const uint64_t e = lookback_exclusive(p.status_c, c, agg);
        if (lane == 0) {
            s_excl = e;
            if (c == nct - 1) {
                const uint64_t pbytes = e + agg;
                p.gbase[ntiles] = pbytes;
                reinterpret_cast<uint64_t*>(out)[6] = pbytes;  // header: payload bytes
                *p.total = off_zs + al16(2 * nnc) + pbytes;
            }
        }
    }
    __syncthreads();
    if (t < ntiles) p.gbase[t] = s_excl + wpre + incl - sum;
}

// ------------------------------------------------------------------ K2+K3 write pass
// Shift / lead codes with the final R from the size pass (no guard), warp
// scan of mid-byte counts, packing into shared memory, 16-byte stores of the
// tile payload at its offset.  One CTA per tile, no inter-CTA dependency.
template <typename T, int VPL>
__device__ inline void encode_known_R(const T (&xv)[VPL], int cnt, int len, T mu, int R,
                                      typename Traits<T>::U (&u)[VPL], LaneCode& lc) {
    using TR = Traits<T>;
    using U = typename TR::U;
    const int lane = threadIdx.x & 31;
    const bool raw = R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (R & 7)) & 7);
    const int req = (R + s) >> 3;
#pragma unroll
    for (int i = 0; i < VPL; i++) u[i] = (raw ? TR::bits(xv[i]) : TR::bits(TR::sub(xv[i], mu))) >> s;
    U prev = __shfl_up_sync(0xffffffffu, u[VPL - 1], 1);
    if (lane == 0) prev = 0;
    uint32_t leads = 0, m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        if (i < cnt) {
            int L = TR::clz(u[i] ^ prev) >> 3;
            L = L > 3 ? 3 : L;
            leads |= (uint32_t)L << (2 * i);
            m += req > L ? req - L : 0;
            prev = u[i];
        }
    }
    const uint32_t incl = warp_incl_scan(m);
    lc.leads = leads;
    lc.mexcl = incl - m;
    lc.R = R;
    lc.z = 1 + (uint32_t)((len + 3) / 4) + __shfl_sync(0xffffffffu, incl, 31);
}

template <typename T, int VPL>
struct WriteCfg {
    static constexpr int W = Traits<T>::W;
    static constexpr int B = 32 * VPL;
    static constexpr int BW = B * W;
    static constexpr int QV = VPL * W / 16;
    static constexpr int TB = kWriteTile;
    static constexpr int NWARP = 8;
    static constexpr int BPW = TB / NWARP;
    static constexpr int MAXZ = 1 + B / 4 + W * B;
    static constexpr int STG = (16 + TB * MAXZ + 16 + 15) / 16 * 16;
    static constexpr int SMEM = STG + TB * BW;   // staging + the tile's input values
};

template <typename T, int VPL>
__global__ void __launch_bounds__(256) k_enc_write(const T* __restrict__ x, Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = WriteCfg<T, VPL>;
    constexpr int W = TR::W;
    extern __shared__ __align__(16) uint8_t stg[];
    pdl_wait();
    pdl_trigger();
    const uint64_t nnc = *p.nnc;
    const uint64_t t = blockIdx.x;
    if (t * C::TB >= nnc) return;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    const uint64_t off_pl = off_zs + al16(2 * nnc);
    const uint16_t* zsize = reinterpret_cast<const uint16_t*>(out + off_zs);
    const U* ncmu = reinterpret_cast<const U*>(p.ncmu);
    const uint64_t nBfull = p.n / C::B;
    // metadata of this warp's blocks (lanes 0..BPW-1), then their values via cp.async
    const uint64_t ncw = t * C::TB + warp * C::BPW;
    const bool mv = lane < C::BPW && ncw + lane < nnc;
    const uint32_t mk = mv ? p.nclist[ncw + lane] : 0u;
    const U mmu = mv ? ncmu[ncw + lane] : U(0);
    const uint32_t mR = mv ? p.ncR[ncw + lane] : 0u;
    const uint32_t sin = smem_u32(stg) + C::STG + warp * C::BPW * C::BW;
#pragma unroll
    for (int j = 0; j < C::BPW; j++) {
        const uint32_t k = __shfl_sync(0xffffffffu, mk, j);
        if (ncw + j < nnc && k < nBfull) {
            const T* src = x + (uint64_t)k * C::B + lane * VPL;
#pragma unroll
            for (int q = 0; q < C::QV; q++) cp_async16(sin + j * C::BW + (lane * C::QV + q) * 16, src + q * (16 / W));
        }
    }
    cp_async_commit();
    // in-tile offsets of the blocks from their zsize entries
    const uint32_t zl = t * C::TB + lane < nnc ? zsize[t * C::TB + lane] : 0u;
    const uint32_t zincl = warp_incl_scan(zl);
    const uint64_t base = p.gbase[t];
    const uint32_t Tb = __shfl_sync(0xffffffffu, zincl, 31);
    const int sb = (int)(base & 15);
    {   // zero the staging area the OR reductions assemble the tile in
        const uint32_t nz = (uint32_t)((sb + Tb + 15) >> 4);
        for (uint32_t ch = threadIdx.x; ch < nz; ch += 256) reinterpret_cast<uint4*>(stg)[ch] = make_uint4(0, 0, 0, 0);
    }
    cp_async_wait<0>();
    __syncthreads();
#pragma unroll 1
    for (int j = 0; j < C::BPW; j++) {
        const int bi = warp * C::BPW + j;
        const uint64_t nc = t * C::TB + bi;
        const uint32_t zo = __shfl_sync(0xffffffffu, zincl - zl, bi);
        const uint32_t k = __shfl_sync(0xffffffffu, mk, j);
        const T cmu = TR::from(__shfl_sync(0xffffffffu, mmu, j));
        const int R = (int)__shfl_sync(0xffffffffu, mR, j);
        if (nc >= nnc) break;
        T xv[VPL];
        U u[VPL];
        LaneCode lc;
        if (k < nBfull) {
#pragma unroll
            for (int q = 0; q < C::QV; q++)
                reinterpret_cast<uint4*>(xv)[q] = lds_u128(sin + j * C::BW + (lane * C::QV + q) * 16);
            encode_known_R<T, VPL>(xv, VPL, C::B, cmu, R, u, lc);
            pack_red<T, VPL>(u, lc, VPL, C::B, smem_u32(stg) + sb + zo);
        } else {  // the partial tail block
            const int cnt = load_lane<T, VPL>(x, p.n, k, lane, xv);
            const int len = (int)(p.n - (uint64_t)k * C::B);
            encode_known_R<T, VPL>(xv, cnt, len, cmu, R, u, lc);
            pack_red<T, VPL>(u, lc, cnt, len, smem_u32(stg) + sb + zo);
        }
    }
    __syncthreads();
    // copy the staged tile payload to global memory with 16-byte stores
    uint8_t* g0 = out + off_pl + base;
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(g0), A = a0 & ~uintptr_t(15), E = a0 + Tb;
    const uint32_t nch = (uint32_t)((E - A + 15) >> 4);
    for (uint32_t ch = threadIdx.x; ch < nch; ch += 256) {
        const uintptr_t a = A + 16 * (uintptr_t)ch;
        const uint4 v = *reinterpret_cast<const uint4*>(stg + 16 * ch);
        if (a >= a0 && a + 16 <= E) {
            *reinterpret_cast<uint4*>(a) = v;
        } else {
            const uint8_t* vb = reinterpret_cast<const uint8_t*>(&v);
#pragma unroll
            for (int q = 0; q < 16; q++)
                if (a + q >= a0 && a + q < E) *reinterpret_cast<uint8_t*>(a + q) = vb[q];
        }
    }
}

// ------------------------------------------------------------------ K2 fused encoder
// Single pass over the nonconstant blocks (compacted list): for every tile of
// TB blocks the CTA encodes (Formula 4 R from classify, R2 guard / escalation,
// Formula 5 shift, lead codes, mid-byte counts -> z_k), publishes the tile's
// payload size for a decoupled look-back (Merrill & Garland) before packing,
// packs [R][codes][mid-bytes] with shared-memory OR reductions into a zeroed
// staging area, resolves the tile's payload offset and copies the staged bytes
// out realigned to that offset with 16-byte stores.  This is the paper's
// "zsize + prefix sum" done in the same pass as the encoding.
// Persistent CTAs take tiles by atomic ticket (so every predecessor of a tile
// is resident or done: the look-back always progresses) and prefetch the next
// tile's values with cp.async while the current one is encoded.
template <typename T, int VPL>
struct EncCfg {
    static constexpr int W = Traits<T>::W;
    static constexpr int B = 32 * VPL;
    static constexpr int BW = B * W;
    static constexpr int QV = VPL * W / 16;          // 16-byte chunks per lane per block
    static constexpr int NWARP = 8;
    static constexpr int TB = 32 * 512 / BW;         // blocks per tile: 32 (f32, b=128), 16, 8
    static constexpr int BPW = TB / NWARP;           // blocks per warp
    static constexpr int MAXZ = 1 + B / 4 + W * B;
    static constexpr int STG = (16 + TB * MAXZ + 48 + 15) / 16 * 16;  // zero lead pad + payload + read pad
    static constexpr int IN = TB * BW;
    static constexpr int NSTG = 3;                   // staging areas in rotation (pack, copy-out, re-zero)
    static constexpr int SMEM = NSTG * STG + IN;
    static_assert(TB <= 32 && BPW >= 1, "tile must fit one warp scan");
};

// Round-synchronous tile offsets.  With the static schedule, round r holds
// tiles [rG, rG + G) (one per CTA).  Each tile publishes its payload size
// (flag bit 63 | bytes) as soon as it is encoded; one iteration later every
// CTA reads the whole round's sizes (each warp a slice, loads issued before
// packing and consumed after it, so their latency is hidden), takes the
// prefix up to its own tile, and advances its running base by the round
// total.  No tile waits on a chain of predecessors, and the sizes are
// normally all published by the time they are read (a lagging CTA is waited
// for).  Requires a co-resident grid.
__device__ inline void round_publish(uint64_t* slots, uint64_t tile, uint32_t bytes) {
    st_relaxed(&slots[tile], (1ull << 63) | bytes);
}
template <typename T, int VPL>
__global__ void __launch_bounds__(256, 3) k_encode(const T* __restrict__ x, Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = EncCfg<T, VPL>;
    constexpr int W = TR::W;
    constexpr int B = C::B;
    constexpr int TB = C::TB;
    constexpr int BPW = C::BPW;
    extern __shared__ __align__(16) uint8_t smem[];
    __shared__ uint32_t s_z[TB];
    __shared__ uint64_t s_pre[8], s_tot[8];
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint32_t stg0 = smem_u32(smem), in0 = stg0 + C::NSTG * C::STG;
    // zero the staging areas once; afterwards each is re-zeroed after its copy-out
    for (uint32_t ch = threadIdx.x; ch < C::NSTG * C::STG / 16; ch += 256)
        reinterpret_cast<uint4*>(smem)[ch] = make_uint4(0, 0, 0, 0);
    pdl_wait();
    pdl_trigger();
    const uint64_t nnc = *p.nnc;
    const double eb = *p.eb_abs;
    const uint64_t ntiles = (nnc + TB - 1) / TB;
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    const uint64_t off_pl = off_zs + al16(2 * nnc);
    uint16_t* zsize = reinterpret_cast<uint16_t*>(out + off_zs);
    U* mus = reinterpret_cast<U*>(out + p.off_mu);
    const U* ncmu = reinterpret_cast<const U*>(p.ncmu);
    const uint64_t nBfull = p.n / B;
    __syncthreads();
    // static round robin over the co-resident grid: CTA c takes tiles c, c+G, ...
    uint64_t t = blockIdx.x;
    if (t >= ntiles) return;

    // metadata of the warp's BPW blocks of tile tt (lane j < BPW holds block j)
    struct Meta { uint32_t k, rec; U mu; };
    auto meta = [&](uint64_t tt) -> Meta {
        const uint64_t nc = tt * TB + warp * BPW + lane;
        Meta m{0u, 0u, U(0)};
        if (lane < BPW && nc < nnc) { m.k = p.nclist[nc]; m.mu = ncmu[nc]; m.rec = p.ncR[nc]; }
        return m;
    };
    // cp.async of the warp's blocks of tile tt into the input buffer
    auto issue = [&](uint64_t tt, const Meta& m) {
        const uint32_t dst = in0 + warp * BPW * C::BW;
#pragma unroll
        for (int j = 0; j < BPW; j++) {
            const uint32_t k = __shfl_sync(0xffffffffu, m.k, j);
            if (tt * TB + warp * BPW + j < nnc && k < nBfull) {
                const T* src = x + (uint64_t)k * B + lane * VPL;
#pragma unroll
                for (int q = 0; q < C::QV; q++) cp_async16(dst + j * C::BW + (lane * C::QV + q) * 16, src + q * (16 / W));
            }
        }
        cp_async_commit();
    };
    // copy a staged tile (Tb bytes at staging offset 16) to its payload offset,
    // realigned, with 16-byte stores (byte stores in the two boundary chunks,
    // which the neighbouring tiles share)
    auto copy_out = [&](uint32_t sp, uint64_t tt, uint64_t base, uint32_t Tb) {
        const uint64_t g0 = off_pl + base;
        const uint32_t mis = (uint32_t)(g0 & 15);
        const uint64_t A0 = g0 - mis;
        const uint32_t nch = (mis + Tb + 15) >> 4;
        for (uint32_t ch = threadIdx.x; ch < nch; ch += 256) {
            uint32_t r[4];
            run_load_s<4>(sp + 16 * ch - mis, r);
            uint8_t* dst = out + A0 + 16 * (uint64_t)ch;
            const int64_t lo = (int64_t)mis - 16 * (int64_t)ch, hi = (int64_t)mis + Tb - 16 * (int64_t)ch;
            if (lo <= 0 && hi >= 16) {
                *reinterpret_cast<uint4*>(dst) = make_uint4(r[0], r[1], r[2], r[3]);
            } else {
#pragma unroll
                for (int q = 0; q < 16; q++)
                    if (q >= lo && q < hi) dst[q] = (uint8_t)(r[q >> 2] >> (8 * (q & 3)));
            }
        }
        if (tt == ntiles - 1 && threadIdx.x == 0) {
            const uint64_t pbytes = base + Tb;
            reinterpret_cast<uint64_t*>(out)[6] = pbytes;  // header: payload bytes
            *p.total = off_pl + pbytes;
        }
    };
    Meta cur = meta(t), nxt{0u, 0u, U(0)};
    issue(t, cur);
    // Software pipeline: tile i is encoded, published and packed in iteration
    // i, its offset resolved and its bytes copied out in iteration i+1 (by
    // then its predecessors have published), and its staging area re-zeroed
    // in iteration i+2.  Three staging areas rotate.
    uint64_t t_prev = 0;
    uint64_t run_base = 0;  // payload bytes of all rounds before t_prev's
    uint32_t tb_prev = 0, tb_pp = 0;
    int it = 0;
    for (;; it++) {
        const int sb = it % C::NSTG;
        const uint64_t tn = t + gridDim.x;
        if (tn < ntiles) nxt = meta(tn);  // used after barrier #1
        cp_async_wait<0>();
        __syncwarp();
        // ---- encode the warp's blocks (registers)
        U u[BPW][VPL];
        LaneCode lc[BPW];
#pragma unroll
        for (int j = 0; j < BPW; j++) {
            const uint64_t nc = t * TB + warp * BPW + j;
            lc[j].z = 0;
            lc[j].R = 0;
            if (nc < nnc) {
                const uint32_t k = __shfl_sync(0xffffffffu, cur.k, j);
                const T mu = TR::from(__shfl_sync(0xffffffffu, cur.mu, j));
                const uint32_t rec = __shfl_sync(0xffffffffu, cur.rec, j);
                T xv[VPL];
                if (k < nBfull) {
                    const uint32_t sa = in0 + (warp * BPW + j) * C::BW;
#pragma unroll
                    for (int q = 0; q < C::QV; q++)
                        reinterpret_cast<uint4*>(xv)[q] = lds_u128(sa + (lane * C::QV + q) * 16);
                    encode_block<T, VPL>(xv, VPL, B, mu, (int)(rec & 0x7F), (rec & 0x80) != 0, eb, u[j], lc[j]);
                } else {  // the partial tail block, straight from global memory
                    const int cnt = load_lane<T, VPL>(x, p.n, k, lane, xv);
                    const int len = (int)(p.n - (uint64_t)k * B);
                    encode_block<T, VPL>(xv, cnt, len, mu, (int)(rec & 0x7F), (rec & 0x80) != 0, eb, u[j], lc[j]);
                }
                if (lane == 0 && lc[j].R >= TR::kFull) mus[k] = 0;  // raw: mu = +0 (R15)
            }
            if (lane == 0) s_z[warp * BPW + j] = lc[j].z;
        }
        __syncthreads();  // #1: s_z complete, the input buffer is free
        if (tn < ntiles) issue(tn, nxt);
        // tile scan of z (every warp, redundantly) -> in-tile offsets, tile size
        const uint32_t zl = lane < TB ? s_z[lane] : 0u;
        const uint32_t zincl = warp_incl_scan(zl);
        const uint32_t Tb = __shfl_sync(0xffffffffu, zincl, 31);
        if (threadIdx.x == 0) round_publish(p.status_c, t, Tb);
        if (threadIdx.x < TB && t * TB + threadIdx.x < nnc) zsize[t * TB + threadIdx.x] = (uint16_t)zl;
        {   // re-zero the staging area of the tile copied out last iteration
            const uint32_t sz = stg0 + ((it + 1) % C::NSTG) * C::STG;
            const uint32_t nch = (16 + tb_pp + 48 + 15) >> 4;
            for (uint32_t ch = threadIdx.x; ch < nch; ch += 256)
                asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(sz + 16 * ch), "r"(0u) : "memory");
        }
        // ---- the previous tile's round: this warp's slice of the published sizes
        constexpr int QW = 3;  // entries per lane: G <= 8 warps x 32 x QW
        const uint64_t G = gridDim.x;
        const uint64_t per_w = (G + 7) / 8;
        const uint64_t r0 = t_prev / G * G, r1 = umin64(r0 + G, ntiles);
        uint64_t rv[QW];
#pragma unroll
        for (int q = 0; q < QW; q++) {
            const uint64_t o = 32 * q + lane, idx = r0 + warp * per_w + o;
            rv[q] = (it > 0 && o < per_w && idx < r1) ? ld_relaxed(&p.status_c[idx]) : (1ull << 63);
        }
        // ---- pack into the zeroed staging area (16-byte lead pad)
        const uint32_t sp = stg0 + sb * C::STG + 16;
#pragma unroll
        for (int j = 0; j < BPW; j++) {
            const int bi = warp * BPW + j;
            const uint64_t nc = t * TB + bi;
            const uint32_t zo = __shfl_sync(0xffffffffu, zincl - zl, bi);
            if (nc < nnc) {
                const uint32_t k = __shfl_sync(0xffffffffu, cur.k, j);
                if (k < nBfull) {
                    pack_red<T, VPL>(u[j], lc[j], VPL, B, sp + zo);
                } else {
                    const uint64_t first = (uint64_t)k * B + (uint64_t)lane * VPL;
                    const int cnt = first >= p.n ? 0 : (int)umin64(VPL, p.n - first);
                    pack_red<T, VPL>(u[j], lc[j], cnt, (int)(p.n - (uint64_t)k * B), sp + zo);
                }
            }
        }
        // ---- the previous tile: offset (sum of the slices), then copy-out
        {
            uint64_t pre = 0, tot = 0;
#pragma unroll
            for (int q = 0; q < QW; q++) {
                const uint64_t o = 32 * q + lane, idx = r0 + warp * per_w + o;
                if (it > 0 && o < per_w && idx < r1) {
#ifdef SZX_EXP_NOWAIT
                    rv[q] |= 1ull << 63;
#endif
                    while (!(rv[q] >> 63)) {  // a lagging CTA has not published yet
                        __nanosleep(32);
                        rv[q] = ld_relaxed(&p.status_c[idx]);
                    }
                    const uint64_t val = rv[q] & ~(1ull << 63);
                    tot += val;
                    pre += idx < t_prev ? val : 0;
                }
            }
            pre = warp_sum64(pre);
            tot = warp_sum64(tot);
            if (lane == 0) { s_pre[warp] = pre; s_tot[warp] = tot; }
        }
        __syncthreads();  // #2: this tile staged; the previous tile's round sizes summed
        if (it > 0) {
            uint64_t pre = 0, tot = 0;
#pragma unroll
            for (int w = 0; w < 8; w++) { pre += s_pre[w]; tot += s_tot[w]; }
            copy_out(stg0 + ((it + C::NSTG - 1) % C::NSTG) * C::STG + 16, t_prev, run_base + pre, tb_prev);
            run_base += tot;
        }
        tb_pp = tb_prev;
        tb_prev = Tb;
        t_prev = t;
        if (tn >= ntiles) break;
        t = tn;
        cur = nxt;
    }
    // drain: the last tile of this CTA (its round's sizes, then copy-out)
    {
        const uint64_t G = gridDim.x;
        const uint64_t r0 = t_prev / G * G;
        uint64_t pre = 0;
        for (uint64_t idx = r0 + threadIdx.x; idx < t_prev; idx += 256) {
            uint64_t v = ld_relaxed(&p.status_c[idx]);
            while (!(v >> 63)) {
                __nanosleep(32);
                v = ld_relaxed(&p.status_c[idx]);
            }
            pre += v & ~(1ull << 63);
        }
        pre = warp_sum64(pre);
        __syncthreads();  // s_pre may still be read by the last iteration
        if (lane == 0) s_pre[warp] = pre;
        __syncthreads();
        pre = 0;
#pragma unroll
        for (int w = 0; w < 8; w++) pre += s_pre[w];
        copy_out(stg0 + (it % C::NSTG) * C::STG + 16, t_prev, run_base + pre, tb_prev);
    }
}

__global__ void k_empty_header(uint8_t* out, uint32_t dtype, uint32_t mode, uint32_t b, double eb_user,
                               const uint64_t* range_keys, uint64_t* total) {
    uint64_t* h = reinterpret_cast<uint64_t*>(out);
    h[0] = 0x31585A53ull | (1ull << 32) | ((uint64_t)dtype << 40) | ((uint64_t)mode << 48);
    h[1] = b;
    h[2] = 0;
    h[3] = (uint64_t)__double_as_longlong(eb_user);
    // REL: the (global) range of a sharded array, or no values at all -> 0
    const double e = eb_from_range(mode, eb_user, range_keys);
    h[4] = (uint64_t)__double_as_longlong(e);
    h[5] = 0;
    h[6] = 0;
    h[7] = 0;
    if (total) *total = 64;
}

}  // namespace szx
