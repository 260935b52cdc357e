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
//   k_encode_fused (K2+K3+K4 fused, szx_encode.cuh; b = 128) persistent
//                        cooperative kernel: compute warps take 4*NW-block
//                        tiles by ticket, stage their own blocks with
//                        cp.async, encode (normalise, Formula 4 R, Formula 5
//                        shift, lead codes, R2 guard) and pack the tile in
//                        shared memory; one scanner warp in CTA 0 turns the
//                        published tile sizes into payload offsets (grid-wide
//                        forward scan); the tile is copied out NS-1 tiles
//                        later with 16-byte stores.
//   k_enc_size / k_zscan / k_enc_write  the three-pass encoder for b != 128
//                        (sizes, device-wide scan, write).
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
    const double* eb_in;       // non-null: the absolute bound, given (szx_compress_shard)
    uint32_t* ctr;             // [4] tile tickets, init 0
    uint64_t* status_b;        // classify look-back, init 0
    uint64_t* status_c;        // offset-scan look-back, init 0
    uint64_t* status_e;        // fused encoder: tile sizes (one word per tile), init 0
    uint64_t* prefix_e;        // fused encoder: tile payload offsets from the scanner, init 0
    void* stats;               // 2 keys per block (min, max)
    uint32_t* nclist;          // ids of the nonconstant blocks, in block order
    void* ncmu;                // their mu (bits), same order
    uint8_t* ncR;              // classify: R_init | proven << 7; size pass: final R
    uint64_t* gbase;           // payload offset of each write tile (+ total)
    uint8_t* nccodes;          // float32 b = 128: the 32 lead-code bytes of every full nonconstant
                               // block (size pass -> write pass), in nonconstant order; else null
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
        using LY = Lay<T, VPL>;
        using V = typename LY::V;
        const V* p = reinterpret_cast<const V*>(x + first);
#pragma unroll
        for (int q = 0; q < LY::NQ; q++) reinterpret_cast<V*>(v)[q] = ld_stream<V>(p + q);
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
    using LY = Lay<T, VPL>;
    using V = typename LY::V;
    constexpr int NV = LY::NQ;                       // chunk loads per lane per block
    const uint64_t nBf = p.n / B;                    // full blocks
    uint64_t k0 = gw * UNR;
    // fast path: UNR full blocks per warp, all loads issued first, no bounds checks
    for (; k0 + UNR <= nBf; k0 += nw * UNR) {
        const V* src = reinterpret_cast<const V*>(x + k0 * B) + lane * NV;
        T v[UNR][VPL];
#pragma unroll
        for (int u = 0; u < UNR; u++)
#pragma unroll
            for (int q = 0; q < NV; q++) reinterpret_cast<V*>(v[u])[q] = ld_stream<V>(src + u * (B * (int)sizeof(T) / LY::CB) + q);
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
// 256 threads x BPT blocks (8 BPT bitmap words) per CTA tile; BPT = 8 for
// large fields, fewer for small ones so that the grid still covers the SMs
// (the per-block work is a chain of dependent double-precision steps).
constexpr int kClassifyBlocks = 2048;     // largest tile (BPT = 8)
constexpr int kClassifyMinBlocks = 256;   // smallest tile (BPT = 1): sizes the look-back words

// COOP = false: tiles by ticket, nonconstant-count scan by decoupled look-back
// (large arrays).  COOP = true: one tile per CTA of a co-resident (cooperative)
// grid and one grid-wide prefix instead: the look-back's depth grows with the
// tile count, the prefix's does not (small arrays, where more, smaller tiles
// shorten every thread's chain of dependent steps).
template <typename T, int BPT, bool COOP = false>
__global__ void __launch_bounds__(256) k_classify(Plan p, uint8_t* __restrict__ out) {
    static_assert(BPT == 1 || BPT == 2 || BPT == 4 || BPT == 8, "BPT");
    constexpr int CB = 256 * BPT;
    using TR = Traits<T>;
    using U = typename TR::U;
    __shared__ uint64_t s_tile, s_base, s_agg;
    __shared__ uint64_t s_w[32];
    __shared__ uint32_t s_cnt[64], s_pre[64];  // [8 * BPT] used
    pdl_wait();
    pdl_trigger();
    if (!COOP && threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[0], 1u);
    __syncthreads();
    const uint64_t tile = COOP ? (uint64_t)blockIdx.x : s_tile;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t base = tile * CB;
    const double eb = eb_from_range(p.mode, p.eb_user, p.range_keys, p.eb_in);
    const int pe = expo_f64(eb);
    const U* stats = reinterpret_cast<const U*>(p.stats);
    uint32_t* bitmap = reinterpret_cast<uint32_t*>(out + kHeaderBytes);
    U* mus = reinterpret_cast<U*>(out + p.off_mu);

    uint32_t ncmask = 0;
    U rmu[BPT];
    uint32_t rrec[2] = {0u, 0u};  // per j: R_init | guard_proven << 7 (one byte each)
    // all eight blocks' keys first: the stores below (mu, bitmap) could alias the
    // stats for the compiler, which would otherwise serialise one load round trip
    // per block
    U kmn[BPT], kmx[BPT];
#pragma unroll
    for (int j = 0; j < BPT; j++) {
        const uint64_t k = base + j * 256 + threadIdx.x;
        kmn[j] = k < p.nB ? stats[2 * k] : U(0);
        kmx[j] = k < p.nB ? stats[2 * k + 1] : U(0);
    }
#pragma unroll
    for (int j = 0; j < BPT; j++) {
        const uint64_t k = base + j * 256 + threadIdx.x;
        bool nc = false;
        rmu[j] = 0;
        if (k < p.nB) {
            BlockClass<T> c = classify<T>(kmn[j], kmx[j], eb);
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
        const uint32_t c0 = 2 * lane < 8 * BPT ? s_cnt[2 * lane] : 0u;
        const uint32_t c1 = 2 * lane + 1 < 8 * BPT ? s_cnt[2 * lane + 1] : 0u;
        const uint32_t incl = warp_incl_scan(c0 + c1);
        const uint32_t ex = incl - c0 - c1;
        s_pre[2 * lane] = ex;
        s_pre[2 * lane + 1] = ex + c0;
        const uint32_t agg = __shfl_sync(0xffffffffu, incl, 31);
        if (lane == 0) s_agg = agg;
        if (!COOP) {
            const uint64_t G = lookback_exclusive(p.status_b, tile, agg);
            if (lane == 0) s_base = G;
        }
    }
    if (COOP) {
        __syncthreads();
        const uint64_t G = grid_excl_prefix(p.status_b, p.status_b + gridDim.x, &p.ctr[1], s_agg, s_w, gridDim.x);
        if (threadIdx.x == 0) s_base = G;
    }
    if (threadIdx.x == 0) {
        {
            const uint64_t G = s_base, agg = s_agg;
            const uint64_t ntiles = (p.nB + CB - 1) / CB;
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
    for (int j = 0; j < BPT; j++) {
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
    if constexpr (VPL >= 4) {
#pragma unroll
        for (int q = 0; q < VPL / 4; q++) {
            const int cb = lane * (VPL / 4) + q;
            if (cb < ncode) red_or_byte(dst + 1 + cb, lc.leads >> (8 * q));
        }
    } else {  // 4 / VPL lanes share a code byte
        if ((int)code_byte<VPL>(lane) < ncode) red_or_byte(dst + 1 + code_byte<VPL>(lane), lc.leads << code_shift<VPL>(lane));
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

// R2 guard / escalation only (R2): returns the final R of a block
// whose per-element check was not proven unnecessary by classify.
template <typename T, int VPL>
__device__ inline int guard_R(const T (&xv)[VPL], int cnt, T mu, int R, double eb) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    for (;;) {
        if (R >= TR::kFull) return TR::kFull;
        const int s = (8 - (R & 7)) & 7;
        const U keep = ~((U(1) << (8 * W - R)) - U(1));
        bool ok = true;
#pragma unroll
        for (int i = 0; i < VPL; i++) {
            if (i < cnt) {
                const U u = TR::bits(TR::sub(xv[i], mu)) >> s;
                const T xp = TR::add(TR::from((u << s) & keep), mu);
                ok &= fabs(__dsub_rn((double)xv[i], (double)xp)) <= eb;
            }
        }
        if (__all_sync(0xffffffffu, ok)) return R;
        R += 1;
    }
}

// ---------------------------------------------------------- float32 fast path
// Full float32 blocks of b = 128 (4 values per lane) with a FINAL R (the guard
// has run): shifted words, lead codes and the per-value mid-byte counts, all
// branch-free.  Identical output to encode_block/encode_known_R.
// min(3, leading zero bytes of d): the 2-bit lead code (R6) in 4 instructions
__device__ __forceinline__ uint32_t lead_bytes3(uint32_t d) {
    // (bfind.shiftamt -- FLO.SH without the 31-x fix-up -- measured 3 % slower in the write pass)
    return (uint32_t)__clz(d | 0xFFu) >> 3;
}

struct Lane4 {
    uint32_t u[4];      // shifted words
    uint32_t leads;     // 2-bit codes, LSB-first
    uint32_t msum;      // mid-bytes of this lane (consumed by the scan)
};
__device__ __forceinline__ void lane_encode_f32x4(const float (&xv)[4], float mu, int R, Lane4& e) {
    const int lane = threadIdx.x & 31;
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
#pragma unroll
    for (int i = 0; i < 4; i++)
        e.u[i] = (raw ? __float_as_uint(xv[i]) : __float_as_uint(__fsub_rn(xv[i], mu))) >> s;
    uint32_t prev = __shfl_up_sync(0xffffffffu, e.u[3], 1);
    prev = lane == 0 ? 0u : prev;
    uint32_t leads = 0, msum = 0;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const uint32_t L = lead_bytes3(e.u[i] ^ prev);
        prev = e.u[i];
        leads |= L << (2 * i);
        msum += req - umin_(L, req);
    }
    e.leads = leads;
    e.msum = msum;
}

// Mid-bytes of this lane only (the size pass): no codes kept.
__device__ __forceinline__ uint32_t lane_msum_f32x4(const float (&xv)[4], float mu, int R) {
    const int lane = threadIdx.x & 31;
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
    uint32_t u[4];
#pragma unroll
    for (int i = 0; i < 4; i++) u[i] = (raw ? __float_as_uint(xv[i]) : __float_as_uint(__fsub_rn(xv[i], mu))) >> s;
    uint32_t prev = __shfl_up_sync(0xffffffffu, u[3], 1);
    prev = lane == 0 ? 0u : prev;
    uint32_t msum = 0;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const uint32_t L = lead_bytes3(u[i] ^ prev);
        prev = u[i];
        msum += req - umin_(L, req);
    }
    return msum;
}

// OR v into shared word a unless v == 0 (predicated, no branch)
__device__ __forceinline__ void red_or_nz(uint32_t a, uint32_t v) {
    asm volatile("{\n\t.reg .pred q;\n\tsetp.ne.u32 q, %1, 0;\n\t@q red.shared.or.b32 [%0], %1;\n\t}"
                 ::"r"(a), "r"(v) : "memory");
}

// ---- half-warp variants (8 values per lane, a block per 16 lanes): the
// write pass encodes two blocks per warp instruction stream
struct Lane8 {
    uint32_t u[8];      // shifted words
    uint32_t leads;     // 2-bit codes of the 8 values, LSB-first (16 bits)
    uint32_t msum;      // mid-bytes of this lane
};
__device__ __forceinline__ void lane_encode_f32x8(const float (&xv)[8], float mu, int R, Lane8& e) {
    const int hl = threadIdx.x & 15;
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
#pragma unroll
    for (int i = 0; i < 8; i++)
        e.u[i] = (raw ? __float_as_uint(xv[i]) : __float_as_uint(__fsub_rn(xv[i], mu))) >> s;
    uint32_t prev = __shfl_up_sync(0xffffffffu, e.u[7], 1, 16);
    prev = hl == 0 ? 0u : prev;
    uint32_t leads = 0, msum = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t L = lead_bytes3(e.u[i] ^ prev);
        prev = e.u[i];
        leads |= L << (2 * i);
        msum += req - umin_(L, req);
    }
    e.leads = leads;
    e.msum = msum;
}
// inclusive prefix sum within 16-lane segments
template <int O>
__device__ __forceinline__ uint32_t shfl_up_add16c(uint32_t v) {
    asm volatile(
        "{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
        "shfl.sync.up.b32 t|p, %0, %1, 0x1000, -1;\n\t"
        "@p add.u32 %0, %0, t;\n\t}"
        : "+r"(v)
        : "n"(O));
    return v;
}
__device__ __forceinline__ uint32_t half_incl_scan(uint32_t v) {
    v = shfl_up_add16c<1>(v);
    v = shfl_up_add16c<2>(v);
    v = shfl_up_add16c<4>(v);
    return shfl_up_add16c<8>(v);
}
__device__ inline void red_or_s(uint32_t a, uint32_t v);
// Pack a full float32 block held by a half-warp into the zeroed staging area at dst.
__device__ __forceinline__ void lane_pack_f32x8(const Lane8& e, int R, uint32_t mexcl, uint32_t dst) {
    const int hl = threadIdx.x & 15;
    if (hl == 0) red_or_s(dst & ~3u, (uint32_t)R << (8 * (dst & 3u)));
    {   // this lane's two code bytes (they may straddle a word)
        const uint32_t a = dst + 1 + 2 * hl, sh = 8 * (a & 3u);
        red_or_s(a & ~3u, e.leads << sh);
        const uint32_t w1 = __funnelshift_l(e.leads, 0u, sh);
        red_or_nz((a & ~3u) + 4, w1);
    }
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
    const uint32_t drop = 8u * (4u - req);
    uint32_t a = dst + 33 + mexcl;
#pragma unroll
    for (int h = 0; h < 4; h++) {
        const uint32_t m0 = req - umin_((e.leads >> (4 * h)) & 3u, req);
        const uint32_t m1 = req - umin_((e.leads >> (4 * h + 2)) & 3u, req);
        const uint32_t c0 = (e.u[2 * h] >> drop) & ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8 * m0);
        const uint32_t c1 = (e.u[2 * h + 1] >> drop) & ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8 * m1);
        const uint32_t lo = c0 | __funnelshift_lc(0u, c1, 8 * m0);
        const uint32_t hi = __funnelshift_lc(c1, 0u, 8 * m0);
        const uint32_t sh = 8 * (a & 3u), wa = a & ~3u;
        red_or_s(wa, lo << sh);
        red_or_s(wa + 4, __funnelshift_l(lo, hi, sh));
        red_or_nz(wa + 8, __funnelshift_l(hi, 0u, sh));
        a += m0 + m1;
    }
}

// Lead codes (16 bits, LSB-first) and mid-bytes of this lane's 8 values (size pass)
__device__ __forceinline__ uint32_t lane_codes_f32x8(const float (&xv)[8], float mu, int R, uint32_t& msum) {
    const int hl = threadIdx.x & 15;
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
    uint32_t u[8];
#pragma unroll
    for (int i = 0; i < 8; i++) u[i] = (raw ? __float_as_uint(xv[i]) : __float_as_uint(__fsub_rn(xv[i], mu))) >> s;
    uint32_t prev = __shfl_up_sync(0xffffffffu, u[7], 1, 16);
    prev = hl == 0 ? 0u : prev;
    uint32_t leads = 0;
    msum = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t L = lead_bytes3(u[i] ^ prev);
        prev = u[i];
        leads |= L << (2 * i);
        msum += req - umin_(L, req);
    }
    return leads;
}
// Mid-bytes of this lane's 8 values (size pass, half-warp per block)
__device__ __forceinline__ uint32_t lane_msum_f32x8(const float (&xv)[8], float mu, int R) {
    const int hl = threadIdx.x & 15;
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
    uint32_t u[8];
#pragma unroll
    for (int i = 0; i < 8; i++) u[i] = (raw ? __float_as_uint(xv[i]) : __float_as_uint(__fsub_rn(xv[i], mu))) >> s;
    uint32_t prev = __shfl_up_sync(0xffffffffu, u[7], 1, 16);
    prev = hl == 0 ? 0u : prev;
    uint32_t msum = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t L = lead_bytes3(u[i] ^ prev);
        prev = u[i];
        msum += req - umin_(L, req);
    }
    return msum;
}

// Pack a full float32 block into a zeroed shared staging area at byte address
// dst: [R][32 code bytes][mid-bytes].  Values are placed in pairs: the two
// chunks (<= 8 bytes) are joined with funnel shifts and OR-ed in as at most
// three aligned words.
__device__ __forceinline__ void lane_pack_f32x4(const Lane4& e, int R, uint32_t mexcl, uint32_t dst) {
    const int lane = threadIdx.x & 31;
    if (lane == 0) red_or_s(dst & ~3u, (uint32_t)R << (8 * (dst & 3u)));
    {
        const uint32_t a = dst + 1 + lane;
        red_or_s(a & ~3u, e.leads << (8 * (a & 3u)));
    }
    const bool raw = R >= 32;
    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
    const uint32_t req = ((uint32_t)R + s) >> 3;
    const uint32_t drop = 8u * (4u - req);
    uint32_t a = dst + 33 + mexcl;
#pragma unroll
    for (int h = 0; h < 2; h++) {
        const uint32_t m0 = req - umin_((e.leads >> (4 * h)) & 3u, req);
        const uint32_t m1 = req - umin_((e.leads >> (4 * h + 2)) & 3u, req);
        const uint32_t c0 = (e.u[2 * h] >> drop) & ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8 * m0);
        const uint32_t c1 = (e.u[2 * h + 1] >> drop) & ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8 * m1);
        const uint32_t lo = c0 | __funnelshift_lc(0u, c1, 8 * m0);
        const uint32_t hi = __funnelshift_lc(c1, 0u, 8 * m0);
        const uint32_t sh = 8 * (a & 3u), wa = a & ~3u;
        // at most 8 bytes + 3 of misalignment: the third word is rarely needed
        red_or_s(wa, lo << sh);
        red_or_s(wa + 4, __funnelshift_l(lo, hi, sh));
        red_or_nz(wa + 8, __funnelshift_l(hi, 0u, sh));
        a += m0 + m1;
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
    static constexpr int QV = Lay<T, VPL>::NQ;   // chunks per lane per block
    static constexpr int CB = Lay<T, VPL>::CB;   // chunk bytes
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
        if constexpr (sizeof(T) == 4 && VPL == 4) {
            // fast path: 32 full float32 blocks (the list is in block order, so
            // the last one decides): no per-block bounds or tail tests, and z_k /
            // R collected in lane l for one coalesced store per 32 blocks
            if (c1 - g0 >= 32 && __shfl_sync(0xffffffffu, mk, 31) < nBfull) {
                auto issue_f = [&](int b) {
                    const uint32_t st = sbuf + (b & 1) * C::NB * C::BW;
#pragma unroll
                    for (int j = 0; j < C::NB; j++) {
                        const uint32_t k = __shfl_sync(0xffffffffu, mk, b * C::NB + j);
                        cp_async16(st + j * C::BW + lane * 16, x + (uint64_t)k * B + lane * 4);
                    }
                    cp_async_commit();
                };
                uint32_t zr = 0, rr = 0;
                issue_f(0);
#pragma unroll 1
                for (int b = 0; b < 32 / C::NB; b++) {
                    if (b + 1 < 32 / C::NB) {
                        issue_f(b + 1);
                        cp_async_wait<1>();
                    } else {
                        cp_async_wait<0>();
                    }
                    __syncwarp();
                    const uint32_t st = sbuf + (b & 1) * C::NB * C::BW;
                    // two blocks at once, a half-warp each (8 values per lane)
#pragma unroll
                    for (int j = 0; j < C::NB; j += 2) {
                        const int l = b * C::NB + j;
                        const int h = lane >> 4, hl = lane & 15;
                        float xv[8];
                        reinterpret_cast<uint4*>(xv)[0] = lds_u128(st + (j + h) * C::BW + hl * 32);
                        reinterpret_cast<uint4*>(xv)[1] = lds_u128(st + (j + h) * C::BW + hl * 32 + 16);
                        const float mu = __uint_as_float(__shfl_sync(0xffffffffu, (uint32_t)mmu, l + h));
                        const uint32_t rec = __shfl_sync(0xffffffffu, mrec, l + h);
                        int R = (int)(rec & 0x7F);
                        if (!__all_sync(0xffffffffu, (rec & 0x80) != 0)) {
                            // a block whose R2 check was not proven away: full-warp guard per block
                            float x0[4], x1[4];
                            reinterpret_cast<uint4*>(x0)[0] = lds_u128(st + j * C::BW + lane * 16);
                            reinterpret_cast<uint4*>(x1)[0] = lds_u128(st + (j + 1) * C::BW + lane * 16);
                            const uint32_t rec0 = __shfl_sync(0xffffffffu, mrec, l);
                            const uint32_t rec1 = __shfl_sync(0xffffffffu, mrec, l + 1);
                            const float mu0 = __uint_as_float(__shfl_sync(0xffffffffu, (uint32_t)mmu, l));
                            const float mu1 = __uint_as_float(__shfl_sync(0xffffffffu, (uint32_t)mmu, l + 1));
                            int R0 = (int)(rec0 & 0x7F), R1 = (int)(rec1 & 0x7F);
                            if (!(rec0 & 0x80)) R0 = guard_R<float, 4>(x0, 4, mu0, R0, eb);
                            if (!(rec1 & 0x80)) R1 = guard_R<float, 4>(x1, 4, mu1, R1, eb);
                            R = h ? R1 : R0;
                        }
                        uint32_t ms;
                        const uint32_t lc16 = lane_codes_f32x8(xv, mu, R, ms);
                        reinterpret_cast<uint16_t*>(p.nccodes)[(g0 + l + h) * 16 + hl] = (uint16_t)lc16;
                        const uint32_t z0 = 33u + warp_sum(h ? 0u : ms);
                        const uint32_t z1 = 33u + warp_sum(h ? ms : 0u);
                        const uint32_t R0 = __shfl_sync(0xffffffffu, (uint32_t)R, 0);
                        const uint32_t R1 = __shfl_sync(0xffffffffu, (uint32_t)R, 16);
                        zr = lane == l ? z0 : zr;
                        rr = lane == l ? R0 : rr;
                        zr = lane == l + 1 ? z1 : zr;
                        rr = lane == l + 1 ? R1 : rr;
                    }
                    __syncwarp();
                }
                zsize[gi] = (uint16_t)zr;
                p.ncR[gi] = (uint8_t)rr;
                if (rr >= 32u) mus[mk] = 0;  // raw (NaN, Formula 4 or escalation): mu = +0 (R15)
                continue;
            }
        }
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
                        cp_async_chunk<C::CB>(st + j * C::BW + (lane * C::QV + q) * C::CB, src + q * (C::CB / W));
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
                        using V = typename Lay<T, VPL>::V;
                        reinterpret_cast<V*>(x0)[q] = lds_chunk<V>(st + j * C::BW + (lane * C::QV + q) * C::CB);
                        reinterpret_cast<V*>(x1)[q] = lds_chunk<V>(st + (j + 1) * C::BW + (lane * C::QV + q) * C::CB);
                    }
                    int R0 = (int)(rec0 & 0x7F), R1 = (int)(rec1 & 0x7F);
                    uint32_t z0, z1 = 0u;
                    if constexpr (sizeof(T) == 4 && VPL == 4) {
                        if (!(rec0 & 0x80)) R0 = guard_R<T, VPL>(x0, VPL, mu0, R0, eb);
                        if (two && !(rec1 & 0x80)) R1 = guard_R<T, VPL>(x1, VPL, mu1, R1, eb);
                        Lane4 e0, e1;
                        lane_encode_f32x4(x0, mu0, R0, e0);
                        lane_encode_f32x4(x1, mu1, R1, e1);
                        p.nccodes[nc * 32 + lane] = (uint8_t)e0.leads;
                        z0 = 33u + warp_sum(e0.msum);
                        if (two) {
                            p.nccodes[(nc + 1) * 32 + lane] = (uint8_t)e1.leads;
                            z1 = 33u + warp_sum(e1.msum);
                        }
                    } else {
                        z0 = size_block<T, VPL>(x0, mu0, R0, (rec0 & 0x80) != 0, eb);
                        z1 = two ? size_block<T, VPL>(x1, mu1, R1, (rec1 & 0x80) != 0, eb) : 0u;
                    }
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
                        for (int q = 0; q < C::QV; q++) {
                            using V = typename Lay<T, VPL>::V;
                            reinterpret_cast<V*>(xv)[q] = lds_chunk<V>(st + (j + h) * C::BW + (lane * C::QV + q) * C::CB);
                        }
                        encode_block<T, VPL>(xv, VPL, B, mu, (int)(rec & 0x7F), (rec & 0x80) != 0, eb, uu, lc);
                        if constexpr (sizeof(T) == 4 && VPL == 4) p.nccodes[(nc + h) * 32 + lane] = (uint8_t)lc.leads;
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
    static constexpr int QV = Lay<T, VPL>::NQ;
    static constexpr int CB = Lay<T, VPL>::CB;
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
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    // tiles c, c + G, ...: the grid is capped on the host (a few CTAs per resident
    // slot), so a sparse field does not pay for a wave of CTAs with no tile
    for (uint64_t t = blockIdx.x; t * C::TB < nnc; t += gridDim.x) {
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
    // whole tile of full blocks (the list is in block order: the tile's last block decides)
    const bool tfull = (t + 1) * C::TB <= nnc && p.nclist[(t + 1) * C::TB - 1] < nBfull;
#pragma unroll
    for (int j = 0; j < C::BPW; j++) {
        const uint32_t k = __shfl_sync(0xffffffffu, mk, j);
        if (tfull || (ncw + j < nnc && k < nBfull)) {
            const T* src = x + (uint64_t)k * C::B + lane * VPL;
#pragma unroll
            for (int q = 0; q < C::QV; q++) cp_async_chunk<C::CB>(sin + j * C::BW + (lane * C::QV + q) * C::CB, src + q * (C::CB / W));
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
    bool packed = false;
    if constexpr (sizeof(T) == 4 && VPL == 4) {
        if (tfull) {  // branch-free body: every block of the tile is a full float32 block
            // two blocks per step, a half-warp each (8 values per lane)
            const int h = lane >> 4, hl = lane & 15;
#pragma unroll
            for (int q = 0; q < C::BPW / 2; q++) {
                const int j = 2 * q + h;
                const int bi = warp * C::BPW + j;
                const uint32_t zo = __shfl_sync(0xffffffffu, zincl - zl, bi);
                const float cmu = __uint_as_float(__shfl_sync(0xffffffffu, (uint32_t)mmu, j));
                const int R = (int)__shfl_sync(0xffffffffu, mR, j);
                float xv[8];
                reinterpret_cast<uint4*>(xv)[0] = lds_u128(sin + j * C::BW + hl * 32);
                reinterpret_cast<uint4*>(xv)[1] = lds_u128(sin + j * C::BW + hl * 32 + 16);
                Lane8 e;
                // lead codes from the size pass; only the shift is redone here
                e.leads = reinterpret_cast<const uint16_t*>(p.nccodes)[(t * C::TB + bi) * 16 + hl];
                {
                    const bool raw = R >= 32;
                    const uint32_t s = raw ? 0u : ((8u - ((uint32_t)R & 7u)) & 7u);
                    const uint32_t req = ((uint32_t)R + s) >> 3;
                    e.msum = 0;
#pragma unroll
                    for (int i = 0; i < 8; i++) {
                        e.u[i] = (raw ? __float_as_uint(xv[i]) : __float_as_uint(__fsub_rn(xv[i], cmu))) >> s;
                        e.msum += req - umin_((e.leads >> (2 * i)) & 3u, req);
                    }
                }
                const uint32_t incl = half_incl_scan(e.msum);
                lane_pack_f32x8(e, R, incl - e.msum, smem_u32(stg) + sb + zo);
            }
            packed = true;
        }
    }
    if (!packed) {
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
            for (int q = 0; q < C::QV; q++) {
                using V = typename Lay<T, VPL>::V;
                reinterpret_cast<V*>(xv)[q] = lds_chunk<V>(sin + j * C::BW + (lane * C::QV + q) * C::CB);
            }
            if constexpr (sizeof(T) == 4 && VPL == 4) {
                Lane4 e;
                lane_encode_f32x4(xv, cmu, R, e);
                const uint32_t incl = warp_incl_scan(e.msum);
                lane_pack_f32x4(e, R, incl - e.msum, smem_u32(stg) + sb + zo);
            } else {
                encode_known_R<T, VPL>(xv, VPL, C::B, cmu, R, u, lc);
                pack_red<T, VPL>(u, lc, VPL, C::B, smem_u32(stg) + sb + zo);
            }
        } else {  // the partial tail block
            const int cnt = load_lane<T, VPL>(x, p.n, k, lane, xv);
            const int len = (int)(p.n - (uint64_t)k * C::B);
            encode_known_R<T, VPL>(xv, cnt, len, cmu, R, u, lc);
            pack_red<T, VPL>(u, lc, cnt, len, smem_u32(stg) + sb + zo);
        }
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
        } else {  // a boundary chunk shared with the neighbouring tiles: whole words, then bytes
            const uint32_t vw[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
            for (int q = 0; q < 4; q++) {
                const uintptr_t aw = a + 4 * q;
                if (aw >= a0 && aw + 4 <= E) {
                    *reinterpret_cast<uint32_t*>(aw) = vw[q];
                } else if (aw + 4 > a0 && aw < E) {
                    for (int c = 0; c < 4; c++)
                        if (aw + c >= a0 && aw + c < E) *reinterpret_cast<uint8_t*>(aw + c) = (uint8_t)(vw[q] >> (8 * c));
                }
            }
        }
    }
    __syncthreads();  // the staging area and input buffer are reused by the next tile
    }
}

__global__ void k_empty_header(uint8_t* out, uint32_t dtype, uint32_t mode, uint32_t b, double eb_user,
                               const uint64_t* range_keys, uint64_t* total, const double* eb_in = nullptr) {
    uint64_t* h = reinterpret_cast<uint64_t*>(out);
    h[0] = 0x31585A53ull | (1ull << 32) | ((uint64_t)dtype << 40) | ((uint64_t)mode << 48);
    h[1] = b;
    h[2] = 0;
    h[3] = (uint64_t)__double_as_longlong(eb_user);
    // REL: the (global) range of a sharded array, or no values at all -> 0
    const double e = eb_from_range(mode, eb_user, range_keys, eb_in);
    h[4] = (uint64_t)__double_as_longlong(e);
    h[5] = 0;
    h[6] = 0;
    h[7] = 0;
    if (total) *total = 64;
}

}  // namespace szx
