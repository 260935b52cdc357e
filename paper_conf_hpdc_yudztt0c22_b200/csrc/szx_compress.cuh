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
    void* nckeys;              // their (min, max) keys, same order
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
    T mu, r;
};
template <typename T>
__device__ inline BlockClass<T> classify(typename Traits<T>::U kmn, typename Traits<T>::U kmx, double eb) {
    using TR = Traits<T>;
    BlockClass<T> c;
    c.nan = kmn < TR::kKeyNInf || kmx > TR::kKeyPInf;  // R14
    c.constant = false;
    c.mu = T(0);
    c.r = T(0);
    if (!c.nan) {
        const T mn = TR::from(okey_inv(kmn)), mx = TR::from(okey_inv(kmx));
        c.r = TR::half(TR::sub(mx, mn));   // radius r_k (R1)
        c.mu = TR::add(mn, c.r);           // mu_k = mn + r (R1)
        c.constant = ((double)c.r <= eb) && (__dsub_rn((double)mx, (double)c.mu) <= eb) &&
                     (__dsub_rn((double)c.mu, (double)mn) <= eb);  // R2 guard
    }
    return c;
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
#pragma unroll
    for (int j = 0; j < 8; j++) {
        const uint64_t k = base + j * 256 + threadIdx.x;
        bool nc = false;
        if (k < p.nB) {
            BlockClass<T> c = classify<T>(stats[2 * k], stats[2 * k + 1], eb);
            T mu = c.mu;
            if (!c.constant) {
                nc = true;
                if (c.nan || initial_R<T>(c.r, pe, p.r_bias) >= TR::kFull) mu = T(0);  // raw: mu = +0 (R15)
            }
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
    U* nckeys = reinterpret_cast<U*>(p.nckeys);
#pragma unroll
    for (int j = 0; j < 8; j++) {
        const bool nc = (ncmask >> j) & 1u;
        const uint32_t word = __ballot_sync(0xffffffffu, nc);
        if (nc) {
            const uint64_t k = base + j * 256 + threadIdx.x;
            const uint64_t idx = G + s_pre[j * 8 + warp] + __popc(word & ((1u << lane) - 1u));
            p.nclist[idx] = (uint32_t)k;
            nckeys[2 * idx] = stats[2 * k];  // keys in nonconstant order (read by TMA in k_encode)
            nckeys[2 * idx + 1] = stats[2 * k + 1];
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
__device__ inline void encode_block(const T (&xv)[VPL], int cnt, int len, const BlockClass<T>& c,
                                    double eb, int pe, int r_bias, typename Traits<T>::U (&u)[VPL],
                                    LaneCode& lc) {
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
            u[i] = vb >> s;                                                     // Solution C shift
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

// Write the block payload [R][codes][mid-bytes] into shared memory at dst.
template <typename T, int VPL>
__device__ inline void pack_block(const typename Traits<T>::U (&u)[VPL], const LaneCode& lc, int cnt, int len,
                                  uint8_t* dst) {
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
    // mid-bytes: bytes [W-req, W-lead) of each little-endian word (R7).  The
    // lane's run is assembled in registers (last value first, shifting left)
    // and written with 32-bit stores; only the partial end words go byte-wise.
    using U = typename TR::U;
    constexpr int NW = VPL * W / 4;
    uint32_t run[NW];
#pragma unroll
    for (int q = 0; q < NW; q++) run[q] = 0;
    int rlen = 0;
#pragma unroll
    for (int i = VPL - 1; i >= 0; i--) {
        if (i < cnt) {
            const int L = (lc.leads >> (2 * i)) & 3;
            const int mi = req > L ? req - L : 0;
            run_shl<NW>(run, mi);
            U bytes = u[i] >> (8 * (W - req));
            bytes &= mi >= W ? ~U(0) : ((U(1) << (8 * mi)) - U(1));
            run[0] |= (uint32_t)bytes;
            if (W == 8) run[1] |= (uint32_t)((uint64_t)bytes >> 32);
            rlen += mi;
        }
    }
    run_store<NW>(dst + 1 + ncode + lc.mexcl, run, rlen);
}

// ------------------------------------------------------------------ K2+K3+K4
template <typename T, int VPL>
struct EncodeCfg {
    static constexpr int W = Traits<T>::W;
    static constexpr int B = 32 * VPL;
    static constexpr int BW = B * W;                     // bytes per full block
    static constexpr int TB = VPL == 4 ? 32 : 16;        // nonconstant blocks per tile
    static constexpr int NWARP = 8;                      // consumer warps
    static constexpr int NC = NWARP * 32;                // consumer threads
    static constexpr int BPW = TB / NWARP;               // blocks per consumer warp
    static constexpr int NT = NC + 32;                   // + 1 producer warp
    static constexpr int STAGES = W == 4 ? 3 : 2;
    static constexpr int MAXZ = 1 + B / 4 + W * B;       // max z_k
    static constexpr int KEYB = TB * 2 * W;              // (min, max) keys of a tile
    static constexpr int RING = STAGES * (TB * BW + KEYB);
    static constexpr int STG = (16 + TB * MAXZ + 16 + 15) / 16 * 16;
    static constexpr int SMEM = RING + STG;
    static constexpr int MINB = W == 4 ? 3 : 2;          // CTAs per SM (register budget)
};

// Persistent encoder.  Tiles of TB nonconstant blocks are dealt round-robin
// (tile t -> CTA t mod G).  Payload offsets: every tile publishes its
// aggregate z-sum; tile t's exclusive prefix is this CTA's own previous
// inclusive prefix (tile t-G) plus the G-1 aggregates in between, read in
// parallel by all consumer threads -- one L2 round trip instead of a look-back
// walk across a whole round of concurrently running tiles.
template <typename T, int VPL>
__global__ void __launch_bounds__(EncodeCfg<T, VPL>::NT, EncodeCfg<T, VPL>::MINB)
    k_encode(const T* __restrict__ x, Plan p, uint8_t* __restrict__ out) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = EncodeCfg<T, VPL>;
    constexpr int W = TR::W;
    extern __shared__ __align__(128) uint8_t smem[];
    uint8_t* stg = smem + C::RING;
    __shared__ __align__(8) uint64_t full_bar[C::STAGES], empty_bar[C::STAGES];
    __shared__ uint32_t s_blk[C::STAGES][C::TB];
    __shared__ uint32_t s_z[2][C::TB];
    __shared__ uint64_t s_part[2][C::NWARP];
    __shared__ uint32_t s_lc[C::TB][32];  // per block and lane: leads | mid-byte offset << 16
    __shared__ uint8_t s_R[C::TB];

    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t nnc = *p.nnc;
    const uint64_t ntiles = (nnc + C::TB - 1) / C::TB;
    const uint64_t G = gridDim.x;
    if (threadIdx.x == 0) {
        for (int s = 0; s < C::STAGES; s++) {
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], C::NWARP);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const bool tail_partial = (p.n % C::B) != 0;
    auto slot_of = [&](int s, int bi) { return smem + (size_t)s * (C::TB * C::BW + C::KEYB) + (size_t)bi * C::BW; };
    auto keys_of = [&](int s) {
        return reinterpret_cast<const U*>(smem + (size_t)s * (C::TB * C::BW + C::KEYB) + C::TB * C::BW);
    };

    if (warp == C::NWARP) {
        // ---------------- producer: TMA the nonconstant blocks (and their keys) of each tile
        const uint8_t* nckeys = reinterpret_cast<const uint8_t*>(p.nckeys);
        uint64_t t = blockIdx.x;
        uint32_t kcur = 0;
        if (t < ntiles && lane < C::TB && t * C::TB + lane < nnc) kcur = p.nclist[t * C::TB + lane];
        for (int i = 0; t < ntiles; t += G, i++) {
            const int s = i % C::STAGES;
            // prefetch the next tile's block ids while this one is issued
            uint32_t knext = 0;
            const uint64_t tn = t + G;
            if (tn < ntiles && lane < C::TB && tn * C::TB + lane < nnc) knext = p.nclist[tn * C::TB + lane];
            mbar_wait(&empty_bar[s], ((i / C::STAGES) & 1) ^ 1);
            const uint64_t nc = t * C::TB + lane;
            const bool act = lane < C::TB && nc < nnc;
            const bool tail = act && tail_partial && (uint64_t)kcur == p.nB - 1;
            const uint32_t bytes = (act && !tail) ? (uint32_t)C::BW : 0u;  // the partial tail block is read directly
            if (lane < C::TB) s_blk[s][lane] = kcur;
            const uint32_t ntile = (uint32_t)umin64(C::TB, nnc - t * C::TB);
            const uint32_t kbytes = (ntile * 2 * W + 15) & ~15u;  // nckeys has >= 16 B of slack
            const uint32_t total = warp_sum(bytes) + kbytes;
            __syncwarp();
            if (lane == 0) {
                mbar_expect_tx(&full_bar[s], total);
                tma_load_1d(smem + (size_t)s * (C::TB * C::BW + C::KEYB) + C::TB * C::BW,
                            nckeys + t * (uint64_t)C::KEYB, kbytes, &full_bar[s]);
            }
            if (bytes) tma_load_1d(slot_of(s, lane), x + (uint64_t)kcur * C::B, bytes, &full_bar[s]);
            __syncwarp();
            if (lane == 0) mbar_arrive(&full_bar[s]);
            kcur = knext;
        }
        return;
    }

    // ---------------- consumers
    const double eb = *p.eb_abs;
    const int pe = expo_f64(eb);
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    const uint64_t off_pl = off_zs + al16(2 * nnc);
    uint16_t* zsize = reinterpret_cast<uint16_t*>(out + off_zs);
    U* mus = reinterpret_cast<U*>(out + p.off_mu);
    uint64_t incl_own = 0;  // inclusive payload prefix of this CTA's previous tile (t - G)
    int i = 0;
    for (uint64_t t = blockIdx.x; t < ntiles; t += G, i++) {
        const int s = i % C::STAGES, par = i & 1;
        mbar_wait(&full_bar[s], (i / C::STAGES) & 1);
        const U* keys = keys_of(s);
        // encode one block at a time; the shifted words go back into the
        // block's ring slot (same size as the input) and the lane state into
        // shared memory until packing
#pragma unroll 1
        for (int j = 0; j < C::BPW; j++) {
            const int bi = warp * C::BPW + j;
            const uint64_t nc = t * C::TB + bi;
            uint4* slot = reinterpret_cast<uint4*>(slot_of(s, bi)) + lane * (VPL * W / 16);
            uint32_t z = 0;
            if (nc < nnc) {
                const uint32_t k = s_blk[s][bi];
                const BlockClass<T> cls = classify<T>(keys[2 * bi], keys[2 * bi + 1], eb);
                T xv[VPL];
                int cnt = VPL;
                if (tail_partial && (uint64_t)k == p.nB - 1) {
                    cnt = load_lane<T, VPL>(x, p.n, k, lane, xv);
                } else {
#pragma unroll
                    for (int q = 0; q < VPL * W / 16; q++) reinterpret_cast<uint4*>(xv)[q] = slot[q];
                }
                const int len = (int)umin64(C::B, p.n - (uint64_t)k * C::B);
                U u[VPL];
                LaneCode lc;
                encode_block<T, VPL>(xv, cnt, len, cls, eb, pe, p.r_bias, u, lc);
#pragma unroll
                for (int q = 0; q < VPL * W / 16; q++) slot[q] = reinterpret_cast<const uint4*>(u)[q];
                s_lc[bi][lane] = lc.leads | (lc.mexcl << 16);
                z = lc.z;
                if (lane == 0) {
                    s_R[bi] = (uint8_t)lc.R;
                    if (lc.R >= TR::kFull) mus[k] = 0;  // raw by escalation: mu = +0 (R15)
                }
            }
            if (lane == 0) s_z[par][bi] = z;
        }
        bar_sync_named(1, C::NC);

        // tile scan (every warp, redundantly) and publication of the aggregate
        const uint32_t zl = lane < C::TB ? s_z[par][lane] : 0u;
        const uint32_t zincl = warp_incl_scan(zl);
        const uint32_t agg = __shfl_sync(0xffffffffu, zincl, 31);
        if (threadIdx.x == 0) st_relaxed(&p.status_c[t], kFlagAgg | agg);
        // sum of the aggregates of tiles (t - G, t): spin until each is published
        uint64_t part = 0;
        const uint64_t span = t < G ? t : G - 1;
        for (uint64_t d = threadIdx.x + 1; d <= span; d += C::NC) {
            uint64_t v;
            while (((v = ld_relaxed(&p.status_c[t - d])) & kFlagAgg) == 0) {
            }
            part += v & kValueMask;
        }
        part = warp_sum64(part);
        if (lane == 0) s_part[par][warp] = part;
        bar_sync_named(1, C::NC);
        uint64_t excl = t < G ? 0 : incl_own;
#pragma unroll
        for (int w = 0; w < C::NWARP; w++) excl += s_part[par][w];
        incl_own = excl + agg;
        if (t == ntiles - 1 && threadIdx.x == 0) {
            reinterpret_cast<uint64_t*>(out)[6] = incl_own;  // header: payload bytes
            *p.total = off_pl + incl_own;
        }
        const int sb = (int)(excl & 15);

        // pack payloads into shared memory, write zsize
#pragma unroll 1
        for (int j = 0; j < C::BPW; j++) {
            const int bi = warp * C::BPW + j;
            const uint64_t nc = t * C::TB + bi;
            const uint32_t zo = __shfl_sync(0xffffffffu, zincl - zl, bi);
            const uint32_t zb = __shfl_sync(0xffffffffu, zl, bi);
            if (nc < nnc) {
                const uint64_t k = s_blk[s][bi];
                const int len = (int)umin64(C::B, p.n - k * C::B);
                const int first = lane * VPL;
                const int cnt = first >= len ? 0 : (len - first < VPL ? len - first : VPL);
                const uint4* slot = reinterpret_cast<const uint4*>(slot_of(s, bi)) + lane * (VPL * W / 16);
                U u[VPL];
#pragma unroll
                for (int q = 0; q < VPL * W / 16; q++) reinterpret_cast<uint4*>(u)[q] = slot[q];
                const uint32_t st = s_lc[bi][lane];
                LaneCode lc;
                lc.leads = st & 0xFFFFu;
                lc.mexcl = st >> 16;
                lc.R = s_R[bi];
                lc.z = zb;
                pack_block<T, VPL>(u, lc, cnt, len, stg + sb + zo);
                if (lane == 0) zsize[nc] = (uint16_t)zb;
            }
        }
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_bar[s]);  // this warp is done with the ring stage
        bar_sync_named(1, C::NC);

        // copy the staged tile payload to global memory with 16-byte stores
        uint8_t* g0 = out + off_pl + excl;
        const uintptr_t a0 = reinterpret_cast<uintptr_t>(g0), A = a0 & ~uintptr_t(15), E = a0 + agg;
        const uint32_t nch = (uint32_t)((E - A + 15) >> 4);
        for (uint32_t ch = threadIdx.x; ch < nch; ch += C::NC) {
            const uintptr_t a = A + 16 * (uintptr_t)ch;
            if (a >= a0 && a + 16 <= E) {
                *reinterpret_cast<uint4*>(a) = *reinterpret_cast<const uint4*>(stg + 16 * ch);
            } else {
                for (int q = 0; q < 16; q++)
                    if (a + q >= a0 && a + q < E) *reinterpret_cast<uint8_t*>(a + q) = stg[16 * ch + q];
            }
        }
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
