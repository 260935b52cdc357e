// szx_decompress.cuh -- SZx decompression kernels for sm_100a.
//
//   k_index   (K5a) the paper's "prefix-sum step to compute the starting
//             location of each block", as two chained
//             single-pass decoupled look-back scans per CTA of 256 tiles
//             (tile = 32 blocks = one bitmap word):
//               (a) nonconstant index of each tile = prefix of popcounts,
//               (b) payload byte offset of each tile = prefix of its zsize
//                   sums (the CTA's zsize range is staged in shared memory).
//             Totals are validated against the header (nNC, payload size).
//   k_decode  (K5)  persistent and warp-specialised: a producer warp reads a
//             tile's metadata and issues ONE TMA bulk copy of the tile's
//             contiguous payload (plus one for its 32 mu values) into a
//             shared-memory ring; 8 consumer warps rebuild the values with
//             the five steps of Fig. 10 and write them with
//             16-byte stores.  The leading-byte dependence chains
//             (Challenge 2) are resolved with a warp scan of
//             byte-mask transfer functions instead of the paper's log-step
//             index propagation: a lane's values map an
//             incoming previous word c to (c & M) | D, and composing such
//             maps is associative.
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
    uint32_t* ncpre;           // [nW]      nonconstant index of each tile's first block
    uint64_t* tbase;           // [nW + 1]  payload offset of each tile (tbase[nW] = total)
    int32_t* err;              // 0 ok, else SZX_ECORRUPT
};

// Stream facts read from the 64-byte header in device memory, validated
// against the caller's shape.
struct DHdr {
    uint64_t nnc, payload_bytes, off_zs, off_pl;
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
    __syncthreads();  // s_w may still be read by a previous scan
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

constexpr int kIndexTiles = 256;  // tiles (bitmap words) per k_index CTA

template <int W>
__global__ void __launch_bounds__(256) k_index(DPlan p, const uint8_t* __restrict__ in) {
    __shared__ uint64_t s_tile, s_ga, s_gb, s_w[8];
    __shared__ uint16_t s_zs[kIndexTiles * 32];
    const DHdr hd = read_dheader<W>(in, p);
    if (!hd.ok) {
        if (blockIdx.x == 0 && threadIdx.x == 0) set_corrupt(p.err);
        return;
    }
    if (threadIdx.x == 0) s_tile = atomicAdd(&p.ctr[0], 1u);
    __syncthreads();
    const uint64_t t = s_tile;
    const uint64_t ntiles = (p.nW + kIndexTiles - 1) / kIndexTiles;
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    const uint64_t w = t * kIndexTiles + threadIdx.x;
    // (a) nonconstant index of each tile
    uint32_t word = w < p.nW ? reinterpret_cast<const uint32_t*>(in + kHeaderBytes)[w] : 0u;
    if (w == p.nW - 1 && (p.nB & 31)) word &= (1u << (p.nB & 31)) - 1u;  // ignore padding bits
    const uint32_t cnt = __popc(word);
    uint64_t aggA;
    const uint64_t exA = cta_scan256(cnt, &aggA, s_w);
    if (warp == 0) {
        const uint64_t e = lookback_exclusive(p.status_a, t, aggA);
        if (lane == 0) s_ga = e;
    }
    __syncthreads();
    const uint64_t GA = s_ga;
    const uint64_t ncb = GA + exA;
    if (w < p.nW) p.ncpre[w] = (uint32_t)ncb;
    bool ok = GA + aggA <= hd.nnc;
    // (b) stage this CTA's zsize entries [GA, GA + aggA) and sum per tile
    const uint16_t* zs = reinterpret_cast<const uint16_t*>(in + hd.off_zs);
    const uint64_t nz = ok ? aggA : 0;
    for (uint64_t j = threadIdx.x; j < nz; j += 256) s_zs[j] = zs[GA + j];
    __syncthreads();
    uint64_t sum = 0;
    if (ok)
        for (uint32_t j = 0; j < cnt; j++) sum += s_zs[exA + j];
    uint64_t aggB;
    const uint64_t exB = cta_scan256(sum, &aggB, s_w);
    if (warp == 0) {
        const uint64_t e = lookback_exclusive(p.status_z, t, aggB);
        if (lane == 0) {
            s_gb = e;
            if (t == ntiles - 1) {
                p.tbase[p.nW] = e + aggB;
                if (GA + aggA != hd.nnc || e + aggB != hd.payload_bytes) set_corrupt(p.err);
            }
        }
    }
    if (!__syncthreads_and(ok ? 1 : 0) && threadIdx.x == 0) set_corrupt(p.err);
    if (w < p.nW) p.tbase[w] = s_gb + exB;
}

template <typename T, int VPL>
struct DecodeCfg {
    static constexpr int W = Traits<T>::W;
    static constexpr int B = 32 * VPL;
    static constexpr int TB = kTileBlocks;                 // blocks per tile (one bitmap word)
    static constexpr int NWARP = 8;                        // consumer warps
    static constexpr int BPW = TB / NWARP;
    static constexpr int NT = (NWARP + 1) * 32;            // + producer warp
    static constexpr int MAXZ = 1 + B / 4 + W * B;
    static constexpr int PAY = (TB * MAXZ + 32 + 15) / 16 * 16;  // + up to 15 lead / trail bytes
    static constexpr int MUB = TB * W;
    static constexpr int STAGE = PAY + MUB;
    static constexpr int STAGES = (W == 4 && VPL == 4) ? 3 : 2;
    static constexpr int SMEM = STAGES * STAGE;
    static constexpr int MINB = (W == 4 && VPL == 4) ? 3 : 2;
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
    // (3) mid-bytes -> own bytes, and the byte-mask transfer function of this lane.
    // The lane's run of mid-bytes is read as aligned words and realigned with
    // funnel shifts; value i takes the next m_i bytes of the run.
    constexpr int NW = VPL * W / 4;
    uint32_t run[NW];
    run_load<NW>(src + 1 + ncode + (incl - m), run);
    U own[VPL];
    U M = ~U(0), D = 0;  // lane map: c -> (c & M) | D
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        own[i] = 0;
        if (i < cnt) {
            const int L = (leads >> (2 * i)) & 3;
            const int mi = req > L ? req - L : 0;
            U bytes = W == 4 ? (U)run[0] : ((U)run[0] | ((U)run[1] << 16 << 16));
            bytes &= mi >= W ? ~U(0) : ((U(1) << (8 * mi)) - U(1));
            own[i] = bytes << (8 * (W - req));
            run_shr<NW>(run, mi);
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

// Fast path of decode_block for a FULL block (every lane holds VPL values):
// no per-value tail guards, explicit ld.shared, clamped funnel shifts.
// src is the shared-memory address of the block payload.
template <typename T, int VPL>
__device__ inline bool decode_full(uint32_t src, uint32_t z, T mu, T (&out)[VPL]) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    constexpr int NCODE = 8 * VPL;     // (32 * VPL) / 4
    constexpr int NW = VPL * W / 4;
    const int lane = threadIdx.x & 31;
    const int R = (int)lds_u8(src);
    if (R < TR::kFloor || R > TR::kFull) return false;
    const bool raw = R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (R & 7)) & 7);
    const int req = (R + s) >> 3;
    // (1) leading numbers: VPL/4 code bytes per lane
    uint32_t leads = 0;
#pragma unroll
    for (int q = 0; q < VPL / 4; q++) leads |= lds_u8(src + 1 + lane * (VPL / 4) + q) << (8 * q);
    uint32_t m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const int L = (leads >> (2 * i)) & 3;
        m += req > L ? req - L : 0;
    }
    const uint32_t incl = warp_incl_scan(m);
    if (1u + NCODE + __shfl_sync(0xffffffffu, incl, 31) != z) return false;
    // (3) this lane's mid-bytes; value i takes the next m_i bytes of the run
    uint32_t run[NW];
    run_load_s<NW>(src + 1 + NCODE + incl - m, run);
    U own[VPL], cmk[VPL];
    U M = ~U(0), D = 0;  // lane map: c -> (c & M) | D
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const int L = (leads >> (2 * i)) & 3;
        const int mi = req > L ? req - L : 0;
        U bytes;
        if (W == 4) {
            bytes = run[0] & ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8 * mi);  // low mi bytes (mi = 4: all)
            run_drop4<NW>(run, mi);
        } else {
            bytes = ((U)run[0] | ((U)run[1] << 16 << 16)) & (mi >= 8 ? ~U(0) : ((U(1) << (8 * mi)) - U(1)));
            run_drop4<NW>(run, mi < 4 ? mi : 4);
            run_drop4<NW>(run, mi > 4 ? mi - 4 : 0);
        }
        own[i] = bytes << (8 * (W - req));
        const int copy = L < req ? L : req;  // (2) bytes copied from the previous value
        cmk[i] = ~(~U(0) >> (8 * copy));     // top `copy` bytes (copy <= 3 < W)
        M &= cmk[i];
        D = (D & cmk[i]) | own[i];
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
    // (4) combine and overwrite the previous value, (5) left shift, add mu
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const U w = (prev & cmk[i]) | own[i];
        prev = w;
        const U vb = w << s;
        out[i] = raw ? TR::from(vb) : TR::add(TR::from(vb), mu);
    }
    return true;
}

template <typename T, int VPL>
__global__ void __launch_bounds__(DecodeCfg<T, VPL>::NT, DecodeCfg<T, VPL>::MINB)
    k_decode(DPlan p, const uint8_t* __restrict__ in, T* __restrict__ y) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = DecodeCfg<T, VPL>;
    extern __shared__ __align__(128) uint8_t smem[];
    __shared__ __align__(8) uint64_t full_bar[C::STAGES], empty_bar[C::STAGES];
    __shared__ __align__(16) uint16_t s_zw[C::STAGES][C::TB + 16];  // zsize window (TMA)
    __shared__ uint32_t s_word[C::STAGES], s_sb[C::STAGES], s_zo[C::STAGES], s_ok[C::STAGES];
    __shared__ uint64_t s_T[C::STAGES];

    pdl_wait();
    pdl_trigger();
    const DHdr hd = read_dheader<TR::W>(in, p);
    if (!hd.ok) return;  // k_index has flagged it
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5;
    if (threadIdx.x == 0) {
        for (int s = 0; s < C::STAGES; s++) {
            mbar_init(&full_bar[s], 1);
            mbar_init(&empty_bar[s], C::NWARP);
        }
        fence_mbar_init();
    }
    __syncthreads();
    const uint64_t G = gridDim.x;

    if (warp == C::NWARP) {
        // ---------------- producer: per tile, TMA bulk copies of the payload, the 32 mu
        // values and the tile's zsize window; metadata fetched 32 tiles per round trip
        const uintptr_t pl = reinterpret_cast<uintptr_t>(in + hd.off_pl);
        const uintptr_t zsb = reinterpret_cast<uintptr_t>(in + hd.off_zs);
        const uintptr_t lim = reinterpret_cast<uintptr_t>(in) + p.in_bytes;
        const uintptr_t lim16 = lim & ~uintptr_t(15);
        const uint32_t* bm = reinterpret_cast<const uint32_t*>(in + kHeaderBytes);
        int i = 0;
        for (uint64_t tb = blockIdx.x; tb < p.nW; tb += 32 * G) {
            // lane l holds the metadata of tile tb + l*G
            const uint64_t tl = tb + (uint64_t)lane * G;
            uint32_t m_word = 0, m_ncb = 0;
            uint64_t m_base = 0, m_end = 0;
            if (tl < p.nW) {
                m_word = bm[tl];
                m_ncb = p.ncpre[tl];
                m_base = p.tbase[tl];
                m_end = p.tbase[tl + 1];
            }
            for (int j = 0; j < 32; j++, i++) {
                const uint64_t t = tb + (uint64_t)j * G;
                if (t >= p.nW) break;
                uint32_t word = __shfl_sync(0xffffffffu, m_word, j);
                const uint32_t ncb = __shfl_sync(0xffffffffu, m_ncb, j);
                const uint64_t base = __shfl_sync(0xffffffffu, m_base, j);
                const uint64_t end = __shfl_sync(0xffffffffu, m_end, j);
                if (t == p.nW - 1 && (p.nB & 31)) word &= (1u << (p.nB & 31)) - 1u;
                const uint32_t cnt = __popc(word);
                const int s = i % C::STAGES;
                mbar_wait(&empty_bar[s], ((i / C::STAGES) & 1) ^ 1);
                uint8_t* pay = smem + (size_t)s * C::STAGE;
                uint8_t* mub = pay + C::PAY;
                const uint64_t Tb = end - base;
                const bool ok = end >= base && Tb <= (uint64_t)C::TB * C::MAXZ && end <= hd.payload_bytes &&
                                (uint64_t)ncb + cnt <= hd.nnc;
                const uintptr_t a0 = pl + base;
                const uintptr_t A = a0 & ~uintptr_t(15);
                const uintptr_t E = ok ? ((a0 + Tb + 15) & ~uintptr_t(15)) : A;
                const uintptr_t Eb = E < lim16 ? E : (lim16 > A ? lim16 : A);  // bulk part inside the buffer
                const uint32_t bulk = (uint32_t)(Eb - A);
                const uint64_t k0 = t * C::TB;
                const bool mu_tma = (k0 + C::TB) <= p.nB;   // full tile of mu values
                const uintptr_t za = (zsb + 2 * (uint64_t)ncb) & ~uintptr_t(15);
                const uint32_t zbytes =
                    (ok && cnt) ? (uint32_t)(((zsb + 2 * ((uint64_t)ncb + cnt) + 15) & ~uintptr_t(15)) - za) : 0u;
                if (lane == 0) {
                    mbar_expect_tx(&full_bar[s], bulk + (mu_tma ? (uint32_t)C::MUB : 0u) + zbytes);
                    if (bulk) tma_load_1d(pay, reinterpret_cast<const void*>(A), bulk, &full_bar[s]);
                    if (mu_tma) tma_load_1d(mub, in + p.off_mu + k0 * C::W, C::MUB, &full_bar[s]);
                    if (zbytes) tma_load_1d(&s_zw[s][0], reinterpret_cast<const void*>(za), zbytes, &full_bar[s]);
                    s_word[s] = word;
                    s_sb[s] = (uint32_t)(a0 & 15);
                    s_zo[s] = (uint32_t)((zsb + 2 * (uint64_t)ncb - za) >> 1);
                    s_ok[s] = ok;
                    s_T[s] = Tb;
                }
                // bytes of the last 16-byte chunk beyond the buffer's 16-byte floor
                for (uintptr_t a = Eb + lane; a < E; a += 32)
                    pay[a - A] = a < lim ? *reinterpret_cast<const uint8_t*>(a) : 0;
                if (!mu_tma) {  // last, partial tile
                    const U* mus = reinterpret_cast<const U*>(in + p.off_mu);
                    if (k0 + lane < p.nB) reinterpret_cast<U*>(mub)[lane] = mus[k0 + lane];
                }
                __syncwarp();
                if (lane == 0) mbar_arrive(&full_bar[s]);
            }
        }
        return;
    }

    // ---------------- consumers
    const uint32_t sbase = smem_u32(smem);
    const uint64_t nW_full = p.n / ((uint64_t)C::TB * C::B);   // tiles whose 32 blocks are all full
    constexpr int NV = VPL * C::W / 16;                          // 16-byte stores per lane per block
    constexpr int QB = C::B * C::W / 16;                         // 16-byte chunks per block
    const uint32_t below = (1u << lane) - 1u;
    int i = 0;
    for (uint64_t t = blockIdx.x; t < p.nW; t += G, i++) {
        const int s = i % C::STAGES;
        mbar_wait(&full_bar[s], (i / C::STAGES) & 1);
        const uint32_t pay = sbase + s * C::STAGE;
        const uint32_t mub = pay + C::PAY;
        const uint32_t word = s_word[s];
        const uint32_t cnt = __popc(word);
        // zsize of the tile's nonconstant blocks (lane r holds the r-th); validate once
        const uint32_t zl = (s_ok[s] && (uint32_t)lane < cnt) ? s_zw[s][s_zo[s] + lane] : 0u;
        const bool zok = (uint32_t)lane >= cnt || (zl >= 2 && zl <= (uint32_t)C::MAXZ);
        const bool ok = s_ok[s] && __all_sync(0xffffffffu, zok) && __reduce_add_sync(0xffffffffu, zl) == s_T[s];
        const uint32_t mine = (word >> (warp * C::BPW)) & ((1u << C::BPW) - 1u);  // my nonconstant blocks
        if (!ok) {
            if (threadIdx.x == 0) set_corrupt(p.err);
        } else if (t < nW_full) {
            // full tile: every block holds B values
            const uint32_t spay = pay + s_sb[s];
            const uint32_t smu = mub + warp * C::BPW * C::W;
            uint4* yq = reinterpret_cast<uint4*>(y + (t * C::TB + warp * C::BPW) * C::B + lane * VPL);
            // constant blocks: retrieve with mu (Fig. 10, state 0)
#pragma unroll
            for (int j = 0; j < C::BPW; j++) {
                if (!((mine >> j) & 1u)) {
                    U mb = lds_u32(smu + j * C::W);
                    if (C::W == 8) mb |= (U)lds_u32(smu + j * C::W + 4) << 16 << 16;
                    T v[VPL];
#pragma unroll
                    for (int q = 0; q < VPL; q++) v[q] = TR::from(mb);
#pragma unroll
                    for (int q = 0; q < NV; q++) yq[j * QB + q] = reinterpret_cast<const uint4*>(v)[q];
                }
            }
            // nonconstant blocks
#pragma unroll 1
            for (uint32_t m = mine; m; m &= m - 1) {
                const int j = __ffs(m) - 1;
                const int idx = warp * C::BPW + j;
                const uint32_t rank = __popc(word & ((1u << idx) - 1u));
                const uint32_t off = __reduce_add_sync(0xffffffffu, (uint32_t)lane < rank ? zl : 0u);
                const uint32_t z = __shfl_sync(0xffffffffu, zl, rank);
                U mb = lds_u32(smu + j * C::W);
                if (C::W == 8) mb |= (U)lds_u32(smu + j * C::W + 4) << 16 << 16;
                T v[VPL];
                if (!decode_full<T, VPL>(spay + off, z, TR::from(mb), v)) {
                    if (lane == 0) set_corrupt(p.err);
                    continue;
                }
#pragma unroll
                for (int q = 0; q < NV; q++) yq[j * QB + q] = reinterpret_cast<const uint4*>(v)[q];
            }
        } else {
            // last (partial) tile: generic path with bounds and tail handling
            const uint8_t* gpay = smem + (size_t)s * C::STAGE;
            const U* gmu = reinterpret_cast<const U*>(gpay + C::PAY);
            const int sb = (int)s_sb[s];
#pragma unroll 1
            for (int j = 0; j < C::BPW; j++) {
                const int idx = warp * C::BPW + j;
                const uint64_t k = t * C::TB + idx;
                if (k >= p.nB) break;
                const int len = (int)umin64(C::B, p.n - k * C::B);
                const T mu = TR::from(gmu[idx]);
                T v[VPL];
                if (!((word >> idx) & 1u)) {
#pragma unroll
                    for (int q = 0; q < VPL; q++) v[q] = mu;
                } else {
                    const uint32_t rank = __popc(word & ((1u << idx) - 1u));
                    const uint32_t off = __reduce_add_sync(0xffffffffu, (uint32_t)lane < rank ? zl : 0u);
                    const uint32_t z = __shfl_sync(0xffffffffu, zl, rank);
                    if (!decode_block<T, VPL>(gpay + sb + off, z, len, mu, v)) {
                        if (lane == 0) set_corrupt(p.err);
                        continue;
                    }
                }
                store_lane<T, VPL>(y, p.n, k, lane, v);
            }
        }
        (void)below;
        __syncwarp();
        if (lane == 0) mbar_arrive(&empty_bar[s]);
    }
}

}  // namespace szx
