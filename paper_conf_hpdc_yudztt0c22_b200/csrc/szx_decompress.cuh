// szx_decompress.cuh -- SZx decompression kernels for sm_100a.
//
// One persistent kernel, k_decode_w, whose grid is co-resident (<= SMs x
// occupancy):
//   (K5a) index phase -- the paper's "prefix-sum step to compute the starting
//         location of each block": per tile (32 blocks = one
//         bitmap word) its nonconstant index (prefix of popcounts) and its
//         payload byte offset (prefix of zsize sums).  Each CTA owns a
//         contiguous tile range; two grid-wide prefixes over CTA aggregates
//         replace chained look-backs.  Totals are validated against the
//         header (nNC, payload size).  A grid barrier follows.
//   (K5)  decode phase -- a warp per 32-block tile (dynamic assignment, two
//         tiles in flight): metadata, mu values and zsize entries from
//         global memory, the tile's payload staged in shared memory with
//         cp.async; values rebuilt with the five steps of Fig. 10
//          and written with 16-byte stores.  The leading-byte
//         dependence chains (Challenge 2) are resolved with a
//         warp scan of byte-mask transfer functions instead of the paper's
//         log-step index propagation: a lane's values map an
//         incoming previous word c to (c & M) | D, and composing such maps is
//         associative.
#pragma once

#include <utility>

#include "szx_device.cuh"

namespace szx {

struct DPlan {
    // host-known shape (from the caller); everything that depends on the
    // compressed content (nNC, payload size) is read from the header on the device
    uint64_t n, nB, nW, in_bytes;
    uint64_t off_mu;
    // block range to reconstruct, [kb0, kb1) (whole stream: 0, nB).  The index
    // phase covers tiles [0, nWi), nWi = ceil(kb1 / 32); only tiles >= t_lo =
    // kb0 / 32 are decoded; y points at the (virtual) element 0 of the stream.
    uint64_t kb0, kb1, nWi, t_lo;
    uint32_t b, dtype;
    uint32_t* ctr;             // [8] init 0: [0] [3] prefix arrivals, [1] [4] tile counters, [2] grid barrier
    uint64_t* slot_a;          // [grid] per-CTA nonconstant counts
    uint64_t* res_a;           // [grid] init 0: their exclusive prefixes
    uint64_t* slot_z;          // [grid] per-CTA payload byte counts
    uint64_t* res_z;           // [grid] init 0: their exclusive prefixes
    uint32_t* nctile;          // [nW]      tiles holding nonconstant blocks (+ a partial last tile)
    uint32_t* n_nctile;        // [1]       their count
    uint32_t* ncpre;           // [nW]      nonconstant index of each tile's first block
    uint64_t* tbase;           // [nW + 1]  payload offset of each tile (tbase[nW] = total)
    int32_t* err;              // 0 ok, else SZX_ECORRUPT
    uint32_t n_icta;           // CTAs that run the index phase (<= gridDim.x)
    uint32_t split;            // work items per nonconstant tile (1, 2 or 4: 32/split blocks each)
    uint32_t ts;               // dense float32 b = 128 stream: lane-per-block (thread-serial) tile decoder
    // quality variant only: the original values, indexed
    // like y, and the accumulators {max |x-x'| (double bits), sum (x-x')^2
    // (double), dkey(min finite x), ~dkey(max finite x)}, initialised by the host
    const void* ref;
    uint64_t* qual;
};

// Per-thread reconstruction-quality accumulators (the fused max-error / PSNR
// of SURVEY 8(f) row 1): Formula 1's max |x - x'| and Formula 7's MSE and
// value range, with the oracle's definitions
// (identical bits -> 0, a NaN otherwise -> +Inf; range over finite x).
struct QualAcc {
    double maxe = 0.0, sse = 0.0;
    uint64_t kmn = ~0ull, kmx = 0ull;
    template <typename T>
    __device__ __forceinline__ void add(T x, T xr) {
        using TR = Traits<T>;
        const double dx = (double)x, dr = (double)xr;
        double e = fabs(__dsub_rn(dx, dr));
        e = (dx != dx || dr != dr) ? __longlong_as_double(0x7FF0000000000000ll) : e;
        e = TR::bits(x) == TR::bits(xr) ? 0.0 : e;
        maxe = e > maxe ? e : maxe;
        sse = __dadd_rn(sse, __dmul_rn(e, e));
        const uint64_t k = dkey((uint64_t)__double_as_longlong(dx));
        const bool fin = fabs(dx) < __longlong_as_double(0x7FF0000000000000ll);
        kmn = fin && k < kmn ? k : kmn;
        kmx = fin && k > kmx ? k : kmx;
    }
    // 16-byte chunks of decoded values against the same chunks of the original
    template <typename T, int NV, typename V = uint4>
    __device__ __forceinline__ void add16(const V* ref, const V (&v)[NV]) {
#pragma unroll
        for (int q = 0; q < NV; q++) {
            const V r = ld_stream<V>(ref + q);
            const T* a = reinterpret_cast<const T*>(&r);
            const T* b = reinterpret_cast<const T*>(&v[q]);
#pragma unroll
            for (int i = 0; i < (int)sizeof(V) / (int)sizeof(T); i++) add<T>(a[i], b[i]);
        }
    }
    // warp reduction, then one set of atomics per warp
    __device__ void flush(uint64_t* q) {
        uint64_t m = (uint64_t)__double_as_longlong(maxe);
        double ss = sse;
#pragma unroll
        for (int o = 16; o; o >>= 1) {
            const uint64_t m2 = __shfl_xor_sync(0xffffffffu, m, o);
            m = m2 > m ? m2 : m;
            ss = __dadd_rn(ss, __shfl_xor_sync(0xffffffffu, ss, o));
        }
        const uint64_t a = warp_min(kmn), b = warp_max(kmx);
        if ((threadIdx.x & 31) == 0) {
            atomicMax((unsigned long long*)&q[0], (unsigned long long)m);  // e >= 0: bit order = value order
            atomicAdd(reinterpret_cast<double*>(&q[1]), ss);
            atomicMin((unsigned long long*)&q[2], (unsigned long long)a);
            atomicMin((unsigned long long*)&q[3], (unsigned long long)~b);
        }
    }
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

// --------------------------------------------------------------- index phase
// Decoder prologue (Fig. 10 needs, for every 32-block tile t, where its
// nonconstant blocks start in the zsize array and in the payload):
//   ncpre[t] = popcount of the bitmap words before t,
//   tbase[t] = sum of the zsizes of the nonconstant blocks before t.
// CTA c owns a contiguous range of tiles.  Two grid-wide prefixes over CTA
// aggregates (grid_excl_prefix: the grid is co-resident) give the CTA its
// starting nonconstant index and payload offset; it then scans its range in
// chunks of 256 tiles.  Run by all 256 threads; s_zs: 256*32 u16 scratch.
#ifndef SZX_DMINB
#define SZX_DMINB (SZX_DQUARTER ? 2 : 3)  // decoder CTAs per SM (register budget of the block decoder)
#endif
#ifndef SZX_STCS
#define SZX_STCS 1
#endif
#ifndef SZX_DF64HALF
#define SZX_DF64HALF 1       // float64 b = 128: half-warp block decoder (8 doubles per lane)
#endif
#ifndef SZX_DNR
#define SZX_DNR 1        // float32 b = 128 half-warp decoder: non-raw fast form
#endif
#ifndef SZX_DQUARTER
#define SZX_DQUARTER 0   // float32 b = 128: quarter-warp (1) or half-warp (0) block decoder
#endif
#ifndef SZX_IDXCOOP
#define SZX_IDXCOOP 1    // index phase: warp-cooperative per-tile zsize sums on dense tiles
#endif
#ifndef SZX_DMINB64
#define SZX_DMINB64 2    // float64 b = 128 decoder: CTAs per SM (register budget of the half-warp f64 form)
#endif
#ifndef SZX_IDXRED
#define SZX_IDXRED 1           // index phase: redundant bitmap prefix instead of the first grid prefix
#endif
#ifndef SZX_IDXRED_MAXW
#define SZX_IDXRED_MAXW 4096   // ... for bitmaps up to this many 32-block words (16 KB; larger: measured slower)
#endif
constexpr int kIndexChunk = 256;

// Copy zs[i0, i0 + cnt) (cnt <= 32 * kIndexChunk) into shared memory with
// aligned 16-byte loads.  The zsize section is 16-byte aligned and padded to
// a multiple of 16 bytes, so the rounded-out loads stay inside it.
__device__ inline void stage_u16(uint16_t* s_dst, const uint16_t* __restrict__ zs, uint64_t i0, uint64_t cnt) {
    const uint64_t a = i0 & ~uint64_t(7);
    const uint32_t head = (uint32_t)(i0 - a);
    const uint32_t nq = (uint32_t)((head + cnt + 7) / 8);
    for (uint32_t q = threadIdx.x; q < nq; q += kIndexChunk) {
        const uint4 v = *reinterpret_cast<const uint4*>(zs + a + 8 * q);
        const uint32_t e[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
        for (int k = 0; k < 8; k++) {
            const int64_t d = (int64_t)(8 * q + k) - head;
            if (d >= 0 && (uint64_t)d < cnt) s_dst[d] = (uint16_t)(e[k >> 1] >> (16 * (k & 1)));
        }
    }
}

// diagnostic timing builds only: index-phase stamps of thread 0 per index CTA
// (after the first prefix, after the second prefix, after the per-tile pass)
#ifndef SZX_TIMELINE
#define SZX_TIMELINE 0
#endif
#if SZX_TIMELINE
__device__ uint64_t g_tli[2048 * 8];
#define SZX_TLI(k)                                                                    \
    do {                                                                              \
        if (threadIdx.x == 0 && blockIdx.x < 2048) {                                  \
            uint64_t t_;                                                              \
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_) : : "memory");       \
            g_tli[(uint64_t)blockIdx.x * 8 + (k)] = t_;                               \
        }                                                                             \
    } while (0)
#else
#define SZX_TLI(k) do { } while (0)
#endif

template <int W>
__device__ inline void index_phase(const DPlan& p, const uint8_t* __restrict__ in, const DHdr& hd,
                                   uint16_t* s_zs, uint64_t* s_w) {
    const uint64_t G = p.n_icta, c = blockIdx.x;  // the first n_icta CTAs share the index work
    const uint64_t w0 = p.nWi * c / G, w1 = p.nWi * (c + 1) / G;
    const uint32_t* bm = reinterpret_cast<const uint32_t*>(in + kHeaderBytes);
    const uint16_t* zs = reinterpret_cast<const uint16_t*>(in + hd.off_zs);
    auto word_at = [&](uint64_t w) -> uint32_t {
        uint32_t x = bm[w];
        if (w == p.nW - 1 && (p.nB & 31)) x &= (1u << (p.nB & 31)) - 1u;  // ignore padding bits
        return x;
    };
    // tiles the nonconstant warps visit: those with nonconstant blocks, and a
    // partial last tile (it is decoded whole by the generic path)
    const uint64_t nW_full = p.n / ((uint64_t)kTileBlocks * 32 * (p.b / 32));
    auto nc_tile = [&](uint64_t w, uint32_t word) -> uint64_t {
        return ((word != 0u || w >= nW_full) && w >= p.t_lo) ? 1u : 0u;
    };
    // (1) nonconstant blocks (low 32 bits) and such tiles (high 32 bits) in the
    // range -> starting nonconstant index and list position.  Both fit 32 bits:
    // nB <= kMaxN / 32 = 2^31 (static_assert beside kMaxN in szx_api.cu).
    // Bitmaps up to SZX_IDXRED_MAXW words: every index CTA also counts the
    // words before its range itself (16-byte loads, mostly L2 hits), which
    // replaces the first grid-wide prefix; larger ones take the prefix.
    const bool red = SZX_IDXRED && p.nWi <= (uint64_t)SZX_IDXRED_MAXW;
    uint64_t cnt = 0, pre = 0;
    if (red) {
        const uint64_t nq = (w1 + 3) / 4;  // 4-word groups of [0, w1) (the bitmap section is 16-byte padded)
#pragma unroll 8
        for (uint64_t qq = threadIdx.x; qq < nq; qq += kIndexChunk) {
            const uint4 v = *reinterpret_cast<const uint4*>(bm + 4 * qq);
            const uint32_t e[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
            for (int k = 0; k < 4; k++) {
                const uint64_t w = 4 * qq + k;
                uint32_t x = e[k];
                if (w == p.nW - 1 && (p.nB & 31)) x &= (1u << (p.nB & 31)) - 1u;
                const uint64_t a = w < w1 ? (__popc(x) | (nc_tile(w, x) << 32)) : 0u;
                if (w < w0) pre += a;
                else cnt += a;
            }
        }
    } else {
        for (uint64_t w = w0 + threadIdx.x; w < w1; w += kIndexChunk) {
            const uint32_t x = word_at(w);
            cnt += __popc(x) | (nc_tile(w, x) << 32);
        }
    }
    const uint64_t aggP = cta_sum64(cnt, s_w);
    SZX_TLI(0);
    const uint64_t exP = red ? cta_sum64(pre, s_w)
                             : grid_excl_prefix(p.slot_a, p.res_a, &p.ctr[0], aggP, s_w, (uint32_t)G);
    SZX_TLI(1);
    const uint64_t aggA = aggP & 0xFFFFFFFFu, exA = exP & 0xFFFFFFFFu;
    uint64_t runT = exP >> 32;
    const bool ok = exA + aggA <= hd.nnc;
    // (2) their payload bytes -> starting payload offset.  A range of at most
    // one chunk keeps its zsizes in shared memory for step (3).
    const bool one = w1 - w0 <= (uint64_t)kIndexChunk;
    uint64_t zsum = 0;
    if (ok) {
        if (one) {
            stage_u16(s_zs, zs, exA, aggA);
            __syncthreads();
            for (uint32_t j = threadIdx.x; j < aggA; j += kIndexChunk) zsum += s_zs[j];
        } else {
            for (uint64_t i = exA + threadIdx.x; i < exA + aggA; i += kIndexChunk) zsum += zs[i];
        }
    }
    const uint64_t aggZ = cta_sum64(zsum, s_w);
    SZX_TLI(2);
    const uint64_t exZ = grid_excl_prefix(p.slot_z, p.res_z, &p.ctr[3], aggZ, s_w, (uint32_t)G);
    SZX_TLI(3);
    // (3) per tile: ncpre and tbase
    uint64_t runA = exA, runZ = exZ;
    for (uint64_t wc = w0; wc < w1; wc += kIndexChunk) {
        const uint64_t w = wc + threadIdx.x;
        const uint32_t word = w < w1 ? word_at(w) : 0u;
        const uint32_t cw = __popc(word);
        const uint64_t isnc = w < w1 ? nc_tile(w, word) : 0u;
        uint64_t totP;
        const uint64_t exq = cta_scan256(cw | (isnc << 32), &totP, s_w);
        const uint64_t ex = exq & 0xFFFFFFFFu, tot = totP & 0xFFFFFFFFu;
        if (w < w1) {
            p.ncpre[w] = (uint32_t)(runA + ex);
            if (isnc) p.nctile[runT + (exq >> 32)] = (uint32_t)w;
        }
        runT += totP >> 32;
        if (!one) {
            if (ok) stage_u16(s_zs, zs, runA, tot);
            __syncthreads();
        }
        // per-tile payload bytes.  Dense tiles: the warp sums each of its 32
        // tiles' zsizes together (consecutive u16 reads; a thread-serial loop
        // over 32 zsizes per thread hits 2 banks from 32 threads)
        uint64_t sum = 0;
        if (ok && (!SZX_IDXCOOP || __reduce_min_sync(0xffffffffu, cw) < 16u)) {
            for (uint32_t j = 0; j < cw; j++) sum += s_zs[ex + j];  // a warp with a sparse tile: serial sums
        } else if (ok) {
            const int lane = threadIdx.x & 31;
#pragma unroll 4
            for (int k = 0; k < 32; k++) {
                const uint32_t exk = __shfl_sync(0xffffffffu, (uint32_t)ex, k);
                const uint32_t cwk = __shfl_sync(0xffffffffu, cw, k);
                uint32_t v = (uint32_t)lane < cwk ? (uint32_t)s_zs[exk + lane] : 0u;
#pragma unroll
                for (int o = 16; o > 0; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
                if (lane == k) sum = v;
            }
        }
        uint64_t totz;
        const uint64_t exz = cta_scan256(sum, &totz, s_w);
        if (w < w1) p.tbase[w] = runZ + exz;
        runA += tot;
        runZ += totz;
        __syncthreads();  // s_zs is refilled by the next chunk
    }
    SZX_TLI(4);
    if (threadIdx.x == 0) {
        if (!ok) set_corrupt(p.err);
        if (c == G - 1) {
            p.tbase[p.nWi] = runZ;
            *p.n_nctile = (uint32_t)runT;
            // totals: exact for the whole stream, bounded for a prefix of it
            if (p.nWi == p.nW ? (runA != hd.nnc || runZ != hd.payload_bytes)
                              : (runA > hd.nnc || runZ > hd.payload_bytes))
                set_corrupt(p.err);
        }
    }
}

template <typename T, int VPL>
__device__ inline void store_lane(T* __restrict__ y, uint64_t n, uint64_t k, int lane, const T (&v)[VPL]) {
    constexpr int B = 32 * VPL;
    const uint64_t first = k * B + (uint64_t)lane * VPL;
    if ((k + 1) * B <= n) {
        using LY = Lay<T, VPL>;
        using V = typename LY::V;
        V* q = reinterpret_cast<V*>(y + first);
#pragma unroll
        for (int i = 0; i < LY::NQ; i++) q[i] = reinterpret_cast<const V*>(v)[i];
        return;
    }
#pragma unroll
    for (int i = 0; i < VPL; i++)
        if (first + i < n) y[first + i] = v[i];
}

namespace gsrc {
// generic-address loads: the source is either a shared-memory staging slot or
// the stream in global memory (fallback for oversized tiles)
__device__ inline uint32_t ldg_u8(const uint8_t* p) { return *p; }
__device__ inline uint32_t ldg_u32(const void* p) { return *reinterpret_cast<const uint32_t*>(p); }
// run of bytes at an arbitrary address, realigned; aligned words that start at
// or past `lim` (one past the last valid byte) read as 0.  An aligned word
// holding at least one stream byte never leaves the (>=16-B aligned) buffer.
// the aligned word at w, with the bytes at or past lim read as 0 (never loaded:
// the caller's buffer may end, or be uninitialised, right after the stream)
__device__ inline uint32_t ldg_u32_lim(uintptr_t w, uintptr_t lim) {
    if (w + 4 <= lim) return ldg_u32(reinterpret_cast<const void*>(w));
    uint32_t v = 0;
    for (uintptr_t c = w; c < lim; c++) v |= ldg_u8(reinterpret_cast<const uint8_t*>(c)) << (8 * (uint32_t)(c - w));
    return v;
}
template <int NW>
__device__ inline void run_load(const uint8_t* p, uintptr_t lim4, uint32_t (&r)[NW]) {
    const uintptr_t a = reinterpret_cast<uintptr_t>(p);
    const uintptr_t base = a & ~uintptr_t(3);
    const uint32_t sh = 8 * (uint32_t)(a & 3);
    uint32_t lo = ldg_u32_lim(base, lim4);
#pragma unroll
    for (int q = 0; q < NW; q++) {
        const uintptr_t aq = base + 4 * (q + 1);
        const uint32_t hi = ldg_u32_lim(aq, lim4);
        r[q] = __funnelshift_r(lo, hi, sh);
        lo = hi;
    }
}
}  // namespace gsrc

// Where a nonconstant block's payload is read from: the stream in global
// memory (bounded by the end of the buffer) or a shared-memory staging slot.
struct SrcG {
    const uint8_t* p;
    uintptr_t lim;
    __device__ uint32_t u8(uint32_t o) const { return gsrc::ldg_u8(p + o); }
    template <int NW>
    __device__ void run(uint32_t o, uint32_t (&r)[NW]) const { gsrc::run_load<NW>(p + o, lim, r); }
};
struct SrcS {
    uint32_t a;  // shared-window address
    __device__ uint32_t u8(uint32_t o) const { return lds_u8(a + o); }
    template <int NW>
    __device__ void run(uint32_t o, uint32_t (&r)[NW]) const { run_load_s<NW>(a + o, r); }
};

// Decode one nonconstant block (any length) whose payload (z bytes) starts at src (global).
template <typename T, int VPL, typename Src>
__device__ inline bool decode_block_g(const Src src, uint32_t z, int len, T mu,
                                      T (&out)[VPL]) {
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    const int lane = threadIdx.x & 31;
    const int ncode = (len + 3) / 4;
    const int R = (int)src.u8(0);
    if (R < TR::kFloor || R > TR::kFull) return false;
    const bool raw = R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (R & 7)) & 7);
    const int req = (R + s) >> 3;
    const int first = lane * VPL;
    const int cnt = first >= len ? 0 : min(VPL, len - first);
    // (1) read the leading numbers
    uint32_t leads = 0;
    if constexpr (VPL >= 4) {
#pragma unroll
        for (int q = 0; q < VPL / 4; q++) {
            const int cb = lane * (VPL / 4) + q;
            if (cb < ncode) leads |= src.u8(1 + cb) << (8 * q);
        }
    } else {  // 4 / VPL lanes share a code byte
        if ((int)code_byte<VPL>(lane) < ncode)
            leads = (src.u8(1 + code_byte<VPL>(lane)) >> code_shift<VPL>(lane)) & ((1u << (2 * VPL)) - 1u);
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
    src.template run<NW>(1 + ncode + (incl - m), run);
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

// ===================================================================== K5w
// Warp-granular decoder: a warp owns whole 32-block tiles (grid-stride), reads
// the tile's metadata, mu values, zsize entries and the nonconstant payloads
// straight from global memory (read-only path), and writes 16-byte stores.
// No shared-memory ring, no block-level barriers: latency is hidden by having
// many independent warps per SM, and the per-tile bookkeeping is amortised
// over 32 blocks per warp.


// Fast path for the headline shape (float32, b = 128: 4 values per lane),
// written branch-free: per value one bit-field extract, min/sub for the
// mid-byte count, a funnel-shift window into the lane's run (two 2-word run
// loads cover the lane's <= 16 bytes), one LOP3 per map composition, and an
// unpredicated warp scan of the lead-byte maps (a lane's own map composed
// with itself is itself, so lanes below the shuffle distance need no guard).
template <typename Src>
__device__ __forceinline__ bool decode_full_f32x4(const Src src, uint32_t z, float mu, float (&out)[4]) {
    const int lane = threadIdx.x & 31;
    const uint32_t R = src.u8(0);
    if (R < 9u || R > 32u) return false;
    const bool raw = R >= 32u;
    const uint32_t s = raw ? 0u : ((8u - (R & 7u)) & 7u);
    const uint32_t req = (R + s) >> 3;           // 2..4 kept bytes
    const uint32_t leads = src.u8(1 + lane);
    uint32_t m[4], nm[4];
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const uint32_t L = (leads >> (2 * i)) & 3u;
        const uint32_t copy = L < req ? L : req;
        m[i] = req - copy;
        nm[i] = 0xFFFFFFFFu >> (8 * copy);      // bytes NOT copied from the previous value
    }
    const uint32_t m01 = m[0] + m[1];
    const uint32_t msum = m01 + m[2] + m[3];
    const uint32_t incl = warp_incl_scan(msum);
    if (33u + __shfl_sync(0xffffffffu, incl, 31) != z) return false;
    const uint32_t o = 33u + incl - msum;
    uint32_t ra[2], rb[2];
    src.template run<2>(o, ra);
    src.template run<2>(o + m01, rb);
    const uint32_t drop = 8u * (4u - req);
    auto lowmask = [](uint32_t mm) { return ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8u * mm); };
    uint32_t own[4];
    own[0] = (ra[0] & lowmask(m[0])) << drop;
    own[1] = (__funnelshift_rc(ra[0], ra[1], 8u * m[0]) & lowmask(m[1])) << drop;
    own[2] = (rb[0] & lowmask(m[2])) << drop;
    own[3] = (__funnelshift_rc(rb[0], rb[1], 8u * m[2]) & lowmask(m[3])) << drop;
    // lane map c -> (c & M) | D
    uint32_t cM = ~(nm[0] | nm[1] | nm[2] | nm[3]);
    uint32_t cD = own[0];
#pragma unroll
    for (int i = 1; i < 4; i++) cD = (cD & ~nm[i]) | own[i];
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t pM = __shfl_up_sync(0xffffffffu, cM, d);
        const uint32_t pD = __shfl_up_sync(0xffffffffu, cD, d);
        cD = (pD & cM) | cD;
        cM = pM & cM;
    }
    uint32_t prev = __shfl_up_sync(0xffffffffu, cD, 1);
    prev = lane == 0 ? 0u : prev;
#pragma unroll
    for (int i = 0; i < 4; i++) {
        const uint32_t w = (prev & ~nm[i]) | own[i];
        prev = w;
        out[i] = raw ? __uint_as_float(w) : __fadd_rn(__uint_as_float(w << s), mu);
    }
    return true;
}

// ---- two float32 blocks of b = 128 per warp: a half-warp per block, 8 values
// per lane.  Same arithmetic as decode_full_f32x4 (Fig. 10's five steps), but
// every per-lane step -- R / code parsing, the mid-byte scan, the lead-byte
// map scan, the z check -- is paid once per 8 values instead of once per 4.
// Inclusive prefix sum within 16-lane segments (predicated by shfl's in-segment flag)
template <int O>
__device__ __forceinline__ uint32_t shfl_up_add16(uint32_t v) {
    asm volatile(
        "{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
        "shfl.sync.up.b32 t|p, %0, %1, 0x1000, -1;\n\t"
        "@p add.u32 %0, %0, t;\n\t}"
        : "+r"(v)
        : "n"(O));
    return v;
}
// Half-warp h decodes the block whose payload starts at shared address a
// (z bytes); returns false (for the whole half) on a malformed block.
__device__ __forceinline__ bool decode_half_f32x8(uint32_t a, uint32_t z, float mu, float (&out)[8]) {
    const int sl = threadIdx.x & 15;
    const uint32_t R = lds_u8(a);
    const bool bad = R < 9u || R > 32u;
    const bool raw = R >= 32u;
    const uint32_t s = raw ? 0u : ((8u - (R & 7u)) & 7u);
    const uint32_t r8 = bad ? 32u : (R + s);            // kept bits: 8 x (2..4 bytes)
    const uint32_t drop = 32u - r8;
    const uint32_t leads = lds_u8(a + 1 + 2 * sl) | (lds_u8(a + 2 + 2 * sl) << 8);
    // per value, in bits: c8 = 8 x bytes copied from the previous value
    // (min(lead, req), step 2), m8 = 8 x mid-bytes read (step 3); nm masks the
    // bytes NOT copied
    uint32_t m8[8], nm[8];
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t c8 = umin((leads >> (2 * i) << 3) & 24u, r8);
        m8[i] = r8 - c8;
        nm[i] = 0xFFFFFFFFu >> c8;
    }
    const uint32_t b01 = m8[0] + m8[1], b23 = m8[2] + m8[3], b45 = m8[4] + m8[5];
    const uint32_t msum = (b01 + b23 + b45 + m8[6] + m8[7]) >> 3;
    uint32_t incl = shfl_up_add16<1>(msum);
    incl = shfl_up_add16<2>(incl);
    incl = shfl_up_add16<4>(incl);
    incl = shfl_up_add16<8>(incl);
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 15, 16);
    const bool ok = !bad && 33u + tot == z;
    const uint32_t o = a + 33u + incl - msum;
    uint32_t r[4][2];
    run_load_s<2>(o, r[0]);
    run_load_s<2>(o + (b01 >> 3), r[1]);
    run_load_s<2>(o + ((b01 + b23) >> 3), r[2]);
    run_load_s<2>(o + ((b01 + b23 + b45) >> 3), r[3]);
    // value i's mid-bytes moved to their place under the copied top bytes:
    // sw & nm (the bytes below them are zero after the shift)
    uint32_t sw[8];
#pragma unroll
    for (int q = 0; q < 4; q++) {
        sw[2 * q] = r[q][0] << drop;
        sw[2 * q + 1] = __funnelshift_rc(r[q][0], r[q][1], m8[2 * q]) << drop;
    }
    // lane map c -> (c & M) | D, then its exclusive scan within the half
    uint32_t cM = ~(nm[0] | nm[1] | nm[2] | nm[3] | nm[4] | nm[5] | nm[6] | nm[7]);
    uint32_t cD = sw[0] & nm[0];
#pragma unroll
    for (int i = 1; i < 8; i++) cD = (cD & ~nm[i]) | (sw[i] & nm[i]);
#pragma unroll
    for (int d = 1; d < 16; d <<= 1) {
        const uint32_t pM = __shfl_up_sync(0xffffffffu, cM, d, 16);
        const uint32_t pD = __shfl_up_sync(0xffffffffu, cD, d, 16);
        // lanes below d in the half get their own map back: composing a map
        // with itself leaves it unchanged
        cD = (pD & cM) | cD;
        cM = pM & cM;
    }
    uint32_t prev = __shfl_up_sync(0xffffffffu, cD, 1, 16);
    prev = sl == 0 ? 0u : prev;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t w = (prev & ~nm[i]) | (sw[i] & nm[i]);
        prev = w;
        out[i] = raw ? __uint_as_float(w) : __fadd_rn(__uint_as_float(w << s), mu);
    }
    return ok;
}

// decode_half_f32x8 for non-raw blocks (9 <= R < 32, read by the caller):
// the shifts by the block constants drop and s are multiplications by powers
// of two (FMA pipe), the code cap min(code, req) is applied once per lane to
// the packed codes, and there is no raw select per value.
__device__ __forceinline__ bool decode_half_f32x8_nr(uint32_t a, uint32_t R, uint32_t z, float mu,
                                                     float (&out)[8]) {
    const int sl = threadIdx.x & 15;
    const uint32_t s = (8u - (R & 7u)) & 7u;
    const uint32_t r8 = R + s;                     // kept bits: 16, 24 or 32
    // opaque powers of two: the shifts by drop and s become IMADs (FMA pipe), not SHFs
    const uint32_t pdrop = launder(1u << (32u - r8));
    const uint32_t ps = launder(1u << s);
    uint32_t codes = lds_u8(a + 1 + 2 * sl) | (lds_u8(a + 2 + 2 * sl) << 8);
    codes ^= codes & (codes >> 1) & (r8 == 16u ? 0x5555u : 0u);  // req = 2: code 3 copies 2 bytes
    uint32_t m8[8], nm[8];
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t c8 = i == 0 ? (codes << 3) & 24u : i == 1 ? (codes << 1) & 24u : (codes >> (2 * i - 3)) & 24u;
        m8[i] = r8 - c8;
        nm[i] = 0xFFFFFFFFu >> c8;
    }
    const uint32_t b01 = m8[0] + m8[1], b23 = m8[2] + m8[3], b45 = m8[4] + m8[5];
    const uint32_t msum = (b01 + b23 + b45 + m8[6] + m8[7]) >> 3;
    uint32_t incl = shfl_up_add16<1>(msum);
    incl = shfl_up_add16<2>(incl);
    incl = shfl_up_add16<4>(incl);
    incl = shfl_up_add16<8>(incl);
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 15, 16);
    const bool ok = 33u + tot == z;
    const uint32_t o = a + 33u + incl - msum;
    uint32_t r[4][2];
    run_load_s<2>(o, r[0]);
    run_load_s<2>(o + (b01 >> 3), r[1]);
    run_load_s<2>(o + ((b01 + b23) >> 3), r[2]);
    run_load_s<2>(o + ((b01 + b23 + b45) >> 3), r[3]);
    uint32_t sw[8];
#pragma unroll
    for (int q = 0; q < 4; q++) {
        sw[2 * q] = r[q][0] * pdrop;
        sw[2 * q + 1] = __funnelshift_rc(r[q][0], r[q][1], m8[2 * q]) * pdrop;
    }
    uint32_t cM = ~(nm[0] | nm[1] | nm[2] | nm[3] | nm[4] | nm[5] | nm[6] | nm[7]);
    uint32_t cD = sw[0] & nm[0];
#pragma unroll
    for (int i = 1; i < 8; i++) cD = bitsel(cD, sw[i], nm[i]);
#pragma unroll
    for (int d = 1; d < 16; d <<= 1) {
        const uint32_t pM = __shfl_up_sync(0xffffffffu, cM, d, 16);
        const uint32_t pD = __shfl_up_sync(0xffffffffu, cD, d, 16);
        cD = (pD & cM) | cD;
        cM = pM & cM;
    }
    uint32_t prev = __shfl_up_sync(0xffffffffu, cD, 1, 16);
    prev = sl == 0 ? 0u : prev;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t w = bitsel(prev, sw[i], nm[i]);
        prev = w;
        out[i] = __fadd_rn(__uint_as_float(w * ps), mu);
    }
    return ok;
}

// ---- two float64 blocks of b = 128 per warp: a half-warp per block, 8 doubles
// per lane (Fig. 10's five steps).  A value copies at most 3 leading bytes, all
// in the high word, so the lead-byte chains (the map scan) run on 32-bit high
// words; the low words are the value's own mid-bytes.  Non-raw blocks
// (12 <= R < 64).
__device__ __forceinline__ bool decode_half_f64x8_nr(uint32_t a, uint32_t R, uint32_t z, double mu,
                                                     double (&out)[8]) {
    const int sl = threadIdx.x & 15;
    const uint32_t s = (8u - (R & 7u)) & 7u;
    const uint32_t r8 = R + s;  // kept bits: 16 .. 64
    const uint32_t drop = 64u - r8;
    uint32_t codes = lds_u8(a + 1 + 2 * sl) | (lds_u8(a + 2 + 2 * sl) << 8);
    codes ^= codes & (codes >> 1) & (r8 == 16u ? 0x5555u : 0u);  // req = 2: code 3 copies 2 bytes
    uint32_t m8[8], nmh[8];
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t c8 = ((codes >> (2 * i)) & 3u) << 3;
        m8[i] = r8 - c8;
        nmh[i] = 0xFFFFFFFFu >> c8;  // high-word bytes NOT copied from the previous value
    }
    uint32_t msum = 0;
#pragma unroll
    for (int i = 0; i < 8; i++) msum += m8[i];
    msum >>= 3;
    uint32_t incl = shfl_up_add16<1>(msum);
    incl = shfl_up_add16<2>(incl);
    incl = shfl_up_add16<4>(incl);
    incl = shfl_up_add16<8>(incl);
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 15, 16);
    const bool ok = 33u + tot == z;
    uint32_t off = a + 33u + incl - msum;
    uint32_t own_lo[8], own_hi[8];
#pragma unroll
    for (int i = 0; i < 8; i++) {
        uint32_t r[2];
        run_load_s<2>(off, r);
        uint64_t c = ((uint64_t)r[1] << 32) | r[0];
        c = m8[i] >= 64u ? c : (c & ((1ull << m8[i]) - 1ull));
        const uint64_t own = c << drop;  // the mid-bytes under the copied ones
        own_lo[i] = (uint32_t)own;
        own_hi[i] = (uint32_t)(own >> 32);
        off += m8[i] >> 3;
    }
    uint32_t cM = ~(nmh[0] | nmh[1] | nmh[2] | nmh[3] | nmh[4] | nmh[5] | nmh[6] | nmh[7]);
    uint32_t cD = own_hi[0] & nmh[0];
#pragma unroll
    for (int i = 1; i < 8; i++) cD = bitsel(cD, own_hi[i], nmh[i]);
#pragma unroll
    for (int d = 1; d < 16; d <<= 1) {
        const uint32_t pM = __shfl_up_sync(0xffffffffu, cM, d, 16);
        const uint32_t pD = __shfl_up_sync(0xffffffffu, cD, d, 16);
        cD = (pD & cM) | cD;
        cM = pM & cM;
    }
    uint32_t prev = __shfl_up_sync(0xffffffffu, cD, 1, 16);
    prev = sl == 0 ? 0u : prev;
#pragma unroll
    for (int i = 0; i < 8; i++) {
        const uint32_t wh = bitsel(prev, own_hi[i], nmh[i]);
        prev = wh;
        const uint64_t w = ((uint64_t)wh << 32) | own_lo[i];
        out[i] = __dadd_rn(__longlong_as_double((long long)(w << s)), mu);
    }
    return ok;
}

// ---- four float32 blocks of b = 128 per warp: a quarter-warp (8 lanes) per
// block, 16 values per lane.  Fig. 10's five steps as in
// decode_half_f32x8; the per-lane steps (R and code parsing, the mid-byte
// scan, the lead-byte map scan, the z check) are paid once per 16 values and
// the scans take three shuffle steps.  Shifts by the block constants drop and
// s are multiplications by powers of two (FMA pipe), so the integer ALU only
// sees the per-value extract / mask / select work.  Non-raw blocks only
// (9 <= R < 32): the caller routes raw or malformed blocks to the generic path.
template <int O>
__device__ __forceinline__ uint32_t shfl_up_add8(uint32_t v) {
    asm volatile(
        "{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
        "shfl.sync.up.b32 t|p, %0, %1, 0x1800, -1;\n\t"
        "@p add.u32 %0, %0, t;\n\t}"
        : "+r"(v)
        : "n"(O));
    return v;
}
// quarter q decodes the block whose payload starts at shared address a (z
// bytes, R read by the caller); returns false (whole quarter) on a malformed block
__device__ __forceinline__ bool decode_quarter_f32x16(uint32_t a, uint32_t R, uint32_t z, float mu,
                                                      float (&out)[16]) {
    const int ql = threadIdx.x & 7;
    const uint32_t s = (8u - (R & 7u)) & 7u;
    const uint32_t r8 = R + s;                       // kept bits: 16, 24 or 32
    const uint32_t pdrop = launder(1u << (32u - r8));  // x 2^drop: the kept bytes to the top (IMAD)
    const uint32_t ps = launder(1u << s);              // x 2^s: Formula 5's left shift (IMAD)
    // this lane's 16 codes (4 bytes at a + 1 + 4 ql, any alignment)
    uint32_t codes;
    {
        const uint32_t ca = a + 1u + 4u * (uint32_t)ql;
        const uint32_t w0 = lds_u32(ca & ~3u), w1 = lds_u32((ca & ~3u) + 4u);
        codes = __funnelshift_r(w0, w1, 8u * (ca & 3u));
    }
    // copy = min(code, req): only req = 2 caps a code (3 -> 2): clear the low bit of every 3
    {
        const uint32_t m = r8 == 16u ? 0x55555555u : 0u;
        codes ^= codes & (codes >> 1) & m;
    }
    // c8 = 8 x bytes copied from the previous value (step 2); m8 = 8 x mid-bytes (step 3);
    // nm = mask of the bytes NOT copied
    uint32_t m8[16], nm[16];
#pragma unroll
    for (int i = 0; i < 16; i++) {
        const uint32_t c8 = i == 0 ? (codes << 3) & 24u : i == 1 ? (codes << 1) & 24u : (codes >> (2 * i - 3)) & 24u;
        m8[i] = r8 - c8;
        nm[i] = 0xFFFFFFFFu >> c8;
    }
    uint32_t pre[8];  // bit offset of pair p within the lane's run
    pre[0] = 0;
#pragma unroll
    for (int p = 1; p < 8; p++) pre[p] = pre[p - 1] + m8[2 * p - 2] + m8[2 * p - 1];
    const uint32_t msum = (pre[7] + m8[14] + m8[15]) >> 3;
    uint32_t incl = shfl_up_add8<1>(msum);
    incl = shfl_up_add8<2>(incl);
    incl = shfl_up_add8<4>(incl);
    const uint32_t tot = __shfl_sync(0xffffffffu, incl, 7, 8);
    const bool ok = 33u + tot == z;
    const uint32_t o = a + 33u + incl - msum;
    // value i's mid-bytes moved to their place under the copied top bytes
    uint32_t sw[16];
#pragma unroll
    for (int p = 0; p < 8; p++) {
        uint32_t r[2];
        run_load_s<2>(o + (pre[p] >> 3), r);
        sw[2 * p] = r[0] * pdrop;
        sw[2 * p + 1] = __funnelshift_rc(r[0], r[1], m8[2 * p]) * pdrop;
    }
    // lane map c -> (c & M) | D, then its exclusive scan within the quarter
    uint32_t orm = nm[0];
#pragma unroll
    for (int i = 1; i < 16; i++) orm |= nm[i];
    uint32_t cM = ~orm;
    uint32_t cD = sw[0] & nm[0];
#pragma unroll
    for (int i = 1; i < 16; i++) cD = (cD & ~nm[i]) | (sw[i] & nm[i]);
#pragma unroll
    for (int d = 1; d < 8; d <<= 1) {
        const uint32_t pM = __shfl_up_sync(0xffffffffu, cM, d, 8);
        const uint32_t pD = __shfl_up_sync(0xffffffffu, cD, d, 8);
        cD = (pD & cM) | cD;   // lanes below d get their own map back (idempotent)
        cM = pM & cM;
    }
    uint32_t prev = __shfl_up_sync(0xffffffffu, cD, 1, 8);
    prev = ql == 0 ? 0u : prev;
#pragma unroll
    for (int i = 0; i < 16; i++) {
        const uint32_t w = (prev & ~nm[i]) | (sw[i] & nm[i]);
        prev = w;
        out[i] = __fadd_rn(__uint_as_float(w * ps), mu);
    }
    return ok;
}

// decode_full with the payload in global memory
template <typename T, int VPL, typename Src>
__device__ inline bool decode_full_g(const Src src, uint32_t z, T mu, T (&out)[VPL]) {
    if constexpr (sizeof(T) == 4 && VPL == 4) {
        return decode_full_f32x4<Src>(src, z, mu, out);
    }
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int W = TR::W;
    constexpr int NCODE = 8 * VPL;
    constexpr int NW = VPL * W / 4;
    const int lane = threadIdx.x & 31;
    const int R = (int)src.u8(0);
    if (R < TR::kFloor || R > TR::kFull) return false;
    const bool raw = R >= TR::kFull;
    const int s = raw ? 0 : ((8 - (R & 7)) & 7);
    const int req = (R + s) >> 3;
    uint32_t leads = 0;
#pragma unroll
    for (int q = 0; q < VPL / 4; q++) leads |= src.u8(1 + lane * (VPL / 4) + q) << (8 * q);
    if constexpr (VPL < 4) leads = (src.u8(1 + code_byte<VPL>(lane)) >> code_shift<VPL>(lane)) & ((1u << (2 * VPL)) - 1u);
    uint32_t m = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const int L = (leads >> (2 * i)) & 3;
        m += req > L ? req - L : 0;
    }
    const uint32_t incl = warp_incl_scan(m);
    if (1u + NCODE + __shfl_sync(0xffffffffu, incl, 31) != z) return false;
    uint32_t run[NW];
    src.template run<NW>(1 + NCODE + incl - m, run);
    U own[VPL], cmk[VPL];
    U M = ~U(0), D = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const int L = (leads >> (2 * i)) & 3;
        const int mi = req > L ? req - L : 0;
        U bytes;
        if (W == 4) {
            bytes = run[0] & ~__funnelshift_lc(0u, 0xFFFFFFFFu, 8 * mi);
            run_drop4<NW>(run, mi);
        } else {
            bytes = ((U)run[0] | ((U)run[1] << 16 << 16)) & (mi >= 8 ? ~U(0) : ((U(1) << (8 * mi)) - U(1)));
            run_drop4<NW>(run, mi < 4 ? mi : 4);
            run_drop4<NW>(run, mi > 4 ? mi - 4 : 0);
        }
        own[i] = bytes << (8 * (W - req));
        const int copy = L < req ? L : req;
        cmk[i] = ~(~U(0) >> (8 * copy));
        M &= cmk[i];
        D = (D & cmk[i]) | own[i];
    }
    U cM = M, cD = D;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        const U pM = __shfl_up_sync(0xffffffffu, cM, o);
        const U pD = __shfl_up_sync(0xffffffffu, cD, o);
        if (lane >= o) { cD = (pD & cM) | cD; cM = pM & cM; }
    }
    U prev = __shfl_up_sync(0xffffffffu, cD, 1);
    if (lane == 0) prev = 0;
#pragma unroll
    for (int i = 0; i < VPL; i++) {
        const U w = (prev & cmk[i]) | own[i];
        prev = w;
        const U vb = w << s;
        out[i] = raw ? TR::from(vb) : TR::add(TR::from(vb), mu);
    }
    return true;
}

// store of decompressed output (streaming: evict-first)
template <typename V>
__device__ inline void st_out(V* p, V v) {
#if SZX_STCS
    __stcs(p, v);
#else
    *p = v;
#endif
}
// 16-byte store of decompressed output
__device__ inline void st_out16(uint4* p, uint4 v) {
#if SZX_STCS
    __stcs(p, v);
#else
    *p = v;
#endif
}

template <typename T, int VPL>
struct DecWCfg {
#ifndef SZX_DSLOT
#define SZX_DSLOT 3072
#endif
    static constexpr int NT = 256, NWARP = NT / 32;
    static constexpr int SLOT = SZX_DSLOT;          // tile payload bytes staged in shared memory
    static constexpr int SLOT_ALLOC = SLOT + 64;    // + over-read pad of the last block's run loads
#ifndef SZX_FILLW
#define SZX_FILLW 2
#endif
#ifndef SZX_SWITCH
#define SZX_SWITCH 2
#endif
    static constexpr int FILLW = SZX_FILLW;         // fill warps per CTA (the rest decode)
#ifndef SZX_TSFL16
#define SZX_TSFL16 1   // thread-serial decoder: transpose 16 values per flush (64-byte block segments)
#endif
#ifndef SZX_TSFL
#define SZX_TSFL 16    // values per transpose flush (32: 4 KB buffer, whole-line stores; needs a larger region)
#endif
#ifndef SZX_TSCLAMP
#define SZX_TSCLAMP 1  // thread-serial decoder: payload reads clamped to the warp's region (no over-read pad)
#endif
#ifndef SZX_TSASM
#define SZX_TSASM 1  // thread-serial window slide as one PTX block
#endif
#ifndef SZX_TSUNC
#define SZX_TSUNC 0  // thread-serial window: unpredicated look-ahead load (measured slower)
#endif
#ifndef SZX_TSPF
#define SZX_TSPF 0   // thread-serial tiles: bulk L2 prefetch of the next tile's payload
#endif
#ifndef SZX_DREGION
#define SZX_DREGION 9216
#endif
    // per-warp shared region: the two staging slots of the segment decoder, or
    // (thread-serial tiles) a 1 KB transpose buffer + one staging area + over-read pad
    static constexpr int REGION = SZX_DREGION > 2 * SLOT_ALLOC ? SZX_DREGION : 2 * SLOT_ALLOC;
    static constexpr int TS_TB = SZX_TSFL == 32 ? 4096 : SZX_TSFL16 ? 2048 : 1024;  // transpose buffer: 32 blocks x FL values
    static constexpr int TS_PAD = SZX_TSCLAMP ? 16 : 576;   // reads clamped to the region, or > 12 + 128 x 4
                                                            // bytes a corrupt lane may over-read
    static constexpr int TS_STAGE = REGION - TS_TB - TS_PAD;
    static constexpr int SMEM = NWARP * REGION;
    static_assert(SMEM >= kIndexChunk * 32 * 2, "index-phase scratch aliases the slots");
};

// Diagnostic timing builds only (-DSZX_TIMELINE=1, scripts/timeline.py): per
// warp of k_decode_w, %globaltimer at kernel entry, index ready, fill done,
// nonconstant tiles done.
#if SZX_TIMELINE
constexpr int kTlCtas = 2048;
__device__ uint64_t g_tl[kTlCtas * 8 * 4];
#define SZX_TL(k)                                                                                 \
    do {                                                                                          \
        if ((threadIdx.x & 31) == 0 && blockIdx.x < kTlCtas) {                                    \
            uint64_t t_;                                                                          \
            asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t_) : : "memory");                   \
            g_tl[((uint64_t)blockIdx.x * 8 + (threadIdx.x >> 5)) * 4 + (k)] = t_;                 \
        }                                                                                         \
    } while (0)
#else
#define SZX_TL(k) \
    do {          \
    } while (0)
#endif


// ---- thread-serial tile decoder (float32, b = 128): lane j decodes block j
// of a 32-block tile alone, Fig. 10's five steps value after value
// -- no cross-lane scans: the lead-byte chain is the lane's own
// `prev`, the mid-bytes come from a 3-word window sliding over the block's
// staged payload.  Every 8 values the warp transposes its 32 x 8 values
// through shared memory and stores them as 32-byte block segments.
// a: shared address of the lane's payload [R][32 code bytes][mid-bytes];
// tb: 1 KB transpose buffer; yt: the tile's first output value; word: the
// tile's nonconstant bitmap (lanes of constant blocks run on dummy input and
// store nothing).  Returns false (this lane) on a size mismatch.
template <int... Is, typename F>
__device__ __forceinline__ void unroll_i_impl(F&& f, std::integer_sequence<int, Is...>) { (f(std::integral_constant<int, Is>{}), ...); }
template <int N, typename F>
__device__ __forceinline__ void unroll_i(F&& f) { unroll_i_impl(f, std::make_integer_sequence<int, N>{}); }

template <bool RAWOK>
__device__ __forceinline__ bool ts_decode_f32(uint32_t a, uint32_t R, uint32_t zz, float mu, uint32_t tb,
                                              float* __restrict__ yt, uint32_t word, uint32_t lastw) {
    // SZX_TSCLAMP: every payload read is clamped to lastw (the region's last
    // word), so a corrupt lane cannot leave its warp's region without a pad
    auto ldc = [&](uint32_t ad) -> uint32_t { return lds_u32(SZX_TSCLAMP ? umin(ad, lastw) : ad); };
    const int lane = threadIdx.x & 31;
    const bool raw = RAWOK && R >= 32u;
    const uint32_t s = raw ? 0u : ((8u - (R & 7u)) & 7u);
    const uint32_t r8 = raw ? 32u : R + s;              // kept bits, whole bytes: 16, 24 or 32
    const uint32_t pdrop = launder(1u << (32u - r8));   // (shifts as IMADs on the FMA pipe)
    const uint32_t ps = launder(1u << s);
    const uint32_t fix = r8 == 16u ? 0x55555555u : 0u;  // req = 2: code 3 copies 2 bytes
    const uint32_t mb = a + 33u, wp = mb & ~3u, pos0 = 8u * (mb & 3u);
    // window (lo, hi, nx) = words k, k+1, k+2 of the run from wp; pos = absolute
    // bit position from wp (lo holds bits [32 k, 32 k + 32)), lim = 32 (k + 1)
    uint32_t lo = ldc(wp), hi = ldc(wp + 4), nx = ldc(wp + 8);
    uint32_t pos = pos0, lim = 32u, prev = 0;
    const uint32_t wp8 = wp + 8u;
    const uint32_t sw = ((uint32_t)lane >> 2) & 1u;     // transpose swizzle (bank-conflict free)
    // the lead codes: group g's 4 code bytes start at a + 1 + 4 g; the aligned
    // words cw0 (this group's first) and cw1 (next) are loaded a group ahead
    const uint32_t cb0 = (a + 1u) & ~3u, csh = 8u * (a + 1u);
    uint32_t cw0 = ldc(cb0), cw1 = ldc(cb0 + 4u);
    // one value (index II of its 16-value code group, codes cw): Fig. 10 steps 2-5
    auto value = [&](auto IIc, uint32_t cw) -> float {
        constexpr int II = decltype(IIc)::value;
            // step 2: c8 = 8 x bytes copied from the previous value; step 3: m8 = 8 x mid-bytes
            const uint32_t c8 = II == 0 ? (cw << 3) & 24u : II == 1 ? (cw << 1) & 24u : (cw >> (2 * II - 3)) & 24u;
            const uint32_t nm = 0xFFFFFFFFu >> c8;
            const uint32_t m8 = r8 - c8;
            const uint32_t mid = __funnelshift_r(lo, hi, pos);
            const uint32_t w = bitsel(prev, mid * pdrop, nm);  // steps 2-4
            prev = w;
            const float ov = raw ? __uint_as_float(w) : __fadd_rn(__uint_as_float(w * ps), mu);  // step 5
            pos += m8;
#if SZX_TSASM
            // slide one word (m8 <= 32: at most one per value), in one PTX
            // block so the predicated load lands in nx itself (no move of a
            // just-loaded register)
            asm volatile(
                "{\n\t.reg .pred q;\n\t.reg .u32 ad;\n\t"
                "setp.ge.u32 q, %4, %3;\n\t"
                "@q add.u32 %3, %3, 32;\n\t"
                "@q mov.b32 %0, %1;\n\t"
                "@q mov.b32 %1, %2;\n\t"
                "shr.u32 ad, %3, 3;\n\t"
                "add.u32 ad, ad, %5;\n\t"
#if SZX_TSCLAMP
                "min.u32 ad, ad, %6;\n\t"
#endif
                "@q ld.shared.u32 %2, [ad];\n\t}"
                : "+r"(lo), "+r"(hi), "+r"(nx), "+r"(lim)
                : "r"(pos), "r"(wp8 - 4u), "r"(lastw)
                : "memory");
#elif SZX_TSUNC
            // slide one word (m8 <= 32: at most one per value); nx is re-read
            // every value (unpredicated: no move of a just-loaded register)
            const bool sl = pos >= lim;
            lim += sl ? 32u : 0u;
            lo = sl ? hi : lo;
            hi = sl ? nx : hi;
            nx = lds_u32(wp8 + (lim >> 3) - 4u);
#else
            if (pos >= lim) {  // slide one word (m8 <= 32: at most one per value)
                lim += 32u;
                lo = hi;
                hi = nx;
                nx = lds_u32(wp8 + (lim >> 3) - 4u);  // word k + 2 of the new window
            }
#endif
        return ov;
    };
#if SZX_TSFL == 32
    // 32 values per flush: two code groups, then 32 blocks x 32 values through 4 KB
    // (lane j's chunk c at row j, slot c ^ (j & 7)), stored as 4 blocks x 128 bytes
    // (whole lines) per store instruction
#pragma unroll 1
    for (int f = 0; f < 4; f++) {
        float o[32];
        unroll_i<2>([&](auto Gc) {
            constexpr int gg = decltype(Gc)::value;
            uint32_t cw = __funnelshift_r(cw0, cw1, csh);
            cw0 = cw1;
            cw1 = ldc(cb0 + 8u + 4u * (uint32_t)(2 * f + gg));
            cw ^= cw & (cw >> 1) & fix;
            unroll_i<16>([&](auto I) {
                constexpr int i = decltype(I)::value;
                o[16 * gg + i] = value(std::integral_constant<int, i>{}, cw);
            });
        });
        const uint32_t row = tb + 128u * (uint32_t)lane, sz = (uint32_t)lane & 7u;
#pragma unroll
        for (int c = 0; c < 8; c++)
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(row + 16u * ((uint32_t)c ^ sz)),
                         "r"(__float_as_uint(o[4 * c])), "r"(__float_as_uint(o[4 * c + 1])),
                         "r"(__float_as_uint(o[4 * c + 2])), "r"(__float_as_uint(o[4 * c + 3])) : "memory");
        __syncwarp();
#pragma unroll
        for (int k = 0; k < 8; k++) {
            const uint32_t b = ((uint32_t)lane >> 3) + 4u * (uint32_t)k, c = (uint32_t)lane & 7u;
            const uint4 v = lds_u128(tb + 128u * b + 16u * (c ^ (b & 7u)));
            if ((word >> b) & 1u) st_out16(reinterpret_cast<uint4*>(yt + 128u * b + 32u * (uint32_t)f + 4u * c), v);
        }
        __syncwarp();
    }
#else
#pragma unroll 1
    for (int g = 0; g < 8; g++) {
        uint32_t cw = __funnelshift_r(cw0, cw1, csh);  // this group's 16 lead codes
        cw0 = cw1;
        cw1 = ldc(cb0 + 8u + 4u * (uint32_t)g);        // (read past the codes on the last group: inside the payload / pad)
        cw ^= cw & (cw >> 1) & fix;
        constexpr int FL = SZX_TSFL16 ? 16 : 8;   // values per transpose flush (SZX_TSFL == 32: below)
        unroll_i<16 / FL>([&](auto Hc) {
            constexpr int h = decltype(Hc)::value;
            float o[FL];
            unroll_i<FL>([&](auto I) {
                constexpr int i = decltype(I)::value;
                o[i] = value(std::integral_constant<int, FL * h + i>{}, cw);
            });
#if SZX_TSFL16
            // 32 blocks x 16 values through 2 KB: lane j's chunk c at row j, slot c ^ ((j >> 1) & 3);
            // read back as 8 blocks x 64 bytes per store instruction
            {
                const uint32_t row = tb + 64u * (uint32_t)lane, sz = ((uint32_t)lane >> 1) & 3u;
#pragma unroll
                for (int c = 0; c < 4; c++)
                    asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(row + 16u * ((uint32_t)c ^ sz)),
                                 "r"(__float_as_uint(o[4 * c])), "r"(__float_as_uint(o[4 * c + 1])),
                                 "r"(__float_as_uint(o[4 * c + 2])), "r"(__float_as_uint(o[4 * c + 3])) : "memory");
                __syncwarp();
#pragma unroll
                for (int k = 0; k < 4; k++) {
                    const uint32_t b = ((uint32_t)lane >> 2) + 8u * (uint32_t)k, c = (uint32_t)lane & 3u;
                    const uint4 v = lds_u128(tb + 64u * b + 16u * (c ^ ((b >> 1) & 3u)));
                    if ((word >> b) & 1u)
                        st_out16(reinterpret_cast<uint4*>(yt + 128u * b + 16u * (uint32_t)g + 4u * c), v);
                }
                __syncwarp();
            }
#else
            const uint32_t row = tb + 32u * (uint32_t)lane;
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(row + 16u * sw), "r"(__float_as_uint(o[0])),
                         "r"(__float_as_uint(o[1])), "r"(__float_as_uint(o[2])), "r"(__float_as_uint(o[3])) : "memory");
            asm volatile("st.shared.v4.u32 [%0], {%1,%2,%3,%4};" ::"r"(row + 16u * (sw ^ 1u)), "r"(__float_as_uint(o[4])),
                         "r"(__float_as_uint(o[5])), "r"(__float_as_uint(o[6])), "r"(__float_as_uint(o[7])) : "memory");
            __syncwarp();
#pragma unroll
            for (int k = 0; k < 2; k++) {
                const uint32_t b = ((uint32_t)lane >> 1) + 16u * (uint32_t)k, c = (uint32_t)lane & 1u;
                const uint4 v = lds_u128(tb + 32u * b + 16u * (c ^ ((b >> 2) & 1u)));
                if ((word >> b) & 1u)
                    st_out16(reinterpret_cast<uint4*>(yt + 128u * b + 16u * (uint32_t)g + 8u * (uint32_t)h + 4u * c), v);
            }
            __syncwarp();
#endif
        });
    }
#endif
    // the block's mid-bytes end exactly at its zsize
    return pos - pos0 == 8u * (zz - 33u);
}

// Per-tile metadata a warp needs before it can store anything.
template <typename U>
struct TileMeta {
    uint32_t word;      // nonconstant bitmap of the tile's 32 blocks
    uint32_t zl;        // lane r: zsize of the tile's r-th nonconstant block
    uint64_t ncb;       // nonconstant index of the tile's first block
    uint64_t base, end; // payload byte range
    U mul;              // lane j: mu of block j
};

template <typename T, int VPL, bool QUAL = false>
__global__ void __launch_bounds__(256, (sizeof(T) == 8 && VPL == 4) ? SZX_DMINB64 : SZX_DMINB) k_decode_w(DPlan p, const uint8_t* __restrict__ in, T* __restrict__ y) {
    using TR = Traits<T>;
    using U = typename TR::U;
    using C = DecWCfg<T, VPL>;
    constexpr int W = TR::W;
    constexpr int B = 32 * VPL;
    constexpr int TB = kTileBlocks;
    constexpr int MAXZ = 1 + B / 4 + W * B;
    using LY = Lay<T, VPL>;
    using V = typename LY::V;
    constexpr int NV = LY::NQ;        // chunk stores per lane per block
    constexpr int QB = B * W / LY::CB;  // chunks per block
    extern __shared__ __align__(16) uint8_t dsm[];
    __shared__ uint64_t s_w[32];
    __shared__ uint32_t s_sel[8][32];  // per warp: the selected blocks of a segment, in rank order
    QualAcc qa;
    const T* __restrict__ ref = static_cast<const T*>(p.ref);
    pdl_wait();
    pdl_trigger();
    SZX_TL(0);
    const DHdr hd = read_dheader<W>(in, p);
    if (!hd.ok) {  // every CTA sees the same header: all leave
        if (blockIdx.x == 0 && threadIdx.x == 0) set_corrupt(p.err);
        return;
    }
    // index phase (the shared staging slots double as its scratch), then a
    // grid barrier: tiles are decoded by whichever warp grabs them
    // (one CTA per SM at most: fewer arrivals at the two grid-wide prefixes)
    if (blockIdx.x < p.n_icta) index_phase<W>(p, in, hd, reinterpret_cast<uint16_t*>(dsm), s_w);
    // (The fill warps need only the bitmap and mu, but starting them before
    // the barrier measured slower: their traffic stretches the latency-bound
    // index phase -- NYX velocity index 16 -> 22 us, Hurricane decode +8 us.)
    grid_barrier(&p.ctr[2]);
    SZX_TLI(5);
    SZX_TL(1);
    const int lane = threadIdx.x & 31;
    const int wid = threadIdx.x >> 5;
    const uint32_t* bm = reinterpret_cast<const uint32_t*>(in + kHeaderBytes);
    const uint16_t* zs = reinterpret_cast<const uint16_t*>(in + hd.off_zs);
    const U* mus = reinterpret_cast<const U*>(in + p.off_mu);
    const uint8_t* pl = in + hd.off_pl;
    const uintptr_t lim = reinterpret_cast<uintptr_t>(in) + p.in_bytes;
    const uint64_t nW_full = p.n / ((uint64_t)TB * B);
    const uint32_t slot0 = smem_u32(dsm + (threadIdx.x >> 5) * C::REGION);
    // blocks of tile t inside the requested range [kb0, kb1)
    auto rmask = [&](uint64_t t) -> uint32_t {
        uint32_t m = 0xFFFFFFFFu;
        const uint64_t k0 = t * TB;
        if (k0 < p.kb0) m &= 0xFFFFFFFFu << (uint32_t)(p.kb0 - k0);
        if (k0 + TB > p.kb1) m &= (1u << (uint32_t)(p.kb1 - k0)) - 1u;
        return m;
    };
    const uint64_t fill_end = umin64(nW_full, p.nWi);

    // ---- fill warps: the constant blocks of every full tile (Fig. 10 state 0:
    // retrieve with mu).  They need only the bitmap word and the tile's mu
    // values, prefetched one tile ahead, so they stream stores.
    auto fill_loop = [&]() {
        auto grab_f = [&]() -> uint64_t {
            uint32_t v = 0;
            if (lane == 0) v = atomicAdd(&p.ctr[1], 1u);
            return p.t_lo + __shfl_sync(0xffffffffu, v, 0);
        };
        uint64_t t = grab_f();
        uint32_t word = 0;
        U mul = 0;
        if (t < fill_end) { word = bm[t]; mul = mus[t * TB + lane]; }
        while (t < fill_end) {
            const uint64_t tn = grab_f();
            uint32_t wn = 0;
            U mn = 0;
            if (tn < fill_end) { wn = bm[tn]; mn = mus[tn * TB + lane]; }
            V* yq = reinterpret_cast<V*>(y + t * TB * B + lane * VPL);
            {
#pragma unroll 2
            for (uint32_t m = ~word & rmask(t); m; m &= m - 1) {
                const int j = __ffs(m) - 1;
                const U mb = __shfl_sync(0xffffffffu, mul, j);
                T v[VPL];
#pragma unroll
                for (int q = 0; q < VPL; q++) v[q] = TR::from(mb);
#pragma unroll
                for (int q = 0; q < NV; q++) st_out(yq + j * QB + q, reinterpret_cast<const V*>(v)[q]);
                if constexpr (QUAL)
                    qa.add16<T, NV, V>(reinterpret_cast<const V*>(ref + t * TB * B + lane * VPL) + j * QB,
                                       reinterpret_cast<const V(&)[NV]>(v));
            }
            }
            t = tn;
            word = wn;
            mul = mn;
        }
    };

    // Dense streams (p.ts): every warp decodes first, then fills the few
    // constant blocks; tiles are claimed 32 at a time and skipped with one
    // ballot when they hold no constant block.
    auto fill_ts = [&]() {
        for (;;) {
            uint32_t c = 0;
            if (lane == 0) c = atomicAdd(&p.ctr[1], 1u);
            const uint64_t t0 = p.t_lo + 32ull * __shfl_sync(0xffffffffu, c, 0);
            if (t0 >= fill_end) break;
            const uint64_t tl = t0 + lane;
            const uint32_t cm = tl < fill_end ? ~bm[tl] & rmask(tl) : 0u;  // constant blocks of tile tl
            for (uint32_t todo = __ballot_sync(0xffffffffu, cm != 0u); todo; todo &= todo - 1) {
                const int jt = __ffs(todo) - 1;
                const uint64_t t = t0 + jt;
                const uint32_t m = __shfl_sync(0xffffffffu, cm, jt);
                const U mul = mus[t * TB + lane];
                V* yq = reinterpret_cast<V*>(y + t * TB * B + lane * VPL);
                for (uint32_t mm = m; mm; mm &= mm - 1) {
                    const int j = __ffs(mm) - 1;
                    const U mb = __shfl_sync(0xffffffffu, mul, j);
                    T v[VPL];
#pragma unroll
                    for (int q = 0; q < VPL; q++) v[q] = TR::from(mb);
#pragma unroll
                    for (int q = 0; q < NV; q++) st_out(yq + j * QB + q, reinterpret_cast<const V*>(v)[q]);
                }
            }
        }
    };
    auto load_meta = [&](uint64_t t, TileMeta<U>& m) {
        uint32_t word = bm[t];
        if (t == p.nW - 1 && (p.nB & 31)) word &= (1u << (p.nB & 31)) - 1u;
        m.word = word;
        m.ncb = p.ncpre[t];
        m.base = p.tbase[t];
        m.end = p.tbase[t + 1];
        const uint64_t k0 = t * TB;
        m.mul = k0 + lane < p.nB ? mus[k0 + lane] : U(0);
    };
    auto load_zl = [&](TileMeta<U>& m) {
        const uint32_t cnt = __popc(m.word);
        m.zl = ((uint32_t)lane < cnt && m.ncb + cnt <= hd.nnc) ? zs[m.ncb + lane] : 0u;
    };
    // A tile's payload is decoded in segments of consecutive nonconstant blocks
    // whose bytes fit one staging slot (a block is at most MAXZ < SLOT bytes):
    // segment i+1 (of this tile or the next one) is staged with cp.async while
    // segment i is decoded, so dense tiles never read payload bytes from
    // global memory inside the decoder.
    struct SegT {
        uint32_t r0, r1;   // ranks [r0, r1) among the tile's nonconstant blocks
        uint32_t off0;     // payload offset of rank r0 within the tile
    };
    // per-lane tile facts after validation
    struct TileZ {
        uint32_t zl, zincl, cnt;
        bool ok;
    };
    auto tile_z = [&](const TileMeta<U>& m) -> TileZ {
        TileZ r;
        r.cnt = __popc(m.word);
        r.zl = m.zl;
        bool ok = m.end >= m.base && m.end <= hd.payload_bytes && m.ncb + r.cnt <= hd.nnc;
        const bool zok = (uint32_t)lane >= r.cnt || (r.zl >= 2 && r.zl <= (uint32_t)MAXZ);
        r.zincl = warp_incl_scan(r.zl);
        r.ok = ok && __all_sync(0xffffffffu, zok) && __shfl_sync(0xffffffffu, r.zincl, 31) == m.end - m.base;
        return r;
    };
    // the segment starting at rank r0: as many blocks of ranks < rmax as fit SLOT - 16 bytes
    auto seg_from = [&](const TileZ& z, uint32_t r0, uint32_t rmax) -> SegT {
        SegT sg;
        sg.r0 = r0;
        sg.off0 = r0 ? __shfl_sync(0xffffffffu, z.zincl, r0 - 1) : 0u;
        const bool fits = (uint32_t)lane >= r0 && (uint32_t)lane < rmax && z.zincl - sg.off0 <= (uint32_t)(C::SLOT - 16);
        sg.r1 = r0 + __popc(__ballot_sync(0xffffffffu, fits));
        if (sg.r1 == r0 && r0 < rmax) sg.r1 = r0 + 1;  // (corrupt sizes: validated separately)
        return sg;
    };
    // cp.async the segment's bytes into slot `sl`
    auto stage_seg = [&](const TileMeta<U>& m, const TileZ& z, const SegT& sg, int sl) {
        if (!z.ok) return;
        const uint32_t off1 = __shfl_sync(0xffffffffu, z.zincl, sg.r1 - 1);
        const uintptr_t g0 = reinterpret_cast<uintptr_t>(pl + m.base + sg.off0);
        const uintptr_t gA = g0 & ~uintptr_t(15);
        uintptr_t gE = (reinterpret_cast<uintptr_t>(pl + m.base + off1) + 15) & ~uintptr_t(15);
        if (gE > gA + C::SLOT) gE = gA + C::SLOT;
        const uint32_t sa = slot0 + sl * C::SLOT_ALLOC;
        for (uintptr_t a = gA + 16 * lane; a < gE; a += 16 * 32) {
            const uintptr_t rem = lim - a;
            cp_async16_zfill(sa + (uint32_t)(a - gA), reinterpret_cast<const void*>(a), rem < 16 ? (uint32_t)rem : 16u);
        }
    };
    // dynamic assignment over the list of tiles holding nonconstant blocks
    // (their cost varies far more than the fill's); a work item is one of the
    // `split` equal parts of such a tile (small arrays: more warps in flight)
    const uint32_t split = p.split;
    uint32_t n_items = 0;  // set once the index is complete
    auto grab = [&](uint32_t& part) -> uint64_t {
        uint32_t v = 0xFFFFFFFFu, pt = 0;
        if (lane == 0) {
            const uint32_t i = atomicAdd(&p.ctr[4], 1u);
            if (i < n_items) {
                v = p.nctile[i / split];
                pt = i % split;
            }
        }
        v = __shfl_sync(0xffffffffu, v, 0);
        part = __shfl_sync(0xffffffffu, pt, 0);
        return v == 0xFFFFFFFFu ? p.nW : (uint64_t)v;
    };
    // ranks [ra, rb) of the tile's nonconstant blocks that lie in part `part`
    auto part_ranks = [&](uint32_t word, uint32_t part, uint32_t& ra, uint32_t& rb) {
        const uint32_t lo = part * (32u / split), hi = lo + 32u / split;
        ra = __popc(word & ((1u << lo) - 1u));
        rb = hi >= 32u ? __popc(word) : __popc(word & ((1u << hi) - 1u));
    };
    // decode the blocks of ranks [r0, r1) of a full tile from the staged slot
    auto decode_seg = [&](uint64_t t, const TileMeta<U>& m, const TileZ& z, const SegT& sg, int sl) {
        const uint32_t sbase = slot0 + sl * C::SLOT_ALLOC +
                               (uint32_t)(reinterpret_cast<uintptr_t>(pl + m.base + sg.off0) & 15) - sg.off0;
        V* yq = reinterpret_cast<V*>(y + t * TB * B + lane * VPL);
        const uint32_t rm = rmask(t);
        // blocks whose rank lies in [r0, r1), restricted to the requested range;
        // lane j holds block j's payload offset and size (one shuffle each per segment)
        const uint32_t rank = __popc(m.word & ((1u << lane) - 1u));
        const bool insg = ((m.word >> lane) & 1u) && rank >= sg.r0 && rank < sg.r1;
        const uint32_t sel = __ballot_sync(0xffffffffu, insg) & rm;
        const uint32_t offl = __shfl_sync(0xffffffffu, z.zincl - z.zl, rank);
        const uint32_t zzl = __shfl_sync(0xffffffffu, z.zl, rank);
        if constexpr (sizeof(T) == 4 && VPL == 4 && SZX_DQUARTER) {
            // four blocks per iteration, a quarter-warp each (16 values per lane).
            // Lane r of s_sel holds the index of the r-th selected block.
            const int q = lane >> 3, ql = lane & 7;
            const uint32_t wq = threadIdx.x >> 5;
            if ((sel >> lane) & 1u) s_sel[wq][__popc(sel & ((1u << lane) - 1u))] = (uint32_t)lane;
            __syncwarp();
            const uint32_t nsel = __popc(sel);
            float* yb = reinterpret_cast<float*>(y) + t * TB * B + ql * 16;
#pragma unroll 1
            for (uint32_t r0 = 0; r0 < nsel; r0 += 4) {
                const bool act = r0 + q < nsel;
                const int jq = (int)s_sel[wq][act ? r0 + q : r0];
                const uint32_t off = __shfl_sync(0xffffffffu, offl, jq);
                const uint32_t zz = __shfl_sync(0xffffffffu, zzl, jq);
                const float mu = __uint_as_float(__shfl_sync(0xffffffffu, (uint32_t)m.mul, jq));
                const uint32_t aq = sbase + off;
                const uint32_t R = lds_u8(aq);
                if (__all_sync(0xffffffffu, R >= 9u && R < 32u)) {
                    float v[16];
                    const bool ok = decode_quarter_f32x16(aq, R, zz, mu, v);
                    if (act) {
                        if (!ok) {
                            if (ql == 0) set_corrupt(p.err);
                        } else {
                            uint4* qo = reinterpret_cast<uint4*>(yb + jq * B);
#pragma unroll
                            for (int c = 0; c < 4; c++) st_out16(qo + c, reinterpret_cast<const uint4*>(v)[c]);
                            if constexpr (QUAL) {
                                const uint4* rq = reinterpret_cast<const uint4*>(ref + t * TB * B + jq * B + ql * 16);
                                qa.add16<T, 4>(rq, reinterpret_cast<const uint4(&)[4]>(v));
                            }
                        }
                    }
                } else {
                    // a raw (R = 32) or malformed block among the four: whole-warp generic decoder
                    const uint32_t nb = nsel - r0 < 4u ? nsel - r0 : 4u;
                    for (uint32_t k = 0; k < nb; k++) {
                        const int j = (int)s_sel[wq][r0 + k];
                        const uint32_t offj = __shfl_sync(0xffffffffu, offl, j);
                        const uint32_t zj = __shfl_sync(0xffffffffu, zzl, j);
                        const T muj = TR::from(__shfl_sync(0xffffffffu, m.mul, j));
                        T v[VPL];
                        if (!decode_full_g<T, VPL>(SrcS{sbase + offj}, zj, muj, v)) {
                            if (lane == 0) set_corrupt(p.err);
                            continue;
                        }
#pragma unroll
                        for (int qq = 0; qq < NV; qq++) st_out(yq + j * QB + qq, reinterpret_cast<const V*>(v)[qq]);
                        if constexpr (QUAL)
                            qa.add16<T, NV, V>(reinterpret_cast<const V*>(ref + t * TB * B + lane * VPL) + j * QB,
                                               reinterpret_cast<const V(&)[NV]>(v));
                    }
                }
            }
            __syncwarp();  // s_sel is rewritten by the next segment
        } else if constexpr (sizeof(T) == 4 && VPL == 4) {
            // two blocks per iteration, a half-warp each (the second half idles
            // on the last block of an odd count)
            const int h = lane >> 4, hl = lane & 15;
            float* yb = reinterpret_cast<float*>(y) + t * TB * B + hl * 8;
#pragma unroll 1
            for (uint32_t bits = sel; bits;) {
                const int j0 = __ffs(bits) - 1;
                bits &= bits - 1;
                const bool two = bits != 0;
                const int j1 = two ? __ffs(bits) - 1 : j0;
                bits &= bits - 1;
                const int jh = h ? j1 : j0;
                const uint32_t off = __shfl_sync(0xffffffffu, offl, jh);
                const uint32_t zz = __shfl_sync(0xffffffffu, zzl, jh);
                const float mu = __uint_as_float(__shfl_sync(0xffffffffu, (uint32_t)m.mul, jh));
                float v[8];
#if SZX_DNR
                const uint32_t Rh = lds_u8(sbase + off);
                const bool ok = __all_sync(0xffffffffu, Rh >= 9u && Rh < 32u)
                                    ? decode_half_f32x8_nr(sbase + off, Rh, zz, mu, v)
                                    : decode_half_f32x8(sbase + off, zz, mu, v);
#else
                const bool ok = decode_half_f32x8(sbase + off, zz, mu, v);
#endif
                if (h == 0 || two) {
                    if (!ok) {
                        if (hl == 0) set_corrupt(p.err);
                    } else {
                        uint4* q = reinterpret_cast<uint4*>(yb + jh * B);
                        st_out16(q, reinterpret_cast<const uint4*>(v)[0]);
                        st_out16(q + 1, reinterpret_cast<const uint4*>(v)[1]);
                        if constexpr (QUAL) {
                            const uint4* rq = reinterpret_cast<const uint4*>(ref + t * TB * B + jh * B + hl * 8);
                            qa.add16<T, 2>(rq, reinterpret_cast<const uint4(&)[2]>(v));
                        }
                    }
                }
            }
        } else if constexpr (sizeof(T) == 8 && VPL == 4 && SZX_DF64HALF) {
            // two float64 blocks per iteration, a half-warp each (8 doubles per lane)
            const int h = lane >> 4, hl = lane & 15;
            double* yb = reinterpret_cast<double*>(y) + t * TB * B + hl * 8;
#pragma unroll 1
            for (uint32_t bits = sel; bits;) {
                const int j0 = __ffs(bits) - 1;
                bits &= bits - 1;
                const bool two = bits != 0;
                const int j1 = two ? __ffs(bits) - 1 : j0;
                bits &= bits - 1;
                const int jh = h ? j1 : j0;
                const uint32_t off = __shfl_sync(0xffffffffu, offl, jh);
                const uint32_t zz = __shfl_sync(0xffffffffu, zzl, jh);
                const double mu = TR::from(__shfl_sync(0xffffffffu, m.mul, jh));
                const uint32_t Rh = lds_u8(sbase + off);
                if (__all_sync(0xffffffffu, Rh >= 12u && Rh < 64u)) {
                    double v[8];
                    const bool ok = decode_half_f64x8_nr(sbase + off, Rh, zz, mu, v);
                    if (h == 0 || two) {
                        if (!ok) {
                            if (hl == 0) set_corrupt(p.err);
                        } else {
                            uint4* qo = reinterpret_cast<uint4*>(yb + jh * B);
#pragma unroll
                            for (int c = 0; c < 4; c++) st_out16(qo + c, reinterpret_cast<const uint4*>(v)[c]);
                            if constexpr (QUAL) {
                                const uint4* rq = reinterpret_cast<const uint4*>(ref + t * TB * B + jh * B + hl * 8);
                                qa.add16<T, 4>(rq, reinterpret_cast<const uint4(&)[4]>(v));
                            }
                        }
                    }
                } else {
                    // a raw (R = 64) or malformed block in the pair: whole-warp generic decoder
                    for (int k2 = 0; k2 < (two ? 2 : 1); k2++) {
                        const int j = k2 ? j1 : j0;
                        const uint32_t offj = __shfl_sync(0xffffffffu, offl, j);
                        const uint32_t zj = __shfl_sync(0xffffffffu, zzl, j);
                        const T muj = TR::from(__shfl_sync(0xffffffffu, m.mul, j));
                        T v[VPL];
                        if (!decode_full_g<T, VPL>(SrcS{sbase + offj}, zj, muj, v)) {
                            if (lane == 0) set_corrupt(p.err);
                            continue;
                        }
#pragma unroll
                        for (int qq = 0; qq < NV; qq++) st_out(yq + j * QB + qq, reinterpret_cast<const V*>(v)[qq]);
                        if constexpr (QUAL)
                            qa.add16<T, NV, V>(reinterpret_cast<const V*>(ref + t * TB * B + lane * VPL) + j * QB,
                                               reinterpret_cast<const V(&)[NV]>(v));
                    }
                }
            }
        } else {
#pragma unroll 1
            for (uint32_t bits = sel; bits; bits &= bits - 1) {
                const int j = __ffs(bits) - 1;
                const uint32_t off = __shfl_sync(0xffffffffu, offl, j);
                const uint32_t zz = __shfl_sync(0xffffffffu, zzl, j);
                const T mu = TR::from(__shfl_sync(0xffffffffu, m.mul, j));
                T v[VPL];
                if (!decode_full_g<T, VPL>(SrcS{sbase + off}, zz, mu, v)) {
                    if (lane == 0) set_corrupt(p.err);
                    continue;
                }
#pragma unroll
                for (int q = 0; q < NV; q++) st_out(yq + j * QB + q, reinterpret_cast<const V*>(v)[q]);
                if constexpr (QUAL)
                    qa.add16<T, NV, V>(reinterpret_cast<const V*>(ref + t * TB * B + lane * VPL) + j * QB,
                                       reinterpret_cast<const V(&)[NV]>(v));
            }
        }
    };
    // the partial last tile: generic decoder, straight from global memory
    auto decode_partial = [&](uint64_t t, const TileMeta<U>& m, const TileZ& z) {
        const uint64_t k0 = t * TB;
        const uint32_t rm = rmask(t);
        const uint8_t* gb = pl + m.base;
        for (int j = 0; j < TB; j++) {
            const uint64_t k = k0 + j;
            if (k >= p.nB) break;
            if (!((rm >> j) & 1u)) continue;
            const int len = (int)umin64(B, p.n - k * B);
            const T mu = TR::from(__shfl_sync(0xffffffffu, m.mul, j));
            T v[VPL];
            if (!((m.word >> j) & 1u)) {
#pragma unroll
                for (int q = 0; q < VPL; q++) v[q] = mu;
            } else {
                const uint32_t r = __popc(m.word & ((1u << j) - 1u));
                const uint32_t off = __shfl_sync(0xffffffffu, z.zincl - z.zl, r);
                const uint32_t zz = __shfl_sync(0xffffffffu, z.zl, r);
                if (!decode_block_g<T, VPL>(SrcG{gb + off, lim}, zz, len, mu, v)) {
                    if (lane == 0) set_corrupt(p.err);
                    continue;
                }
            }
            store_lane<T, VPL>(y, p.n, k, lane, v);
            if constexpr (QUAL) {
                const uint64_t first = k * B + (uint64_t)lane * VPL;
#pragma unroll
                for (int i = 0; i < VPL; i++)
                    if (first + i < p.n) qa.add<T>(ref[first + i], v[i]);
            }
        }
    };


    // Dense float32 b = 128 streams (p.ts): tiles with >= 24 nonconstant blocks
    // whose payload fits the staging area go to the thread-serial decoder, the
    // others to the segment decoder (not pipelined here); the whole tile is
    // staged, then decoded -- the warps of the SM hide each other's staging.
    auto ts_loop = [&]() {
        if constexpr (sizeof(T) == 4 && VPL == 4 && !QUAL) {
            // Tickets are tile numbers (dense streams: nearly every tile holds
            // nonconstant blocks; the rare all-constant ones are skipped), and
            // the per-tile global reads are pipelined so that none is waited for
            // in the iteration that issues it: at the top of tile k the ticket of
            // tile k+2 is taken and the zsizes of tile k+1 requested (its
            // metadata arrived during tile k-1), in the middle of tile k (after
            // its staging is issued) the metadata of tile k+2 is requested.
            auto ticket = [&]() -> uint32_t {
                uint32_t v = 0;
                if (lane == 0) v = atomicAdd(&p.ctr[4], 1u);
                return v;
            };
            auto tile_of = [&](uint32_t raw) -> uint64_t {
                const uint64_t v = p.t_lo + __shfl_sync(0xffffffffu, raw, 0);
                return v < p.nWi ? v : p.nW;
            };
            const uint32_t r0 = ticket(), r1 = ticket();
            uint64_t t = tile_of(r0);
            uint64_t tn = tile_of(r1);
            TileMeta<U> cur, nx, n2;
            if (t < p.nW) {
                load_meta(t, cur);
                load_zl(cur);
            }
            if (tn < p.nW) load_meta(tn, nx);
            const uint32_t region = slot0, tb = region, sa = region + C::TS_TB;
            while (t < p.nW) {
                const uint32_t iraw = ticket();  // tile k+2 (resolved in the middle of this tile)
                if (tn < p.nW) load_zl(nx);
                const TileZ cz = tile_z(cur);
                const uint64_t bytes = cur.end - cur.base;
                uint64_t tnn = p.nW;
                bool asked = false;
                auto ask_next = [&]() {  // the metadata of tile k+2
                    tnn = tile_of(iraw);
                    if (tnn < p.nW) load_meta(tnn, n2);
                    asked = true;
                };
                if (t < nW_full && cur.word == 0u) {
                    // all-constant tile (the fill writes it)
                } else if (!cz.ok) {
                    if (lane == 0) set_corrupt(p.err);
                } else if (t < nW_full && cz.cnt >= 24u && bytes + 15u <= (uint64_t)C::TS_STAGE) {
                    // stage the tile's payload (16-byte chunks), then decode a block per lane
                    const uintptr_t g0 = reinterpret_cast<uintptr_t>(pl + cur.base);
                    const uintptr_t gA = g0 & ~uintptr_t(15);
                    const uintptr_t gE = (reinterpret_cast<uintptr_t>(pl + cur.end) + 15) & ~uintptr_t(15);
                    for (uintptr_t ga = gA + 16 * lane; ga < gE; ga += 16 * 32) {
                        const uintptr_t rem = lim - ga;
                        cp_async16_zfill(sa + (uint32_t)(ga - gA), reinterpret_cast<const void*>(ga), rem < 16 ? (uint32_t)rem : 16u);
                    }
                    cp_async_commit();
                    ask_next();
                    const uint32_t sbase = sa + (uint32_t)(g0 & 15);
                    const bool has = (cur.word >> lane) & 1u;
                    const uint32_t rank = __popc(cur.word & ((1u << lane) - 1u));
                    const uint32_t offl = __shfl_sync(0xffffffffu, cz.zincl - cz.zl, rank & 31u);
                    const uint32_t zz = __shfl_sync(0xffffffffu, cz.zl, rank & 31u);
                    const uint32_t a = has ? sbase + offl : sbase;
                    cp_async_wait<0>();
                    __syncwarp();
                    const uint32_t R = has ? lds_u8(a) : 9u;
                    const bool bad = R < 9u || R > 32u;
                    float* yt = reinterpret_cast<float*>(y) + t * TB * B;
                    const float mu = __uint_as_float((uint32_t)cur.mul);
                    bool ok;
                    const uint32_t lastw = region + C::REGION - 4u;
                    if (__any_sync(0xffffffffu, R >= 32u)) ok = ts_decode_f32<true>(a, R, has ? zz : 33u, mu, tb, yt, cur.word, lastw);
                    else ok = ts_decode_f32<false>(a, R, has ? zz : 33u, mu, tb, yt, cur.word, lastw);
                    if (has && (bad || !ok)) set_corrupt(p.err);
                } else if (t < nW_full) {
                    // segment decoder, one segment at a time
                    uint32_t r0 = 0;
                    while (r0 < cz.cnt) {
                        const SegT sg = seg_from(cz, r0, cz.cnt);
                        stage_seg(cur, cz, sg, 0);
                        cp_async_commit();
                        cp_async_wait<0>();
                        __syncwarp();
                        decode_seg(t, cur, cz, sg, 0);
                        __syncwarp();
                        r0 = sg.r1;
                    }
                } else {
                    decode_partial(t, cur, cz);
                }
                __syncwarp();  // the region is restaged by the next tile
                if (!asked) ask_next();
                t = tn;
                cur = nx;
                tn = tnn;
                nx = n2;
            }
        }
    };
    auto nc_loop = [&]() {
        n_items = *p.n_nctile * split;
        uint32_t part, pn;
        uint64_t t = grab(part);
        if (t >= p.nW) return;
        TileMeta<U> cur, nx;
        load_meta(t, cur);
        load_zl(cur);
        TileZ cz = tile_z(cur);
        uint32_t ra, rb, na = 0, nb = 0;
        part_ranks(cur.word, part, ra, rb);
        SegT sg = seg_from(cz, ra, rb);
        const bool cfull0 = t < nW_full;
        if (cfull0 && cz.ok && rb > ra) stage_seg(cur, cz, sg, 0);
        cp_async_commit();
        uint64_t tn = grab(pn);
        if (tn < p.nW) load_meta(tn, nx);
        int sl = 0;
        while (t < p.nW) {
            const bool cfull = t < nW_full;
            if (!cz.ok && lane == 0 && part == 0) set_corrupt(p.err);
            // the next work item: the rest of this part, or the next part / tile
            bool next_same = cfull && cz.ok && sg.r1 < rb;
            TileZ nz = cz;
            SegT ns = sg;
            if (next_same) {
                ns = seg_from(cz, sg.r1, rb);
                stage_seg(cur, cz, ns, sl ^ 1);
            } else if (tn < p.nW) {
                load_zl(nx);
                nz = tile_z(nx);
                part_ranks(nx.word, pn, na, nb);
                ns = seg_from(nz, na, nb);
                if (tn < nW_full && nz.ok && nb > na) stage_seg(nx, nz, ns, sl ^ 1);
            }
            cp_async_commit();
            cp_async_wait<1>();
            __syncwarp();
            if (cz.ok) {
                if (cfull) decode_seg(t, cur, cz, sg, sl);
                else if (part == 0) decode_partial(t, cur, cz);  // the partial tile: whole, by part 0
            }
            __syncwarp();  // slot `sl` is refilled by the item after next
            sl ^= 1;
            if (next_same) {
                sg = ns;
            } else {
                t = tn;
                part = pn;
                ra = na;
                rb = nb;
                cur = nx;
                cz = nz;
                sg = ns;
                if (t < p.nW) {
                    tn = grab(pn);
                    if (tn < p.nW) load_meta(tn, nx);
                }
            }
        }
        cp_async_wait<0>();
    };
    // The fill warps join the nonconstant tiles once their queue is empty, so
    // the split adapts to the field's fraction of nonconstant blocks.  (Decode
    // warps joining the fill as well, SZX_SWITCH = 3, measured slower: more
    // concurrent fill streams cut the write rate -- NYX density 107 -> 149 us.)
    if (p.ts) {
        ts_loop();
        SZX_TL(2);
        fill_ts();
    } else if (wid < C::FILLW) {
        fill_loop();
        SZX_TL(2);
        if (SZX_SWITCH & 2) nc_loop();
    } else {
        nc_loop();
        if (SZX_SWITCH & 1) fill_loop();
    }
    SZX_TL(3);
    if constexpr (QUAL) qa.flush(p.qual);
}

}  // namespace szx
