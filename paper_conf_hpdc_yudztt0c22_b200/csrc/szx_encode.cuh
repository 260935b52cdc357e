// szx_encode.cuh -- the fused single-pass encoder for b = 128 (float32 and
// float64, sm_100a): k_encode_fused.
//
// One read of the nonconstant blocks' values, one write of the payload.  A CTA
// of NW = 4 compute warps + 1 extra warp works on tiles of 4 x NW = 16
// consecutive entries of k_classify's compacted nonconstant list (tickets in
// order, the next ticket and its metadata prefetched):
//   (1) each warp stages its 4 blocks with cp.async (16-byte chunks swizzled
//       so the quarter-warp reads are bank-conflict free), the next tile's
//       values while the current one is packed;
//   (2) a quarter-warp (8 lanes x 16 values) encodes a block: v_i = d_i - mu
//       (Alg. 1 l.10), Formula 5's shift folded into the lead-byte count, 2-bit
//       codes min(3, identical leading bytes) against the previous value
//       (Sec. 6.1 steps 1-4; u_{-1} = 0, reading R6), mid-byte
//       counts, z_k = 1 + 32 + sum m_i;
//   (3) every warp scans the tile's 16 z_k; warp 0 writes the zsize entries and
//       publishes the tile's payload bytes in its status word;
//   (4) the quarter packs [R][codes][mid-bytes] into a zeroed shared-memory
//       slot (one of NS = 3) with OR reductions (readings R7/R8);
//   (5) the grid's tile scanner -- the extra warp of CTA 0 -- walks the status
//       words in tile order and writes every tile's exclusive payload offset
//       as soon as it and its predecessors have published (the device-wide
//       exclusive scan of block sizes); tile k is copied out NS - 1
//       tiles later with 16-byte stores realigned to its offset.
// The R2 guard runs where k_classify could not prove it away (whole-warp
// check, DESIGN.md s.3); raw blocks (R = full width) and the partial last block
// take a whole-warp generic path.  Byte-identical to the three-pass encoder
// (b != 128) and the oracle.
#pragma once

#include <type_traits>
#include <utility>

#include "szx_compress.cuh"

namespace szx {

#ifndef SZX_EMINB
#define SZX_EMINB 5   // encoder CTAs per SM (register budget)
#endif
#ifndef SZX_ERED3
#define SZX_ERED3 1
#endif
#ifndef SZX_M8PACK
#define SZX_M8PACK 1  // mid-byte counts packed 4 per register (no spill)
#endif
#ifndef SZX_ENW
#define SZX_ENW 4     // compute warps per encoder CTA (tile = 4 x warps nonconstant blocks)
#endif
#ifndef SZX_ENS
#define SZX_ENS 3     // staging slots per encoder CTA (tiles in flight)
#endif
#ifndef SZX_ENS64
#define SZX_ENS64 2   // the same for float64 (shared memory)
#endif
#ifndef SZX_EMINB64
#define SZX_EMINB64 3 // float64 encoder CTAs per SM (register budget)
#endif

// Diagnostic timing builds only (-DSZX_ETIMELINE=1, scripts/enc_timeline.py):
// %globaltimer per tile at publish, prefix written, retire start / end.
#ifndef SZX_ETIMELINE
#define SZX_ETIMELINE 0
#endif
#if SZX_ETIMELINE
constexpr int kEtlTiles = 1 << 17;
__device__ uint64_t g_etl[kEtlTiles * 4];
__device__ inline uint64_t gtimer() {
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)::"memory");
    return t;
}
#define SZX_ETL(tile, k) \
    do { if ((tile) < (uint64_t)kEtlTiles) g_etl[(uint64_t)(tile) * 4 + (k)] = gtimer(); } while (0)
#else
#define SZX_ETL(tile, k) do { } while (0)
#endif

#ifndef SZX_EXP_NOCOPY
#define SZX_EXP_NOCOPY 0  // timing experiments only (invalid streams): skip the copy-out
#endif
#ifndef SZX_EXP_NOPACK
#define SZX_EXP_NOPACK 0  // timing experiments only (invalid streams): skip the pack
#endif
#ifndef SZX_GUARDSTAT
#define SZX_GUARDSTAT 0  // diagnostic builds: count blocks whose R2 guard runs in the fused encoder
#endif
#if SZX_GUARDSTAT
__device__ unsigned long long g_guardstat[2];
#endif

// 16-byte chunk c (0..31) of a staged block sits at swz16(c): lane ql of a
// quarter reads chunks 4 ql .. 4 ql + 3, and the 8 lanes of one LDS.128 phase
// then hit 8 distinct 16-byte bank groups
__device__ __forceinline__ uint32_t swz16(uint32_t c) { return (c & ~7u) | ((c ^ (c >> 2)) & 7u); }
// the same for CPL chunks per quarter lane (4: float32, 8: float64)
template <int CPL>
__device__ __forceinline__ uint32_t swzc(uint32_t c) { return (c & ~7u) | ((c ^ (c / CPL)) & 7u); }

// Forward scanner of tile sizes (one warp for the whole grid): walks the
// status array in tile order, 512 tiles per round trip, and writes every
// tile's exclusive payload offset to prefix[t] (flag bit 63) as soon as the
// tile and all its predecessors have published their sizes.  Tiles never wait
// on each other; only a tile's copy-out waits for its own prefix.  The last
// step completes the stream header (payload bytes) and the total.
__device__ inline void tile_scanner(const uint64_t* status, uint64_t* prefix, uint64_t ntiles, uint8_t* out,
                                    uint64_t* total, uint64_t off_pl) {
#ifndef SZX_ESK
#define SZX_ESK 8
#endif
    constexpr int K = SZX_ESK;     // tiles per lane per window
    constexpr int WIN = 32 * K;
    const int lane = threadIdx.x & 31;
    auto load = [&](uint64_t b, uint64_t (&v)[K]) {
#pragma unroll
        for (int k = 0; k < K; k++) {
            const uint64_t t = b + (uint64_t)(K * lane + k);
            v[k] = t < ntiles ? ld_relaxed(&status[t]) : 0;
        }
    };
    uint64_t base = 0, run = 0;
    uint32_t ns = 32;
    uint64_t va[K], vb[K];
    load(0, va);
    while (base < ntiles) {
        // the next window is read while this one is scanned (it is re-read if this one is short)
        load(base + WIN, vb);
        int first_bad = K;
#pragma unroll
        for (int k = K - 1; k >= 0; k--)
            if (va[k] == 0) first_bad = k;
        const uint32_t gap = __ballot_sync(0xffffffffu, first_bad < K);
        const int gl = gap ? __ffs(gap) - 1 : 32;
        const int gk = __shfl_sync(0xffffffffu, first_bad, gl & 31);
        const int nready = gl == 32 ? WIN : K * gl + gk;
        if (nready == 0) {  // the next tile has not published: back off and re-read
            __nanosleep(ns);
            ns = ns < 512 ? 2 * ns : ns;
            load(base, va);
            continue;
        }
        ns = 32;
        uint64_t loc = 0, pre[K];
#pragma unroll
        for (int k = 0; k < K; k++) {
            pre[k] = loc;
            loc += K * lane + k < nready ? (va[k] & kValueMask) : 0;
        }
        uint64_t incl = loc;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
            const uint64_t tt = __shfl_up_sync(0xffffffffu, incl, o);
            if (lane >= o) incl += tt;
        }
        const uint64_t lex = run + incl - loc;
#pragma unroll
        for (int k = 0; k < K; k++)
            if (K * lane + k < nready) {
                st_relaxed(&prefix[base + K * lane + k], (1ull << 63) | (lex + pre[k]));
                SZX_ETL(base + K * lane + k, 1);
            }
        run += __shfl_sync(0xffffffffu, incl, 31);
        base += (uint64_t)nready;
        if (nready == WIN) {
#pragma unroll
            for (int k = 0; k < K; k++) va[k] = vb[k];
        } else {
            load(base, va);
        }
    }
    if (lane == 0) {
        reinterpret_cast<uint64_t*>(out)[6] = run;  // header: payload bytes
        *total = off_pl + run;
    }
}

// Per-value mid-byte counts (8 x m, <= 64) of a quarter lane's 16 values, one
// byte each in 4 words (16 separate registers spilled to local memory at 72
// registers per thread, the per-SMSP limit of 5 CTAs x 5 warps)
struct M8 {
#if SZX_M8PACK
    uint32_t w[4];
    template <int I>
    __device__ __forceinline__ void set(uint32_t v) {
        w[I >> 2] = (I & 3) ? (w[I >> 2] | (v << (8 * (I & 3)))) : v;
    }
    template <int I>
    __device__ __forceinline__ uint32_t get() const { return __byte_perm(w[I >> 2], 0u, 0x4440u | (I & 3)); }
#else
    uint32_t w[16];
    template <int I>
    __device__ __forceinline__ void set(uint32_t v) { w[I] = v; }
    template <int I>
    __device__ __forceinline__ uint32_t get() const { return w[I]; }
#endif
};
template <int... Is, typename F>
__device__ __forceinline__ void unroll_impl(F&& f, std::integer_sequence<int, Is...>) { (f(std::integral_constant<int, Is>{}), ...); }
// f(integral_constant<int, i>) for i = 0 .. N-1, in order (compile-time indices)
template <int N, typename F>
__device__ __forceinline__ void unroll(F&& f) { unroll_impl(f, std::make_integer_sequence<int, N>{}); }

// ---- quarter-warp block encoder (full float32 block, 9 <= R < 32)
struct QEnc {
    uint32_t v[16];     // normalised words bits(d_i - mu)
    uint32_t codes;     // 2-bit lead codes of the lane's 16 values, LSB-first
    uint32_t msum;      // mid-bytes of the lane
};

// Formula 5: s = (8 - R % 8) % 8, req = (R + s) / 8.  The lead-byte count of
// the shifted words u = v >> s is min(3, (clz(v_i ^ v_{i-1}) + s) / 8): a
// logical shift adds s identical leading zeros to both words; OR-ing 0xFF << s
// into the XOR caps the count at 3.
__device__ __forceinline__ void quarter_encode_f32(const float (&x)[16], float mu, uint32_t R, QEnc& e,
                                                   M8& m8) {
    const int ql = threadIdx.x & 7;
    const uint32_t s = (8u - (R & 7u)) & 7u;
    const uint32_t req = (R + s) >> 3;
    const uint32_t cap = 0xFFu << s;
#pragma unroll
    for (int i = 0; i < 16; i++) e.v[i] = __float_as_uint(__fsub_rn(x[i], mu));
    uint32_t prev = __shfl_up_sync(0xffffffffu, e.v[15], 1, 8);
    prev = ql == 0 ? 0u : prev;
    uint32_t codes = 0, msum = 0;
    unroll<16>([&](auto I) {
        constexpr int i = decltype(I)::value;
        const uint32_t L = ((uint32_t)__clz((e.v[i] ^ prev) | cap) + s) >> 3;
        prev = e.v[i];
        codes |= L << (2 * i);
        const uint32_t m = req - umin(L, req);
        m8.template set<i>(8u * m);
        msum += m;
    });
    e.codes = codes;
    e.msum = msum;
}

// Pack the quarter's block at shared byte address dst: [R][32 code bytes][mid-bytes];
// mexcl = this lane's exclusive mid-byte offset within the block.
__device__ __forceinline__ void quarter_pack_f32(const QEnc& e, const M8& m8, uint32_t R,
                                                 uint32_t mexcl, uint32_t dst) {
    const int ql = threadIdx.x & 7;
    if (ql == 0) red_or_s(dst & ~3u, R << (8u * (dst & 3u)));
    {   // this lane's 4 code bytes at dst + 1 + 4 ql (two words at most)
        const uint32_t a = dst + 1u + 4u * (uint32_t)ql, sh = 8u * (a & 3u);
        red_or_s(a & ~3u, e.codes << sh);
        red_or_nz((a & ~3u) + 4u, __funnelshift_l(e.codes, 0u, sh));
    }
    const uint32_t rs = 32u - R;     // v >> rs = the R kept bits (u >> drop)
    uint32_t a = dst + 33u + mexcl;
    unroll<8>([&](auto H) {
        constexpr int h = decltype(H)::value;
        const uint32_t n0 = m8.template get<2 * h>(), n1 = m8.template get<2 * h + 1>();
        // the mid-bytes: the low m_i bytes of the kept bits (bytes [W-req, W-L) of u)
        const uint32_t c0 = (e.v[2 * h] >> rs) & ~__funnelshift_lc(0u, 0xFFFFFFFFu, n0);
        const uint32_t c1 = (e.v[2 * h + 1] >> rs) & ~__funnelshift_lc(0u, 0xFFFFFFFFu, n1);
        const uint32_t lo = c0 | __funnelshift_lc(0u, c1, n0);
        const uint32_t hi = __funnelshift_lc(c1, 0u, n0);
        const uint32_t sh = 8u * (a & 3u), wa = a & ~3u;
        red_or_s(wa, lo << sh);
        red_or_s(wa + 4u, __funnelshift_l(lo, hi, sh));
#if SZX_ERED3
        red_or_s(wa + 8u, __funnelshift_l(hi, 0u, sh));  // (unconditional: a predicated ATOMS compiles to a branch)
#else
        red_or_nz(wa + 8u, __funnelshift_l(hi, 0u, sh));
#endif
        a += (n0 + n1) >> 3;
    });
}

// ---- the same for float64 blocks of b = 128 (8 lanes x 16 doubles): the lead
// count only needs the high words (three identical leading bytes are decided
// there; a zero high XOR means >= 4 identical bytes, capped at 3 by the OR)
struct QEnc64 {
    uint64_t v[16];
    uint32_t codes;
    uint32_t msum;
};
__device__ __forceinline__ void quarter_encode_f64(const double (&x)[16], double mu, uint32_t R, QEnc64& e,
                                                   M8& m8) {
    const int ql = threadIdx.x & 7;
    const uint32_t s = (8u - (R & 7u)) & 7u;
    const uint32_t req = (R + s) >> 3;  // 2 .. 8
    const uint32_t cap = 0xFFu << s;
#pragma unroll
    for (int i = 0; i < 16; i++) e.v[i] = (uint64_t)__double_as_longlong(__dsub_rn(x[i], mu));
    uint32_t prevh = __shfl_up_sync(0xffffffffu, (uint32_t)(e.v[15] >> 32), 1, 8);
    prevh = ql == 0 ? 0u : prevh;
    uint32_t codes = 0, msum = 0;
    unroll<16>([&](auto I) {
        constexpr int i = decltype(I)::value;
        const uint32_t h = (uint32_t)(e.v[i] >> 32);
        const uint32_t L = ((uint32_t)__clz((h ^ prevh) | cap) + s) >> 3;
        prevh = h;
        codes |= L << (2 * i);
        const uint32_t m = req - umin(L, req);
        m8.template set<i>(8u * m);  // 0 .. 64
        msum += m;
    });
    e.codes = codes;
    e.msum = msum;
}
__device__ __forceinline__ void quarter_pack_f64(const QEnc64& e, const M8& m8, uint32_t R,
                                                 uint32_t mexcl, uint32_t dst) {
    const int ql = threadIdx.x & 7;
    if (ql == 0) red_or_s(dst & ~3u, R << (8u * (dst & 3u)));
    {
        const uint32_t a = dst + 1u + 4u * (uint32_t)ql, sh = 8u * (a & 3u);
        red_or_s(a & ~3u, e.codes << sh);
        red_or_nz((a & ~3u) + 4u, __funnelshift_l(e.codes, 0u, sh));
    }
    const uint32_t rs = 64u - R;  // v >> rs = the R kept bits
    uint32_t a = dst + 33u + mexcl;
    unroll<16>([&](auto I) {
        constexpr int i = decltype(I)::value;
        const uint32_t n = m8.template get<i>();
        // the low m_i bytes of the kept bits, as (lo, hi) words
        const uint64_t k = e.v[i] >> rs;
        const uint64_t c = n >= 64u ? k : (k & ((1ull << n) - 1ull));
        const uint32_t lo = (uint32_t)c, hi = (uint32_t)(c >> 32);
        const uint32_t sh = 8u * (a & 3u), wa = a & ~3u;
        red_or_s(wa, lo << sh);
        red_or_s(wa + 4u, __funnelshift_l(lo, hi, sh));
        red_or_s(wa + 8u, __funnelshift_l(hi, 0u, sh));
        a += n >> 3;
    });
}

template <int O>
__device__ __forceinline__ uint32_t shfl_up_add8e(uint32_t v) {
    asm volatile(
        "{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
        "shfl.sync.up.b32 t|p, %0, %1, 0x1800, -1;\n\t"
        "@p add.u32 %0, %0, t;\n\t}"
        : "+r"(v)
        : "n"(O));
    return v;
}

// Copy the packed tile [0, T) of the staging area (shared address stg, 16-byte
// aligned, 16 readable bytes before it) to global g0, with 16-byte stores; the
// two boundary chunks are shared with the neighbouring tiles and written word-
// or byte-wise.  The realignment is tile-uniform: staging byte s lands at
// global g0 + s, so output chunk ch (at A + 16 ch, A = g0 & ~15) holds staging
// bytes [16 ch - d, +16), d = g0 & 15.
template <int NT>
__device__ __forceinline__ void copy_out_tile(uint32_t stg, uint8_t* g0, uint32_t T) {
    const uintptr_t a0 = reinterpret_cast<uintptr_t>(g0), A = a0 & ~uintptr_t(15), E = a0 + T;
    const uint32_t d = (uint32_t)(a0 - A);
    const uint32_t nch = (uint32_t)((E - A + 15) >> 4);
    const uint32_t wsh = (16u - d) >> 2, sh = 8u * ((16u - d) & 3u);  // window start (in words) within chunks ch-1, ch
    for (uint32_t ch = threadIdx.x; ch < nch; ch += NT) {
        const uint4 p0 = lds_u128(stg + 16u * ch - 16u), p1 = lds_u128(stg + 16u * ch);
        const uint32_t w8[8] = {p0.x, p0.y, p0.z, p0.w, p1.x, p1.y, p1.z, p1.w};
        uint32_t w[5];
        // w[k] = w8[wsh + k] (wsh in 0..4; the branch is uniform over the tile)
        switch (wsh) {
            case 0: w[0] = w8[0]; w[1] = w8[1]; w[2] = w8[2]; w[3] = w8[3]; w[4] = w8[4]; break;
            case 1: w[0] = w8[1]; w[1] = w8[2]; w[2] = w8[3]; w[3] = w8[4]; w[4] = w8[5]; break;
            case 2: w[0] = w8[2]; w[1] = w8[3]; w[2] = w8[4]; w[3] = w8[5]; w[4] = w8[6]; break;
            case 3: w[0] = w8[3]; w[1] = w8[4]; w[2] = w8[5]; w[3] = w8[6]; w[4] = w8[7]; break;
            default: w[0] = w8[4]; w[1] = w8[5]; w[2] = w8[6]; w[3] = w8[7]; w[4] = 0u; break;
        }
        uint4 v;
        v.x = __funnelshift_r(w[0], w[1], sh);
        v.y = __funnelshift_r(w[1], w[2], sh);
        v.z = __funnelshift_r(w[2], w[3], sh);
        v.w = __funnelshift_r(w[3], w[4], sh);
        const uintptr_t a = A + 16 * (uintptr_t)ch;
        if (a >= a0 && a + 16 <= E) {
            *reinterpret_cast<uint4*>(a) = v;
        } else {
            const uint32_t vw[4] = {v.x, v.y, v.z, v.w};
#pragma unroll
            for (int qq = 0; qq < 4; qq++) {
                const uintptr_t aw = a + 4 * qq;
                if (aw >= a0 && aw + 4 <= E) {
                    *reinterpret_cast<uint32_t*>(aw) = vw[qq];
                } else if (aw + 4 > a0 && aw < E) {
                    for (int c = 0; c < 4; c++)
                        if (aw + c >= a0 && aw + c < E) *reinterpret_cast<uint8_t*>(aw + c) = (uint8_t)(vw[qq] >> (8 * c));
                }
            }
        }
    }
}

template <typename T, int NW, int NS>
struct EncCfg {
    static constexpr int W = (int)sizeof(T);
    static constexpr int NTC = 32 * NW;               // compute threads
    static constexpr int NT = NTC + 32;               // + the scanner warp
    static constexpr int TILE = 4 * NW;               // nonconstant blocks per tile (a quarter-warp each)
    static constexpr int BW = 128 * W;                // bytes per block
    static constexpr int CPB = BW / 16;               // 16-byte chunks per block
    static constexpr int CPL = W;                     // chunks per quarter lane (16 values)
    static constexpr int MAXZ = 1 + 32 + BW;          // raw block payload
    static constexpr int IN = TILE * BW;              // the tile's values
    static constexpr int STG = (TILE * MAXZ + 64 + 15) / 16 * 16;
    static constexpr int SMEM = 2 * IN + NS * (16 + STG); // 2 x input | NS x (16-byte pad | staging slot)
};

__device__ __forceinline__ void bar_compute(int nthreads) {
    asm volatile("bar.sync 1, %0;" ::"r"(nthreads) : "memory");
}

// Software-pipelined fused encoder (float32 and float64, b = 128).  NW compute
// warps work on tile k (ticket, staging, encode, z-scan, publish the tile size,
// pack into staging slot k % NS) and copy tile k out NS - 1 tiles later, once
// the grid's tile scanner (the extra warp of CTA 0) has produced its payload
// offset; the scan latency and the jitter of other tiles' publishes overlap
// with the next tiles' work.  Tiles are handed out in ticket order and publish
// without waiting, so the scanner always advances; the grid is co-resident
// (cooperative launch), so the scanner's CTA runs.
template <typename T, int NW, int NS>
__global__ void __launch_bounds__(32 * NW + 32, sizeof(T) == 4 ? SZX_EMINB : SZX_EMINB64) k_encode_fused(const T* __restrict__ x, Plan p,
                                                                         uint8_t* __restrict__ out) {
    using C = EncCfg<T, NW, NS>;
    using TR = Traits<T>;
    using U = typename TR::U;
    constexpr int B = 128;
    constexpr int W = C::W;
    extern __shared__ __align__(16) uint8_t esm[];
    __shared__ uint32_t s_z[C::TILE];
    __shared__ uint64_t s_cur;
    __shared__ uint64_t s_tile[NS], s_excl[NS];
    __shared__ uint32_t s_T[NS];
    pdl_wait();
    pdl_trigger();
    const uint64_t nnc = *p.nnc;
    const double eb = *p.eb_abs;
    const uint64_t ntiles = (nnc + C::TILE - 1) / C::TILE;
    const uint64_t off_zs = p.off_mu + al16((uint64_t)W * p.nB);
    const uint64_t off_pl = off_zs + al16(2 * nnc);
    const int tid = threadIdx.x, lane = tid & 31, warp = tid >> 5;
    const uint32_t ib = smem_u32(esm);
    auto slot_addr = [&](int sl) -> uint32_t { return ib + 2 * C::IN + 16u + (uint32_t)sl * (16u + C::STG); };

    for (uint32_t c = tid; c < NS * (16 + C::STG) / 16; c += C::NT)  // OR reductions assemble tiles in zeroed staging
        asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(ib + 2 * C::IN + 16u * c), "r"(0u) : "memory");
    __syncthreads();

    if (warp == NW) {
        // the grid's tile scanner runs in the extra warp of CTA 0; the others leave
        if (blockIdx.x == 0 && ntiles) tile_scanner(p.status_e, p.prefix_e, ntiles, out, p.total, off_pl);
        return;
    }

    // ---------------- compute warps
    uint16_t* zsize = reinterpret_cast<uint16_t*>(out + off_zs);
    U* mus = reinterpret_cast<U*>(out + p.off_mu);
    const U* ncmu = reinterpret_cast<const U*>(p.ncmu);
    const uint32_t nBfull = (uint32_t)(p.n / B);       // block ids fit 32 bits (kMaxN / 32)
    const uint32_t nnc32 = (uint32_t)nnc;
    const int q = lane >> 3, ql = lane & 7;
    const int j = warp * 4 + q;  // this quarter's block within the tile
    // copy out tile kk (its offset produced by the scanner)
    // pv: thread 0's early read of the tile's prefix word (issued an iteration
    // earlier so its L2 latency overlaps the encode; re-polled if not yet written)
    auto retire = [&](uint32_t kk, uint64_t pv) {
        const int sl = (int)(kk % NS);
        if (tid == 0) {
            SZX_ETL(s_tile[sl], 2);
            uint32_t ns = 32;
            while (!(pv >> 63)) {
                __nanosleep(ns);
                ns = ns < 256 ? 2 * ns : ns;
                pv = ld_relaxed(&p.prefix_e[s_tile[sl]]);
            }
            s_excl[sl] = pv & ~(1ull << 63);
        }
        bar_compute(C::NTC);
        if (!SZX_EXP_NOCOPY) copy_out_tile<C::NTC>(slot_addr(sl), out + off_pl + s_excl[sl], s_T[sl]);
        if (tid == 0) SZX_ETL(s_tile[sl], 3);
        // (the slot is zeroed when it is reused, NS - 1 tiles later)
    };
    // metadata of this warp's 4 blocks of tile t (lanes 0-3); the values are staged by
    // the warp itself into its part of input buffer b (lane l: chunks (l & 7) + 8 kk of block l >> 3)
    struct Meta { uint32_t mk; U mu; uint32_t rec; };
    auto load_meta = [&](uint32_t t) -> Meta {
        Meta m{0xFFFFFFFFu, U(0), 9u | 0x80u};
        const uint32_t nc0 = t * (uint32_t)C::TILE + 4u * (uint32_t)warp;
        if (t < ntiles && lane < 4 && nc0 + lane < nnc32) {
            m.mk = p.nclist[nc0 + lane];
            m.mu = ncmu[nc0 + lane];
            m.rec = p.ncR[nc0 + lane];
        }
        return m;
    };
    auto stage = [&](const Meta& m, int b) {
        const uint32_t bk = __shfl_sync(0xffffffffu, m.mk, lane >> 3);
        if (bk < nBfull) {
            const uint32_t dst = ib + (uint32_t)b * C::IN + (uint32_t)warp * 4u * C::BW + (uint32_t)q * C::BW;
#pragma unroll
            for (int kk = 0; kk < C::CPB / 8; kk++) {
                const uint32_t c = (uint32_t)(ql + 8 * kk);
                cp_async16(dst + 16u * swzc<C::CPL>(c), x + (uint64_t)bk * B + (16 / W) * c);
            }
        }
        cp_async_commit();
    };
    // the warp-layout values of block kq (lane l: values 4 l .. 4 l + 3) from the staged tile
    auto warp_vals = [&](uint32_t wib, int kq, T (&xw)[4]) {
#pragma unroll
        for (int h = 0; h < 4 * W / 16; h++)
            reinterpret_cast<uint4*>(xw)[h] =
                lds_u128(wib + (uint32_t)kq * C::BW + 16u * swzc<C::CPL>((uint32_t)(lane * (4 * W / 16) + h)));
    };
    if (tid == 0) s_cur = atomicAdd(&p.ctr[3], 1u);
    bar_compute(C::NTC);
    uint32_t cur = (uint32_t)s_cur;
    Meta mc = load_meta(cur);
    if (cur < ntiles) stage(mc, 0);
    uint32_t k = 0;
    for (;; k++) {
        const int slot = (int)(k % NS);
        const uint32_t stg = slot_addr(slot);
        const int buf = (int)(k & 1);
        bar_compute(C::NTC);  // (A) s_cur consumed; the slot's previous tile is copied out
        if (cur >= ntiles) break;
        if (k >= NS) {  // zero what the slot's previous tile used (ordered before the pack by (C))
            const uint32_t To = s_T[slot];
            for (uint32_t c = tid; c < (To + 15u) / 16u + 2u; c += C::NTC)
                asm volatile("st.shared.v4.u32 [%0], {%1,%1,%1,%1};" ::"r"(stg + 16u * c), "r"(0u) : "memory");
        }
        if (tid == 0) s_cur = atomicAdd(&p.ctr[3], 1u);  // the next tile (prefetched below)
        uint64_t pv = 0;  // the prefix of the tile retired at the end of this iteration
        if (tid == 0 && k + 1 >= NS) pv = ld_relaxed(&p.prefix_e[s_tile[(k + 1) % NS]]);
        const uint32_t wib = ib + (uint32_t)buf * C::IN + (uint32_t)warp * 4u * C::BW;  // this warp's 4 staged blocks
        const uint32_t mk = __shfl_sync(0xffffffffu, mc.mk, q);
        const T mu = TR::from(__shfl_sync(0xffffffffu, mc.mu, q));
        const uint32_t rec = __shfl_sync(0xffffffffu, mc.rec, q);
        const bool valid = cur * (uint32_t)C::TILE + 4u * (uint32_t)warp + (uint32_t)q < nnc32;
        uint32_t R = rec & 0x7Fu;
        const bool full = mk < nBfull;
        cp_async_wait<0>();
        __syncwarp();  // the warp's own blocks are staged
        {   // R2 guard where classify could not prove it away: whole warp, one block at a time
            const bool ng = valid && full && !(rec & 0x80u) && R < (uint32_t)TR::kFull;
            uint32_t gm = __ballot_sync(0xffffffffu, ng && ql == 0);
#if SZX_GUARDSTAT
            if (lane == 0) {
                atomicAdd(&g_guardstat[0], (unsigned long long)__popc(gm));
                atomicAdd(&g_guardstat[1], 1ull);
            }
#endif
            while (gm) {
                const int gl = __ffs(gm) - 1;
                gm &= gm - 1;
                T xw[4];
                warp_vals(wib, gl >> 3, xw);
                const T gmu = TR::from(__shfl_sync(0xffffffffu, TR::bits(mu), gl));
                const int gR = (int)__shfl_sync(0xffffffffu, R, gl);
                const int fR = guard_R<T, 4>(xw, 4, gmu, gR, eb);
                if ((lane >> 3) == (gl >> 3)) R = (uint32_t)fR;
            }
        }
        const bool fast = !__any_sync(0xffffffffu, valid && (!full || R >= (uint32_t)TR::kFull));
        typename std::conditional<sizeof(T) == 4, QEnc, QEnc64>::type e;
        M8 m8;
        uint32_t mexcl = 0;
        uint32_t zex = 0;   // lane b < TILE: in-tile payload offset of block b
        uint32_t rfin = 0;  // generic path: the final R of block kq in byte kq (after the R2 guard)
        auto generic = [&](bool pack) {
            // whole-warp encoder, one block at a time (raw blocks, the partial last block)
            for (int kq = 0; kq < 4; kq++) {
                const int bj = warp * 4 + kq;
                const bool bv = __shfl_sync(0xffffffffu, valid, 8 * kq);
                const uint32_t bk = __shfl_sync(0xffffffffu, mk, 8 * kq);
                const T bmu = TR::from(__shfl_sync(0xffffffffu, TR::bits(mu), 8 * kq));
                const uint32_t brec = __shfl_sync(0xffffffffu, rec, 8 * kq);
                int bR = pack ? (int)((rfin >> (8 * kq)) & 0xFFu) : (int)__shfl_sync(0xffffffffu, R, 8 * kq);
                if (!bv) {
                    if (!pack && lane == 0) s_z[bj] = 0u;
                    continue;
                }
                T xw[4];
                typename TR::U uu[4];
                LaneCode lc;
                int cnt = 4, len = B;
                if (bk < nBfull) {
                    warp_vals(wib, kq, xw);
                } else {
                    cnt = load_lane<T, 4>(x, p.n, bk, lane, xw);
                    len = (int)(p.n - (uint64_t)bk * B);
                }
                if (!pack && bk >= nBfull && bR < TR::kFull) {
                    // the partial last block: the R2 guard / escalation runs here (R2)
                    encode_block<T, 4>(xw, cnt, len, bmu, bR, (brec & 0x80u) != 0, eb, uu, lc);
                    bR = lc.R;
                } else {
                    encode_known_R<T, 4>(xw, cnt, len, bR >= TR::kFull ? T(0) : bmu, bR, uu, lc);
                }
                if (!pack) {
                    rfin |= (uint32_t)bR << (8 * kq);
                    if (lane == 0) s_z[bj] = lc.z;
                } else {
                    pack_red<T, 4>(uu, lc, cnt, len, stg + __shfl_sync(0xffffffffu, zex, bj));
                    if (lane == 0 && bR >= TR::kFull) mus[bk] = U(0);  // raw: mu = +0 (R15)
                }
            }
        };
        if (fast) {
            T xv[16];
#pragma unroll
            for (int kq = 0; kq < C::CPL; kq++)
                reinterpret_cast<uint4*>(xv)[kq] =
                    lds_u128(wib + (uint32_t)q * C::BW + 16u * swzc<C::CPL>((uint32_t)(C::CPL * ql + kq)));
            if constexpr (sizeof(T) == 4) quarter_encode_f32(xv, mu, valid ? R : 9u, e, m8);
            else quarter_encode_f64(xv, mu, valid ? R : 12u, e, m8);
            uint32_t incl = shfl_up_add8e<1>(e.msum);
            incl = shfl_up_add8e<2>(incl);
            incl = shfl_up_add8e<4>(incl);
            mexcl = incl - e.msum;
            const uint32_t tot = __shfl_sync(0xffffffffu, incl, 7, 8);
            if (ql == 0) s_z[j] = valid ? 33u + tot : 0u;
        } else {
            generic(false);
        }
        bar_compute(C::NTC);  // (C) every block's z_k; the next ticket
        const uint32_t nxt = (uint32_t)s_cur;
        const Meta mn = load_meta(nxt);
        {   // in-tile offsets of the blocks (every warp scans the tile's z_k itself)
            const uint32_t zl = lane < C::TILE ? s_z[lane] : 0u;
            const uint32_t incl = warp_incl_scan(zl);
            const uint32_t zoff = __shfl_sync(0xffffffffu, incl - zl, j);
            const uint32_t T_ = __shfl_sync(0xffffffffu, incl, 31);
            if (warp == 0) {
                const uint32_t ncl = cur * (uint32_t)C::TILE + (uint32_t)lane;
                if (lane < C::TILE && ncl < nnc32) zsize[ncl] = (uint16_t)zl;
                if (lane == 0) {
                    st_relaxed(&p.status_e[cur], kFlagAgg | T_);  // the tile's size, for the scanner
                    SZX_ETL(cur, 0);
                }
            }
            zex = incl - zl;
            if (fast) {
                if (valid && !SZX_EXP_NOPACK) {
                    if constexpr (sizeof(T) == 4) quarter_pack_f32(e, m8, R, mexcl, stg + zoff);
                    else quarter_pack_f64(e, m8, R, mexcl, stg + zoff);
                }
            } else {
                generic(true);
            }
            if (tid == 0) {
                s_T[slot] = T_;
                s_tile[slot] = cur;
            }
        }
        // the next tile's values: its metadata arrived during the scan / pack
        if (nxt < ntiles) stage(mn, buf ^ 1);
        if (k + 1 >= NS) retire(k + 1 - NS, pv);  // (its barrier also orders this pack before the next zeroing)
        cur = nxt;
        mc = mn;
    }
    // drain: the tiles still in their slots, in order
    const uint32_t k0 = k + 1 >= NS ? k + 1 - NS : 0;
    for (uint32_t kk = k0; kk < k; kk++) retire(kk, tid == 0 ? ld_relaxed(&p.prefix_e[s_tile[kk % NS]]) : 0);
}

}  // namespace szx
