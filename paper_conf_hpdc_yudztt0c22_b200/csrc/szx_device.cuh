// szx_device.cuh -- device helpers shared by the SZx sm_100a kernels.
//
// Everything here is written from the paper (HPDC'22, PAPER.md) and the
// readings of DESIGN.md section 3; it shares no code with oracle/.
// All floating-point arithmetic uses explicit round-to-nearest intrinsics
// (__fadd_rn, __fsub_rn, __fmul_rn, __dadd_rn, ...) which are never fused
// into FMAs; the library is additionally built with -fmad=false.
#pragma once

#include <cstdint>
#include <cuda_runtime.h>

namespace szx {

constexpr int kHeaderBytes = 64;
constexpr int kTileBlocks = 32;        // compress/decompress tile = one 32-bit bitmap word
constexpr uint64_t kFlagAgg = 1ull << 62;
constexpr uint64_t kFlagIncl = 2ull << 62;
constexpr uint64_t kValueMask = (1ull << 62) - 1;

__host__ __device__ inline uint64_t al16(uint64_t x) { return (x + 15) & ~uint64_t(15); }
__host__ __device__ inline uint64_t umin64(uint64_t a, uint64_t b) { return a < b ? a : b; }

// ---------------------------------------------------------------- words
template <typename T> struct Traits;
template <> struct Traits<float> {
    using U = uint32_t;
    static constexpr int W = 4;
    static constexpr int kFloor = 9;   // sign + exponent bits (reading R3)
    static constexpr int kFull = 32;   // "fullbits" (Formula 4) -> raw block
    static constexpr uint32_t kKeyPInf = 0xFF800000u;  // okey(+Inf); NaN keys lie outside
    static constexpr uint32_t kKeyNInf = 0x007FFFFFu;  // okey(-Inf)  [kKeyNInf, kKeyPInf]
    __device__ static U bits(float f) { return __float_as_uint(f); }
    __device__ static float from(U u) { return __uint_as_float(u); }
    __device__ static int expo(float f) { return int((__float_as_uint(f) >> 23) & 0xFF) - 127; }
    __device__ static float sub(float a, float b) { return __fsub_rn(a, b); }
    __device__ static float add(float a, float b) { return __fadd_rn(a, b); }
    __device__ static float half(float a) { return __fmul_rn(a, 0.5f); }
    __device__ static int clz(U u) { return __clz(u); }
    __device__ static bool isnan_(float f) { return f != f; }
    // x*0 + acc: stays +-0 while every x is finite, NaN once one is not
    __device__ static float fma0(float x, float acc) { return __fmaf_rn(x, 0.0f, acc); }
    __device__ static float fmin_(float a, float b) { return fminf(a, b); }
    __device__ static float fmax_(float a, float b) { return fmaxf(a, b); }
};
template <> struct Traits<double> {
    using U = uint64_t;
    static constexpr int W = 8;
    static constexpr int kFloor = 12;
    static constexpr int kFull = 64;
    static constexpr uint64_t kKeyPInf = 0xFFF0000000000000ull;
    static constexpr uint64_t kKeyNInf = 0x000FFFFFFFFFFFFFull;
    __device__ static U bits(double f) { return (U)__double_as_longlong(f); }
    __device__ static double from(U u) { return __longlong_as_double((long long)u); }
    __device__ static int expo(double f) { return int(((U)__double_as_longlong(f) >> 52) & 0x7FF) - 1023; }
    __device__ static double sub(double a, double b) { return __dsub_rn(a, b); }
    __device__ static double add(double a, double b) { return __dadd_rn(a, b); }
    __device__ static double half(double a) { return __dmul_rn(a, 0.5); }
    __device__ static int clz(U u) { return __clzll((long long)u); }
    __device__ static bool isnan_(double f) { return f != f; }
    __device__ static double fma0(double x, double acc) { return __fma_rn(x, 0.0, acc); }
    __device__ static double fmin_(double a, double b) { return ::fmin(a, b); }
    __device__ static double fmax_(double a, double b) { return ::fmax(a, b); }
};

__device__ inline int expo_f64(double e) {
    return int(((uint64_t)__double_as_longlong(e) >> 52) & 0x7FF) - 1023;
}

// Opaque copy: stops the optimiser from proving that an integer came from a
// float bitcast and rewriting sign-bit logic as float ops (observed: nvcc
// turned `u | 0x80000000` into FADD -|x|, which canonicalises NaN payloads).
__device__ inline uint32_t launder(uint32_t u) {
    asm("mov.b32 %0, %0;" : "+r"(u));
    return u;
}
__device__ inline uint64_t launder(uint64_t u) {
    asm("mov.b64 %0, %0;" : "+l"(u));
    return u;
}

// Order-preserving unsigned key of a double (total order, -0 < +0).
__host__ __device__ inline uint64_t dkey(uint64_t bits) {
#ifdef __CUDA_ARCH__
    bits = launder(bits);
#endif
    return (bits & 0x8000000000000000ull) ? ~bits : (bits | 0x8000000000000000ull);
}
__host__ __device__ inline uint64_t dkey_inv(uint64_t k) {
    return (k & 0x8000000000000000ull) ? (k & 0x7FFFFFFFFFFFFFFFull) : ~k;
}
// Same for the data word (min/max in the data type).
__device__ inline uint32_t okey(uint32_t u) {
    u = launder(u);
    return (u & 0x80000000u) ? ~u : (u | 0x80000000u);
}
__device__ inline uint32_t okey_inv(uint32_t k) { return (k & 0x80000000u) ? (k & 0x7FFFFFFFu) : ~k; }
__device__ inline uint64_t okey(uint64_t u) { return dkey(u); }
__device__ inline uint64_t okey_inv(uint64_t k) { return dkey_inv(k); }

// eb_abs from the global finite range keys (reading R13): REL x (max - min)
// in double, canonical +0; no finite values -> 0.
__device__ inline double eb_from_range(int mode, double eb_user, const uint64_t* range_keys,
                                       const double* eb_abs_in = nullptr) {
    double e;
    if (eb_abs_in) {  // the caller already holds the (global) absolute bound
        e = *eb_abs_in;
    } else if (mode == 0) {
        e = eb_user;
    } else {
        if (!range_keys || range_keys[0] == ~0ull) {
            e = 0.0;
        } else {
            const uint64_t kmin = range_keys[0], kmax = ~range_keys[1];
            double gmin = __longlong_as_double((long long)dkey_inv(kmin));
            double gmax = __longlong_as_double((long long)dkey_inv(kmax));
            e = __dmul_rn(eb_user, __dsub_rn(gmax, gmin));
        }
    }
    if (e == 0.0) e = 0.0;
    return e;
}

// ---------------------------------------------------------------- warp ops
__device__ inline uint32_t warp_min(uint32_t v) { return __reduce_min_sync(0xffffffffu, v); }
__device__ inline uint32_t warp_max(uint32_t v) { return __reduce_max_sync(0xffffffffu, v); }
__device__ inline uint64_t warp_min(uint64_t v) {
#pragma unroll
    for (int o = 16; o; o >>= 1) { uint64_t t = __shfl_xor_sync(0xffffffffu, v, o); v = t < v ? t : v; }
    return v;
}
__device__ inline uint64_t warp_max(uint64_t v) {
#pragma unroll
    for (int o = 16; o; o >>= 1) { uint64_t t = __shfl_xor_sync(0xffffffffu, v, o); v = t > v ? t : v; }
    return v;
}
__device__ inline uint32_t warp_sum(uint32_t v) { return __reduce_add_sync(0xffffffffu, v); }
__device__ inline uint64_t warp_sum64(uint64_t v) {
#pragma unroll
    for (int o = 16; o; o >>= 1) v += __shfl_xor_sync(0xffffffffu, v, o);
    return v;
}
// inclusive prefix sum over the warp
// (shfl.up's own in-range predicate guards the add: one SHFL + one IADD per step)
template <int O>
__device__ inline uint32_t shfl_up_add(uint32_t v) {
    asm volatile(
        "{\n\t.reg .u32 t;\n\t.reg .pred p;\n\t"
        "shfl.sync.up.b32 t|p, %0, %1, 0, -1;\n\t"
        "@p add.u32 %0, %0, t;\n\t}"
        : "+r"(v)
        : "n"(O));
    return v;
}
__device__ inline uint32_t warp_incl_scan(uint32_t v) {
    v = shfl_up_add<1>(v);
    v = shfl_up_add<2>(v);
    v = shfl_up_add<4>(v);
    v = shfl_up_add<8>(v);
    v = shfl_up_add<16>(v);
    return v;
}

// (c & ~m) | (v & m) in one LOP3 (the compiler otherwise materialises v & m
// separately when it is reused)
__device__ __forceinline__ uint32_t bitsel(uint32_t c, uint32_t v, uint32_t m) {
    uint32_t d;
    asm("lop3.b32 %0, %1, %2, %3, 0xD8;" : "=r"(d) : "r"(c), "r"(v), "r"(m));
    return d;
}

// ---------------------------------------------------------------- PDL
// Programmatic dependent launch: wait until the preceding kernel in the stream
// has completed and its memory is visible (no-op when launched without PDL),
// and let the next kernel start launching while this one drains.
__device__ inline void pdl_wait() { asm volatile("griddepcontrol.wait;" ::: "memory"); }
__device__ inline void pdl_trigger() { asm volatile("griddepcontrol.launch_dependents;" ::: "memory"); }

// ---------------------------------------------------------------- cp.async
__device__ inline void cp_async16(uint32_t saddr, const void* g) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(saddr), "l"(g) : "memory");
}
// 16-byte copy of which only the first `src_bytes` (1..16) are read; the rest is zero-filled
__device__ inline void cp_async16_zfill(uint32_t saddr, const void* g, uint32_t src_bytes) {
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16, %2;" ::"r"(saddr), "l"(g), "r"(src_bytes) : "memory");
}
__device__ inline void cp_async_commit() { asm volatile("cp.async.commit_group;" ::: "memory"); }
template <int N>
__device__ inline void cp_async_wait() { asm volatile("cp.async.wait_group %0;" ::"n"(N) : "memory"); }
__device__ inline uint4 lds_u128(uint32_t a) {
    uint4 v;
    asm volatile("ld.shared.v4.u32 {%0,%1,%2,%3}, [%4];" : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "r"(a));
    return v;
}

// ---------------------------------------------------------------- shared memory
// Explicit ld.shared (generic pointers into the staging buffers otherwise
// compile to generic LD.E).
__device__ inline uint32_t lds_u8(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u8 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
__device__ inline uint32_t lds_u32(uint32_t a) {
    uint32_t v;
    asm volatile("ld.shared.u32 %0, [%1];" : "=r"(v) : "r"(a));
    return v;
}
// Run of bytes starting at an arbitrary shared address, realigned into NW words.
template <int NW>
__device__ inline void run_load_s(uint32_t a, uint32_t (&r)[NW]) {
    // __funnelshift_r wraps its amount mod 32, so 8 a selects the byte offset a & 3
    const uint32_t base = a & ~3u, sh = 8 * a;
    uint32_t lo = lds_u32(base);
#pragma unroll
    for (int q = 0; q < NW; q++) {
        const uint32_t hi = lds_u32(base + 4 * (q + 1));
        r[q] = __funnelshift_r(lo, hi, sh);
        lo = hi;
    }
}
// Drop the first k (0..4) bytes of a run: clamped funnel shifts (a shift of
// 32 yields the next word), no data-dependent word moves.
template <int NW>
__device__ inline void run_drop4(uint32_t (&a)[NW], uint32_t k) {
    const uint32_t sh = 8 * k;
#pragma unroll
    for (int q = 0; q < NW - 1; q++) a[q] = __funnelshift_rc(a[q], a[q + 1], sh);
    a[NW - 1] = __funnelshift_rc(a[NW - 1], 0u, sh);
}

// ---------------------------------------------------------------- byte runs
// A lane's run of mid-bytes (at most VPL*W bytes) held little-endian in NW
// 32-bit words, byte 0 first.  Shifts by k <= 8 bytes across the words.
template <int NW>
__device__ inline void run_shr(uint32_t (&a)[NW], int k) {
    // whole words first (k >> 2 is 0, 1 or 2), then the k & 3 remaining bytes;
    // funnel shifts take their amount mod 32, so 4-byte steps must not reach them
#pragma unroll
    for (int r = 0; r < 2; r++) {
        if (k >= 4) {
#pragma unroll
            for (int q = 0; q < NW - 1; q++) a[q] = a[q + 1];
            a[NW - 1] = 0;
            k -= 4;
        }
    }
    const int sh = 8 * k;
#pragma unroll
    for (int q = 0; q < NW - 1; q++) a[q] = __funnelshift_r(a[q], a[q + 1], sh);
    a[NW - 1] = sh ? a[NW - 1] >> sh : a[NW - 1];
}

// ---------------------------------------------------------------- memory
__device__ inline uint64_t ld_relaxed(const uint64_t* p) {
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ inline void st_relaxed(uint64_t* p, uint64_t v) {
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
// streaming 16-byte load (read once; do not keep in L1)
__device__ inline uint4 ld_stream16(const void* p) {
    uint4 v;
    asm volatile("ld.global.nc.L1::no_allocate.v4.u32 {%0,%1,%2,%3}, [%4];"
                 : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(p));
    return v;
}

// ---------------------------------------------------------------- lane chunks
// A lane's VPL values of a block are LB = VPL x W contiguous bytes, moved as
// NQ chunks of CB = min(LB, 16) bytes (16-byte vectors for b >= 128 float32,
// 4- or 8-byte words for the small blocks b = 32 / 64).
template <int CB> struct ChunkT;
template <> struct ChunkT<4> { using V = uint32_t; };
template <> struct ChunkT<8> { using V = uint2; };
template <> struct ChunkT<16> { using V = uint4; };
template <typename T, int VPL>
struct Lay {
    static constexpr int LB = VPL * (int)sizeof(T);
    static constexpr int CB = LB < 16 ? LB : 16;
    static constexpr int NQ = LB / CB;
    using V = typename ChunkT<CB>::V;
};
// streaming load of one chunk (read once; do not keep in L1)
template <typename V>
__device__ inline V ld_stream(const V* p);
template <>
__device__ inline uint4 ld_stream<uint4>(const uint4* p) { return ld_stream16(p); }
template <>
__device__ inline uint2 ld_stream<uint2>(const uint2* p) {
    uint2 v;
    asm volatile("ld.global.nc.L1::no_allocate.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "l"(p));
    return v;
}
template <>
__device__ inline uint32_t ld_stream<uint32_t>(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.global.nc.L1::no_allocate.u32 %0, [%1];" : "=r"(v) : "l"(p));
    return v;
}
// shared-memory load of one chunk
template <typename V>
__device__ inline V lds_chunk(uint32_t a);
template <>
__device__ inline uint4 lds_chunk<uint4>(uint32_t a) { return lds_u128(a); }
template <>
__device__ inline uint2 lds_chunk<uint2>(uint32_t a) {
    uint2 v;
    asm volatile("ld.shared.v2.u32 {%0,%1}, [%2];" : "=r"(v.x), "=r"(v.y) : "r"(a));
    return v;
}
template <>
__device__ inline uint32_t lds_chunk<uint32_t>(uint32_t a) { return lds_u32(a); }
// asynchronous global -> shared copy of one chunk
template <int CB>
__device__ inline void cp_async_chunk(uint32_t saddr, const void* g) {
    if constexpr (CB == 16) cp_async16(saddr, g);
    else asm volatile("cp.async.ca.shared.global [%0], [%1], %2;" ::"r"(saddr), "l"(g), "n"(CB) : "memory");
}
// Lead codes of a lane (2 bits per value, LSB-first, reading R8): byte
// lane*VPL/4 of the code array, at bit (2*VPL*lane) % 8 when VPL < 4.
template <int VPL>
__device__ inline uint32_t code_byte(int lane) { return (uint32_t)(lane * VPL / 4); }
template <int VPL>
__device__ inline uint32_t code_shift(int lane) { return VPL >= 4 ? 0u : (uint32_t)((2 * VPL * lane) & 7); }

// ---------------------------------------------------------------- addresses
__device__ inline uint32_t smem_u32(const void* p) { return (uint32_t)__cvta_generic_to_shared(p); }

// Decoupled look-back (single-pass prefix scan, Merrill & Garland) over
// per-tile aggregates.  Called by all 32 lanes of ONE warp of the tile's CTA;
// returns the exclusive prefix of `agg` (broadcast to all lanes).  Tile ids
// must be handed out in launch order (atomic ticket) so every predecessor is
// resident or finished: forward progress is guaranteed.
__device__ inline uint64_t lookback_exclusive(uint64_t* status, uint64_t tile, uint64_t agg) {
    const int lane = threadIdx.x & 31;
    if (tile == 0) {
        if (lane == 0) st_relaxed(&status[0], kFlagIncl | agg);
        return 0;
    }
    if (lane == 0) st_relaxed(&status[tile], kFlagAgg | agg);
    uint64_t excl = 0;
    int64_t base = (int64_t)tile - 1;
    while (true) {
        const int64_t idx = base - lane;
        uint64_t s = idx >= 0 ? ld_relaxed(&status[idx]) : kFlagIncl;
        const uint32_t pm = __ballot_sync(0xffffffffu, (s >> 62) == 2);
        const uint32_t im = __ballot_sync(0xffffffffu, (s >> 62) == 0);
        const int firstP = pm ? __ffs(pm) - 1 : 32;
        const uint32_t need = firstP >= 31 ? 0xffffffffu : ((2u << firstP) - 1u);
        if (im & need) continue;  // a predecessor has not published yet: re-read the window
        uint64_t v = (lane <= firstP) ? (s & kValueMask) : 0;
        excl += warp_sum64(v);
        if (firstP < 32) break;
        base -= 32;
    }
    if (lane == 0) st_relaxed(&status[tile], kFlagIncl | (excl + agg));
    return excl;
}

// ------------------------------------------------- co-resident grid helpers
// Used by persistent kernels whose grid never exceeds the number of CTAs the
// device can hold at once (grid <= SMs x occupancy, set on the host), so every
// CTA is running and spinning on another CTA's flag cannot deadlock.

__device__ inline uint32_t ld_acquire_u32(const uint32_t* p) {
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}

// Sum over the CTA (any blockDim that is a multiple of 32, <= 1024); result
// in every thread.  s_w: shared scratch of 32 u64.
__device__ inline uint64_t cta_sum64(uint64_t v, uint64_t* s_w) {
    const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    v = warp_sum64(v);
    __syncthreads();  // s_w may still be read by a previous call
    if (lane == 0) s_w[warp] = v;
    __syncthreads();
    uint64_t t = 0;
    for (int i = 0; i < nwarp; i++) t += s_w[i];
    return t;
}

// Grid-wide exclusive prefix of one aggregate per CTA, in CTA order.  Each
// CTA stores its aggregate and takes an arrival ticket; the last CTA to
// arrive scans all aggregates and publishes each CTA's prefix (flag bit 63)
// in res[]; every CTA waits on its own entry.  Cost: one atomic per CTA and
// about three round trips, with no chained look-back and no all-to-all
// polling.  `res` [gridDim.x] and `*arrive` must be zero.
constexpr uint64_t kSlotFlag = 1ull << 63;
// (over the first G CTAs of the grid; all of them must call it)
__device__ inline uint64_t grid_excl_prefix(uint64_t* slots, uint64_t* res, uint32_t* arrive, uint64_t agg,
                                            uint64_t* s_w /*[32]*/, uint32_t G) {
    __shared__ uint32_t s_last;
    __shared__ uint64_t s_val;
    if (threadIdx.x == 0) {
        st_relaxed(&slots[blockIdx.x], agg);
        __threadfence();
        s_last = atomicAdd(arrive, 1u) == G - 1;
    }
    __syncthreads();
    if (s_last) {
        __threadfence();
        uint64_t run = 0;
        for (uint32_t b0 = 0; b0 < G; b0 += blockDim.x) {
            const uint32_t i = b0 + threadIdx.x;
            const uint64_t v = i < G ? ld_relaxed(&slots[i]) : 0;
            // CTA exclusive scan of v
            const int lane = threadIdx.x & 31, warp = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
            uint64_t incl = v;
#pragma unroll
            for (int o = 1; o < 32; o <<= 1) {
                const uint64_t t = __shfl_up_sync(0xffffffffu, incl, o);
                if (lane >= o) incl += t;
            }
            __syncthreads();
            if (lane == 31) s_w[warp] = incl;
            __syncthreads();
            uint64_t wpre = 0, tot = 0;
            for (int k = 0; k < nwarp; k++) {
                wpre += k < warp ? s_w[k] : 0;
                tot += s_w[k];
            }
            if (i < G) st_relaxed(&res[i], kSlotFlag | (run + wpre + incl - v));
            run += tot;
        }
    }
    if (threadIdx.x == 0) {
        uint64_t v;
        while (!((v = ld_relaxed(&res[blockIdx.x])) & kSlotFlag)) __nanosleep(32);
        s_val = v & ~kSlotFlag;
    }
    __syncthreads();
    return s_val;
}

#ifndef SZX_GBAR_NS
#define SZX_GBAR_NS 256  // grid barrier: polling back-off cap (ns)
#endif
// Grid barrier: every global write made by any thread of any CTA before the
// call is visible to every thread after it.  `ctr` must be zero.
__device__ inline void grid_barrier(uint32_t* ctr) {
    __syncthreads();
    if (threadIdx.x == 0) {
        __threadfence();
        atomicAdd(ctr, 1u);
        uint32_t ns = 32;
        while (ld_acquire_u32(ctr) < gridDim.x) {
            __nanosleep(ns);
            ns = ns < SZX_GBAR_NS ? 2 * ns : ns;
        }
        __threadfence();
    }
    __syncthreads();
}

}  // namespace szx
