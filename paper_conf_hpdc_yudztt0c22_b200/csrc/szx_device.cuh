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
    __device__ static U bits(float f) { return __float_as_uint(f); }
    __device__ static float from(U u) { return __uint_as_float(u); }
    __device__ static int expo(float f) { return int((__float_as_uint(f) >> 23) & 0xFF) - 127; }
    __device__ static float sub(float a, float b) { return __fsub_rn(a, b); }
    __device__ static float add(float a, float b) { return __fadd_rn(a, b); }
    __device__ static float half(float a) { return __fmul_rn(a, 0.5f); }
    __device__ static int clz(U u) { return __clz(u); }
    __device__ static bool isnan_(float f) { return f != f; }
};
template <> struct Traits<double> {
    using U = uint64_t;
    static constexpr int W = 8;
    static constexpr int kFloor = 12;
    static constexpr int kFull = 64;
    __device__ static U bits(double f) { return (U)__double_as_longlong(f); }
    __device__ static double from(U u) { return __longlong_as_double((long long)u); }
    __device__ static int expo(double f) { return int(((U)__double_as_longlong(f) >> 52) & 0x7FF) - 1023; }
    __device__ static double sub(double a, double b) { return __dsub_rn(a, b); }
    __device__ static double add(double a, double b) { return __dadd_rn(a, b); }
    __device__ static double half(double a) { return __dmul_rn(a, 0.5); }
    __device__ static int clz(U u) { return __clzll((long long)u); }
    __device__ static bool isnan_(double f) { return f != f; }
};

__device__ inline int expo_f64(double e) {
    return int(((uint64_t)__double_as_longlong(e) >> 52) & 0x7FF) - 1023;
}

// Order-preserving unsigned key of a double (total order, -0 < +0).
__host__ __device__ inline uint64_t dkey(uint64_t bits) {
    return (bits & 0x8000000000000000ull) ? ~bits : (bits | 0x8000000000000000ull);
}
__host__ __device__ inline uint64_t dkey_inv(uint64_t k) {
    return (k & 0x8000000000000000ull) ? (k & 0x7FFFFFFFFFFFFFFFull) : ~k;
}
// Same for the data word (min/max in the data type).
__device__ inline uint32_t okey(uint32_t u) { return (u & 0x80000000u) ? ~u : (u | 0x80000000u); }
__device__ inline uint32_t okey_inv(uint32_t k) { return (k & 0x80000000u) ? (k & 0x7FFFFFFFu) : ~k; }
__device__ inline uint64_t okey(uint64_t u) { return dkey(u); }
__device__ inline uint64_t okey_inv(uint64_t k) { return dkey_inv(k); }

// eb_abs from the global finite range keys (reading R13): REL x (max - min)
// in double, canonical +0; no finite values -> 0.
__device__ inline double eb_from_range(int mode, double eb_user, const uint64_t* range_keys) {
    double e;
    if (mode == 0) {
        e = eb_user;
    } else {
        uint64_t kmin = range_keys[0], kmax = ~range_keys[1];
        if (range_keys[0] == ~0ull) {
            e = 0.0;
        } else {
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
__device__ inline uint32_t warp_incl_scan(uint32_t v) {
    const int lane = threadIdx.x & 31;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
        uint32_t t = __shfl_up_sync(0xffffffffu, v, o);
        if (lane >= o) v += t;
    }
    return v;
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

}  // namespace szx
