// Microbenchmark: HBM write throughput of different store orders over a
// 537 MB output (the decoder's output size for NYX 512^3 f32).
//   nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o build_exp/write_pattern scripts/write_pattern.cu
#include <cstdio>
#include <cstdint>
#include <cuda_runtime.h>

constexpr uint64_t N16 = (512ull * 512 * 512 * 4) / 16;  // 16-byte chunks

// P0: grid-stride, consecutive threads -> consecutive 16 B
__global__ void p_linear(uint4* y, uint64_t n16) {
    uint4 v = make_uint4(1, 2, 3, 4);
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16; i += (uint64_t)gridDim.x * blockDim.x)
        y[i] = v;
}
// P1: each warp owns tiles of TILE16 chunks (grid-stride over tiles), writes
// them front to back, 512 B per warp store
template <int TILE16>
__global__ void p_tile(uint4* y, uint64_t n16) {
    uint4 v = make_uint4(1, 2, 3, 4);
    const int lane = threadIdx.x & 31;
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nt = n16 / TILE16;
    for (uint64_t t = gw; t < nt; t += nw) {
        uint4* q = y + t * TILE16 + lane;
#pragma unroll 4
        for (int j = 0; j < TILE16 / 32; j++) q[j * 32] = v;
    }
}
// P2: a CTA owns a super tile of 8 warp tiles; warps interleave at 512 B
template <int TILE16>
__global__ void p_cta(uint4* y, uint64_t n16) {
    uint4 v = make_uint4(1, 2, 3, 4);
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5, nwarp = blockDim.x >> 5;
    const uint64_t span = (uint64_t)TILE16 * nwarp;
    const uint64_t nt = n16 / span;
    for (uint64_t t = blockIdx.x; t < nt; t += gridDim.x) {
        uint4* q = y + t * span + w * 32 + lane;
#pragma unroll 4
        for (int j = 0; j < TILE16 / 32; j++) q[(uint64_t)j * 32 * nwarp] = v;
    }
}

// P3: 32-byte stores per thread (st.global.v8.b32, sm_100)
__global__ void p_v8(uint4* y, uint64_t n16) {
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n16 / 2; i += (uint64_t)gridDim.x * blockDim.x) {
        uint4* q = y + 2 * i;
        asm volatile("st.global.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};" ::"l"(q), "r"(1), "r"(2), "r"(3), "r"(4),
                     "r"(5), "r"(6), "r"(7), "r"(8) : "memory");
    }
}
// P4: linear, 4 independent 16 B stores per thread per iteration
__global__ void p_unr(uint4* y, uint64_t n16) {
    uint4 v = make_uint4(1, 2, 3, 4);
    const uint64_t T = (uint64_t)gridDim.x * blockDim.x;
    for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i + 3 * T < n16; i += 4 * T) {
        y[i] = v; y[i + T] = v; y[i + 2 * T] = v; y[i + 3 * T] = v;
    }
}
// P5: per warp, fill a 4 KB shared buffer once, then bulk-copy it (TMA) to
// consecutive 4 KB chunks of its 16 KB tiles
__global__ void p_tma(uint4* y, uint64_t n16) {
    __shared__ __align__(128) uint4 buf[8][256];
    const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
    for (int i = lane; i < 256; i += 32) buf[w][i] = make_uint4(1, 2, 3, 4);
    asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
    __syncwarp();
    const uint64_t gw = ((uint64_t)blockIdx.x * blockDim.x + threadIdx.x) >> 5;
    const uint64_t nw = ((uint64_t)gridDim.x * blockDim.x) >> 5;
    const uint64_t nt = n16 / 1024;
    const uint32_t sa = (uint32_t)__cvta_generic_to_shared(&buf[w][0]);
    for (uint64_t t = gw; t < nt; t += nw) {
        if (lane == 0) {
            for (int j = 0; j < 4; j++)
                asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], 4096;" ::"l"(y + t * 1024 + j * 256), "r"(sa) : "memory");
            asm volatile("cp.async.bulk.commit_group;" ::: "memory");
            asm volatile("cp.async.bulk.wait_group.read 8;" ::: "memory");
        }
        __syncwarp();
    }
    if (lane == 0) asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
}

template <typename F>
float timeit(F f) {
    cudaEvent_t a, b;
    cudaEventCreate(&a); cudaEventCreate(&b);
    for (int i = 0; i < 3; i++) f();
    cudaEventRecord(a);
    const int R = 20;
    for (int i = 0; i < R; i++) f();
    cudaEventRecord(b);
    cudaEventSynchronize(b);
    float ms; cudaEventElapsedTime(&ms, a, b);
    return ms * 1000 / R;
}

int main() {
    uint4* y;
    cudaMalloc(&y, N16 * 16);
    int sms; cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, 0);
    auto rep = [&](const char* name, float us) { printf("%-34s %8.1f us  %7.0f GB/s\n", name, us, N16 * 16 / (us * 1e3)); };
    for (int per : {4, 8, 16}) {
        char nm[64]; snprintf(nm, 64, "linear %d CTA/SM", per);
        rep(nm, timeit([&] { p_linear<<<sms * per, 256>>>(y, N16); }));
    }
    for (int per : {3, 4, 8}) {
        char nm[64];
        snprintf(nm, 64, "warp tile 16KB %d CTA/SM", per);
        rep(nm, timeit([&] { p_tile<1024><<<sms * per, 256>>>(y, N16); }));
        snprintf(nm, 64, "warp tile 2KB %d CTA/SM", per);
        rep(nm, timeit([&] { p_tile<128><<<sms * per, 256>>>(y, N16); }));
        snprintf(nm, 64, "cta interleaved 16KB/warp %d CTA/SM", per);
        rep(nm, timeit([&] { p_cta<1024><<<sms * per, 256>>>(y, N16); }));
    }
    for (int per : {4, 8, 16}) {
        char nm[64];
        snprintf(nm, 64, "v8 32B stores %d CTA/SM", per);
        rep(nm, timeit([&] { p_v8<<<sms * per, 256>>>(y, N16); }));
        snprintf(nm, 64, "unrolled x4 %d CTA/SM", per);
        rep(nm, timeit([&] { p_unr<<<sms * per, 256>>>(y, N16); }));
        snprintf(nm, 64, "tma bulk 4KB %d CTA/SM", per);
        rep(nm, timeit([&] { p_tma<<<sms * per, 256>>>(y, N16); }));
    }
    cudaError_t e = cudaDeviceSynchronize();
    printf("%s\n", cudaGetErrorString(e));
    return 0;
}
