// szx_api.cu -- host side of libszx_b200.so: the C ABI declared in
// include/szx.h.  Validates arguments, lays out the stream (DESIGN.md s.4)
// and the workspace, and enqueues the sm_100a kernels on the caller's
// stream.  No CPU fallback: every compute path runs in the kernels below.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cmath>
#include <cstring>
#include <map>
#include <type_traits>
#include <mutex>
#include <vector>

#include "../../include/szx.h"
#include "szx_compress.cuh"
#include "szx_decompress.cuh"
#include "szx_encode.cuh"

using namespace szx;

namespace {

constexpr uint64_t kMaxN = 1ull << 36;
// the decoder's index phase packs a block count and a tile count into the two
// 32-bit halves of one u64 (szx_decompress.cuh, index_phase); the smallest
// block size (32) bounds the block count
static_assert(kMaxN / 32 < (1ull << 32), "block counts must fit 32 bits");

std::atomic<uint64_t> g_launches{0};
std::atomic<int> g_rbias{0};

// ------------------------------------------------------------ kernel timing
struct Timing {
    std::mutex mu;
    bool on = false;
    std::vector<const char*> names;
    std::vector<double> ms;
    std::vector<uint64_t> cnt;
    struct Pending { int id; cudaEvent_t a, b; };
    std::vector<Pending> pending;
    std::vector<cudaEvent_t> pool;
    int id_of(const char* n) {
        for (size_t i = 0; i < names.size(); i++) if (!strcmp(names[i], n)) return (int)i;
        names.push_back(n); ms.push_back(0); cnt.push_back(0);
        return (int)names.size() - 1;
    }
    cudaEvent_t ev() {
        if (!pool.empty()) { cudaEvent_t e = pool.back(); pool.pop_back(); return e; }
        cudaEvent_t e; cudaEventCreate(&e); return e;
    }
    void resolve() {
        for (auto& p : pending) {
            float t = 0;
            cudaEventSynchronize(p.b);
            cudaEventElapsedTime(&t, p.a, p.b);
            ms[p.id] += t; cnt[p.id] += 1;
            pool.push_back(p.a); pool.push_back(p.b);
        }
        pending.clear();
    }
};
Timing& timing() { static Timing t; return t; }

template <typename F>
void launch(const char* name, cudaStream_t s, F&& f) {
    Timing& T = timing();
    bool on;
    { std::lock_guard<std::mutex> g(T.mu); on = T.on; }
    if (!on) { f(); g_launches++; return; }
    std::lock_guard<std::mutex> g(T.mu);
    cudaEvent_t a = T.ev(), b = T.ev();
    cudaEventRecord(a, s);
    f();
    cudaEventRecord(b, s);
    T.pending.push_back({T.id_of(name), a, b});
    g_launches++;
}

std::atomic<bool> g_timing_on{false};  // mirrors Timing::on without taking its mutex
bool timing_on() { return g_timing_on.load(); }

// cudaLaunchKernelEx with programmatic stream serialization (PDL): the kernel
// may start launching while its predecessor drains; it calls pdl_wait() before
// touching the predecessor's output.  Disabled while per-kernel timing events
// sit between the launches.
template <typename... KArgs, typename... Args>
void launch_pdl(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[1];
    at[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[0].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = timing_on() ? 0 : 1;
    cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

// Cooperative launch (co-residency guaranteed by the driver or the launch
// fails) for the persistent kernels that spin on other CTAs' flags, combined
// with PDL when the driver accepts both attributes; otherwise cooperative only.
template <typename... KArgs, typename... Args>
void launch_coop(void (*k)(KArgs...), dim3 grid, dim3 block, size_t smem, cudaStream_t s, Args... args) {
    cudaLaunchConfig_t cfg = {};
    cfg.gridDim = grid;
    cfg.blockDim = block;
    cfg.dynamicSmemBytes = smem;
    cfg.stream = s;
    cudaLaunchAttribute at[2];
    at[0].id = cudaLaunchAttributeCooperative;
    at[0].val.cooperative = 1;
    at[1].id = cudaLaunchAttributeProgrammaticStreamSerialization;
    at[1].val.programmaticStreamSerializationAllowed = 1;
    cfg.attrs = at;
    cfg.numAttrs = timing_on() ? 1 : 2;
    if (cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...) == cudaSuccess) return;
    cudaGetLastError();
    cfg.numAttrs = 1;
    cudaLaunchKernelEx(&cfg, k, static_cast<KArgs>(args)...);
}

void timing_resolve() {
    Timing& T = timing();
    std::lock_guard<std::mutex> g(T.mu);
    T.resolve();
}

int sm_count() {
    int dev = 0, sms = 148;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    return sms > 0 ? sms : 148;
}

bool have_device() {
    int n = 0;
    if (cudaGetDeviceCount(&n) != cudaSuccess) { cudaGetLastError(); return false; }
    return n > 0;
}

// The library's own temporaries (workspaces of the convenience entry points,
// device buffers of the host entry points) come from the device's default
// stream-ordered pool.  Keep freed memory in the pool instead of returning it
// to the driver at every synchronisation, so repeated calls do not pay for
// mapping hundreds of MB again.
void keep_pool_memory() {
    static thread_local int done_dev = -1;
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return; }
    if (done_dev == dev) return;
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, dev) == cudaSuccess) {
        uint64_t thr = ~0ull;
        cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &thr);
    }
    cudaGetLastError();
    done_dev = dev;
}

uint64_t* pinned_u64() {
    static thread_local uint64_t* p = nullptr;
    if (!p && cudaMallocHost(&p, 64) != cudaSuccess) { cudaGetLastError(); p = nullptr; }
    return p;
}

bool aligned16(const void* p) { return (reinterpret_cast<uintptr_t>(p) & 15) == 0; }
int wbytes(szx_dtype_t dt) { return dt == SZX_F64 ? 8 : 4; }
bool block_ok(uint32_t b) { return b == 32 || b == 64 || b == 128 || b == 256; }
uint64_t cdiv(uint64_t a, uint64_t b) { return (a + b - 1) / b; }

// ------------------------------------------------------------ compress layout
struct CLayout {
    uint64_t nB, nW, nTB, nTC, nTE;
    uint64_t off_keys, off_zero, zero_bytes, off_scal, off_stats, off_nclist, off_nckeys, off_ncR, off_gbase,
        off_codes, codes_bytes, total;
};
CLayout clayout(uint64_t n, int W, uint32_t b) {
    CLayout L{};
    L.nB = cdiv(n, b);
    L.nW = cdiv(L.nB, 32);
    L.nTB = cdiv(L.nB, kClassifyMinBlocks);  // look-back words for the smallest classify tile
    L.nTC = cdiv(cdiv(L.nB, kWriteTile), 256);  // k_zscan CTAs (look-back status words)
    L.off_keys = 0;
    L.off_zero = 16;
    L.nTE = cdiv(L.nB, 4 * SZX_ENW) + 1;  // k_encode_fused tiles (scanner status words)
    L.zero_bytes = al16(16 + 16 * L.nTB + 8 * L.nTC + 16 * L.nTE);  // classify: 2 words per tile
    L.off_scal = L.off_zero + L.zero_bytes;
    L.off_stats = L.off_scal + 32;
    L.off_nclist = al16(L.off_stats + 2ull * W * L.nB);
    L.off_nckeys = al16(L.off_nclist + 4 * L.nB + 4);
    L.off_ncR = al16(L.off_nckeys + 2ull * W * L.nB + 16);
    L.off_gbase = al16(L.off_ncR + L.nB);
    L.off_codes = al16(L.off_gbase + 8 * (cdiv(L.nB, kWriteTile) + 2));
    L.codes_bytes = (W == 4 && b == 128) ? 32 * L.nB : 0;  // lead codes, size pass -> write pass
    L.total = al16(L.off_codes + L.codes_bytes) + 256;
    return L;
}

Plan make_plan(const CLayout& L, uint8_t* ws, uint64_t n, szx_dtype_t dt, szx_ebmode_t mode,
               double eb, uint32_t b, const uint64_t* range_keys) {
    Plan p{};
    p.n = n; p.nB = L.nB; p.nW = L.nW;
    p.off_mu = kHeaderBytes + al16(cdiv(L.nB, 8));
    p.b = b; p.dtype = (uint32_t)dt; p.mode = (uint32_t)mode;
    p.r_bias = g_rbias.load();
    p.eb_user = eb;
    p.range_keys = range_keys ? const_cast<uint64_t*>(range_keys) : reinterpret_cast<uint64_t*>(ws + L.off_keys);
    p.ctr = reinterpret_cast<uint32_t*>(ws + L.off_zero);
    p.status_b = reinterpret_cast<uint64_t*>(ws + L.off_zero + 16);
    p.status_c = p.status_b + 2 * L.nTB;
    p.status_e = p.status_c + L.nTC;
    p.prefix_e = p.status_e + L.nTE;
    p.eb_abs = reinterpret_cast<double*>(ws + L.off_scal);
    p.nnc = reinterpret_cast<uint64_t*>(ws + L.off_scal + 8);
    p.total = reinterpret_cast<uint64_t*>(ws + L.off_scal + 16);
    p.stats = ws + L.off_stats;
    p.nclist = reinterpret_cast<uint32_t*>(ws + L.off_nclist);
    p.ncmu = ws + L.off_nckeys;
    p.ncR = ws + L.off_ncR;
    p.gbase = reinterpret_cast<uint64_t*>(ws + L.off_gbase);
    p.nccodes = L.codes_bytes ? ws + L.off_codes : nullptr;
    return p;
}

int check_compress_args(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                        uint32_t b, const void* d_out) {
    if (dt != SZX_F32 && dt != SZX_F64) return SZX_EINVAL;
    if (mode != SZX_ABS && mode != SZX_REL) return SZX_EINVAL;
    if (!(eb >= 0.0) || !std::isfinite(eb)) return SZX_EINVAL;
    if (!block_ok(b) || n > kMaxN) return SZX_EINVAL;
    if (!d_out || !aligned16(d_out)) return SZX_EINVAL;
    if (n && (!d_in || !aligned16(d_in))) return SZX_EINVAL;
    return SZX_OK;
}

#ifndef SZX_CARVE
#define SZX_CARVE 0
#endif
// every kernel asks for the same L1/shared split, so consecutive kernels do
// not make the SMs drain and reconfigure the carve-out
template <typename K>
void carve(K k) {
    if (SZX_CARVE) cudaFuncSetAttribute(k, cudaFuncAttributePreferredSharedMemoryCarveout, SZX_CARVE);
}

// blocks per warp in flight in the stats pass: 128 bytes of loads per lane (at most 16 blocks)
template <typename T, int VPL>
constexpr int stats_unroll() {
    constexpr int u = 128 / (VPL * (int)sizeof(T));
    return u < 1 ? 1 : (u > 16 ? 16 : u);
}

// Per-device kernel set-up.  Function attributes (dynamic shared memory limit,
// carve-out) belong to the device context, and the occupancy that sizes the
// persistent grids is a property of the device, so both are cached per
// (device, kernel, dynamic smem), under a mutex (callers may be several host
// threads, each driving its own device).
struct KernelSetup {
    std::mutex mu;
    struct Key {
        int dev;
        const void* fn;
        size_t smem;
        bool operator<(const Key& o) const {
            if (dev != o.dev) return dev < o.dev;
            if (fn != o.fn) return fn < o.fn;
            return smem < o.smem;
        }
    };
    std::map<Key, int> occ;
};
KernelSetup& kernel_setup() { static KernelSetup k; return k; }

// Blocks of `k` per SM at 256 threads with `smem` dynamic bytes on the current
// device (attributes set on first use per device); `dflt` if the query fails.
template <typename K>
int kernel_occupancy(K k, size_t smem, int dflt, int threads = 256) {
    int dev = 0;
    if (cudaGetDevice(&dev) != cudaSuccess) { cudaGetLastError(); return dflt; }
    KernelSetup& S = kernel_setup();
    std::lock_guard<std::mutex> g(S.mu);
    const KernelSetup::Key key{dev, reinterpret_cast<const void*>(k), smem};
    auto it = S.occ.find(key);
    if (it != S.occ.end()) return it->second;
    carve(k);
    if (smem > 48 * 1024) cudaFuncSetAttribute(k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, k, threads, smem) != cudaSuccess || occ <= 0) {
        cudaGetLastError();
        occ = dflt;
    }
    S.occ[key] = occ;
    return occ;
}

// grid-stride streaming pass: enough CTAs to fill every SM, each warp keeping
// UNR blocks (128 bytes per lane) of loads in flight
template <typename T, int VPL>
void enqueue_stats(const void* d_in, const Plan& p, int want_range, cudaStream_t s) {
    constexpr int UNR = stats_unroll<T, VPL>();
    const int occ = kernel_occupancy(k_block_stats<T, VPL, UNR>, 0, 4);
    uint64_t grid = cdiv(p.nB, 8 * UNR);
    const uint64_t cap = (uint64_t)sm_count() * occ;
    if (grid > cap) grid = cap;
    if (grid == 0) grid = 1;
    launch("k_block_stats", s, [&] {
        k_block_stats<T, VPL, UNR><<<(unsigned)grid, 256, 0, s>>>(static_cast<const T*>(d_in), p, want_range);
    });
}

// classify, then the encoder: size pass (z_k and R per nonconstant block),
// offset scan, write pass.  Grids are sized for the worst case (every block
// nonconstant); CTAs beyond the device-side count exit at once.
template <typename T, int VPL>
void enqueue_encode(const void* d_in, const Plan& p, const CLayout& L, uint8_t* out, cudaStream_t s) {
    kernel_occupancy(k_zscan<Traits<T>::W>, 0, 1);
    {
#ifndef SZX_CLS_COOP
#define SZX_CLS_COOP 1   // classify: co-resident one-tile-per-CTA form when the tiles fit the grid
#endif
#ifndef SZX_CLS_TPSM
#define SZX_CLS_TPSM 4   // classify (co-resident form): at most this many tiles per SM (0 = occupancy; 2 -> 4: NYX classify 19.4 -> 16.8 us)
#endif
        // co-resident form: the smallest tile (blocks per thread) whose tile count
        // fits the co-resident grid; else tiles by ticket with a look-back scan
        bool done = false;
        auto coop = [&](auto kern, int bpt) {
            if (done) return;
            const int occ = kernel_occupancy(kern, 0, 1);
            uint64_t cap = (uint64_t)sm_count() * occ;
            if (SZX_CLS_TPSM) cap = std::min<uint64_t>(cap, (uint64_t)SZX_CLS_TPSM * sm_count());
            const uint64_t tiles = std::max<uint64_t>(1, cdiv(L.nB, 256ull * bpt));
            if (tiles > cap) return;
            done = true;
            launch("k_classify", s, [&] { launch_coop(kern, dim3((unsigned)tiles), dim3(256), 0, s, p, out); });
        };
        if (SZX_CLS_COOP) {
            coop(k_classify<T, 1, true>, 1);
            coop(k_classify<T, 2, true>, 2);
            coop(k_classify<T, 4, true>, 4);
            coop(k_classify<T, 8, true>, 8);
        }
        if (!done) {
            kernel_occupancy(k_classify<T, 8>, 0, 1);
            const uint64_t grid = std::max<uint64_t>(1, cdiv(L.nB, (uint64_t)kClassifyBlocks));
            launch("k_classify", s, [&] { launch_pdl(k_classify<T, 8>, dim3((unsigned)grid), dim3(256), 0, s, p, out); });
        }
    }
#ifndef SZX_FUSED
#define SZX_FUSED 1   // float32 b = 128: the fused single-pass encoder (szx_encode.cuh)
#endif
    if constexpr (VPL == 4) {
        if (SZX_FUSED) {
            // b = 128: the fused encoder; float64 keeps 2 staging slots (smem)
            constexpr int NS = sizeof(T) == 4 ? SZX_ENS : SZX_ENS64;
            using EC = EncCfg<T, SZX_ENW, NS>;
            auto kern = k_encode_fused<T, SZX_ENW, NS>;
            const int occ_e = kernel_occupancy(kern, EC::SMEM, 1, EC::NT);
            const uint64_t egrid = std::max<uint64_t>(
                1, std::min<uint64_t>(cdiv(L.nB, EC::TILE), (uint64_t)sm_count() * occ_e));
            launch("k_encode", s, [&] {
                launch_coop(kern, dim3((unsigned)egrid), dim3(EC::NT), EC::SMEM, s, static_cast<const T*>(d_in), p, out);
            });
            return;
        }
    }
    const int occ = kernel_occupancy(k_enc_size<T, VPL>, SizeCfg<T, VPL>::SMEM, 2);
    uint64_t grid = cdiv(L.nB, 8);
    const uint64_t cap = (uint64_t)sm_count() * occ;
    if (grid > cap) grid = cap;
    if (grid == 0) grid = 1;
    launch("k_enc_size", s, [&] {
        launch_pdl(k_enc_size<T, VPL>, dim3((unsigned)grid), dim3(256), SizeCfg<T, VPL>::SMEM, s,
                   static_cast<const T*>(d_in), p, out);
    });
    launch("k_zscan", s, [&] { launch_pdl(k_zscan<Traits<T>::W>, dim3((unsigned)L.nTC), dim3(256), 0, s, p, out); });
    using C = WriteCfg<T, VPL>;
#ifndef SZX_DITEMS
#define SZX_DITEMS 2        // decoder: target nonconstant work items per decode warp (tile split)
#endif
#ifndef SZX_DTS_MINT
#define SZX_DTS_MINT 4      // ... only with at least this many tiles per warp of the grid
#endif
#ifndef SZX_DTS
#define SZX_DTS 1           // decoder: thread-serial tiles on dense float32 b = 128 streams
#endif
#ifndef SZX_DSPLIT
#define SZX_DSPLIT 0        // decoder: force the tile split (1, 2, 4); 0 = by size
#endif
#ifndef SZX_ICTA_CHUNK
#define SZX_ICTA_CHUNK 0    // decoder: index CTAs <= 256-tile chunks (measured slower: the index work per CTA grows)
#endif
#ifndef SZX_ICTA_PER_SM
#define SZX_ICTA_PER_SM 1   // decoder CTAs per SM that run the index phase
#endif
#ifndef SZX_WGRIDK
#define SZX_WGRIDK 8
#endif
    const int occ_w = kernel_occupancy(k_enc_write<T, VPL>, C::SMEM, 1);
    const uint64_t wgrid = std::max<uint64_t>(1, std::min<uint64_t>(cdiv(L.nB, kWriteTile),
                                                                    (uint64_t)SZX_WGRIDK * sm_count() * occ_w));
    launch("k_enc_write", s, [&] {
        launch_pdl(k_enc_write<T, VPL>, dim3((unsigned)wgrid), dim3(256), C::SMEM, s,
                   static_cast<const T*>(d_in), p, out);
    });
}

template <typename F>
void dispatch(szx_dtype_t dt, uint32_t b, F&& f);

// Enqueue the whole compression.  Returns SZX_OK or an error.
int enqueue_compress(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                     uint32_t b, void* d_out, uint64_t cap, void* d_ws, uint64_t ws_bytes,
                     uint64_t** d_total_out, cudaStream_t s, uint64_t* user_total = nullptr) {
    int rc = check_compress_args(d_in, dt, n, mode, eb, b, d_out);
    if (rc) return rc;
    if (!have_device()) return SZX_ECUDA;
    if (cap < szx_compress_bound(n, dt, b)) return SZX_ENOSPC;
    const int W = wbytes(dt);
    CLayout L = clayout(n, W, b);
    if (!d_ws || !aligned16(d_ws)) return SZX_EINVAL;
    if (ws_bytes < L.total) return SZX_ENOSPC;
    uint8_t* ws = static_cast<uint8_t*>(d_ws);
    uint8_t* out = static_cast<uint8_t*>(d_out);
    Plan p = make_plan(L, ws, n, dt, mode, eb, b, nullptr);
    if (user_total) p.total = user_total;  // the kernels write the stream length straight there
    *d_total_out = p.total;
    if (n == 0) {
        launch("k_empty_header", s, [&] { k_empty_header<<<1, 1, 0, s>>>(out, dt, mode, b, eb, nullptr, p.total); });
        return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
    }
    cudaMemsetAsync(ws + L.off_keys, 0xFF, 16, s);
    cudaMemsetAsync(ws + L.off_zero, 0, L.zero_bytes, s);
    dispatch(dt, b, [&](auto tag, auto vpl) {
        using T = decltype(tag);
        constexpr int V = decltype(vpl)::value;
        enqueue_stats<T, V>(d_in, p, mode == SZX_REL, s);
        enqueue_encode<T, V>(d_in, p, L, out, s);
    });
    return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
}

template <int V> struct IC { static constexpr int value = V; };
template <typename F>
void dispatch(szx_dtype_t dt, uint32_t b, F&& f) {
    // b = 32 x VPL: a warp owns a block, VPL values per lane
    auto go = [&](auto tag) {
        switch (b) {
            case 32: f(tag, IC<1>()); break;
            case 64: f(tag, IC<2>()); break;
            case 128: f(tag, IC<4>()); break;
            default: f(tag, IC<8>()); break;
        }
    };
    if (dt == SZX_F32) go(float());
    else go(double());
}

int64_t finish_sync(cudaStream_t s, const uint64_t* d_val, uint64_t* out_val) {
    uint64_t* h = pinned_u64();
    if (!h) return SZX_ECUDA;
    if (cudaMemcpyAsync(h, d_val, 8, cudaMemcpyDeviceToHost, s) != cudaSuccess) return SZX_ECUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) return SZX_ECUDA;
    timing_resolve();
    *out_val = h[0];
    return SZX_OK;
}

// ------------------------------------------------------------ decompress layout
// Sized from the shape only (n, b): the number of nonconstant blocks is read
// from the stream header on the device, so the layout covers nNC <= nB.
constexpr uint64_t kMaxDecodeGrid = 2048;  // co-resident CTAs of k_decode_w (slot arrays)

struct DLayout {
    uint64_t nB, nW;
    uint64_t zero_bytes, off_nctile, off_ncpre, off_tbase, total;
};
DLayout dlayout(uint64_t n, uint32_t b) {
    DLayout L{};
    L.nB = cdiv(n, b);
    L.nW = cdiv(L.nB, 32);
    L.zero_bytes = 32 + 16 + 16 + 4 * 8 * kMaxDecodeGrid;  // ctr[8], err, n_nctile, slot_a, res_a, slot_z, res_z
    L.off_nctile = L.zero_bytes;
    L.off_ncpre = al16(L.off_nctile + 4 * L.nW);
    L.off_tbase = al16(L.off_ncpre + 4 * L.nW + 4);
    L.total = al16(L.off_tbase + 8 * (L.nW + 1)) + 256;
    return L;
}

int parse_header(const uint8_t* b, uint64_t nbytes, szx_header_t* h) {
    if (!b || !h || nbytes < 64) return SZX_ECORRUPT;
    if (memcmp(b, "SZX1", 4) != 0 || b[4] != 1 || b[7] != 0) return SZX_ECORRUPT;
    uint64_t q[8];
    memcpy(q, b, 64);
    h->version = b[4];
    h->dtype = b[5];
    h->eb_mode = b[6];
    h->block_size = (uint32_t)(q[1] & 0xFFFFFFFFu);
    h->n = q[2];
    memcpy(&h->eb_user, &q[3], 8);
    memcpy(&h->eb_abs, &q[4], 8);
    h->n_nonconst = q[5];
    h->payload_bytes = q[6];
    if (h->dtype > 1 || h->eb_mode > 1 || !block_ok(h->block_size) || h->n > kMaxN) return SZX_ECORRUPT;
    const uint64_t W = h->dtype ? 8 : 4;
    const uint64_t nB = cdiv(h->n, h->block_size);
    if (h->n_nonconst > nB) return SZX_ECORRUPT;
    const uint64_t maxz = 1 + h->block_size / 4 + W * h->block_size;
    if (h->payload_bytes > h->n_nonconst * maxz) return SZX_ECORRUPT;
    h->stream_bytes = kHeaderBytes + al16(cdiv(nB, 8)) + al16(W * nB) + al16(2 * h->n_nonconst) + h->payload_bytes;
    return SZX_OK;
}

// Only h->n, h->dtype and h->block_size are used on the host; the kernels
// read and validate the content-dependent header fields on the device.
// Reconstructs blocks [kb0, kb1) (kb1 = UINT64_MAX: to the end) into d_out,
// whose element 0 is the first value of block kb0.
int enqueue_decompress(const void* d_in, uint64_t in_bytes, const szx_header_t* h, void* d_out,
                       uint64_t cap, void* d_ws, uint64_t ws_bytes, int32_t** d_err_out, cudaStream_t s,
                       uint64_t kb0 = 0, uint64_t kb1 = UINT64_MAX, const void* d_ref = nullptr,
                       uint64_t* d_qual = nullptr) {
    if (!d_in || !aligned16(d_in) || !h) return SZX_EINVAL;
    if (h->dtype > 1 || !block_ok(h->block_size) || h->n > kMaxN) return SZX_EINVAL;
    if (in_bytes < kHeaderBytes) return SZX_ECORRUPT;
    const uint64_t W = h->dtype ? 8 : 4;
    const uint64_t nBh = cdiv(h->n, h->block_size);
    if (kb1 > nBh) kb1 = nBh;
    if (kb0 > kb1) return SZX_EINVAL;
    const uint64_t e0 = kb0 * h->block_size, e1 = std::min<uint64_t>(h->n, kb1 * h->block_size);
    const uint64_t n_out = e1 - e0;
    if (cap < W * n_out) return SZX_ENOSPC;
    if (n_out && (!d_out || !aligned16(d_out))) return SZX_EINVAL;
    if (d_ref && (!aligned16(d_ref) || !d_qual)) return SZX_EINVAL;
    DLayout L = dlayout(h->n, h->block_size);
    if (!d_ws || !aligned16(d_ws)) return SZX_EINVAL;
    if (ws_bytes < L.total) return SZX_ENOSPC;
    uint8_t* ws = static_cast<uint8_t*>(d_ws);
    DPlan p{};
    p.n = h->n; p.nB = L.nB; p.nW = L.nW;
    p.kb0 = kb0; p.kb1 = kb1;
    p.nWi = cdiv(kb1, 32); p.t_lo = kb0 / 32;
    p.in_bytes = in_bytes;
    p.off_mu = kHeaderBytes + al16(cdiv(L.nB, 8));
    p.b = h->block_size;
    p.dtype = h->dtype;
    p.ctr = reinterpret_cast<uint32_t*>(ws);
    p.err = reinterpret_cast<int32_t*>(ws + 32);
    p.n_nctile = reinterpret_cast<uint32_t*>(ws + 48);
    p.slot_a = reinterpret_cast<uint64_t*>(ws + 64);
    p.res_a = p.slot_a + kMaxDecodeGrid;
    p.slot_z = p.res_a + kMaxDecodeGrid;
    p.res_z = p.slot_z + kMaxDecodeGrid;
    p.nctile = reinterpret_cast<uint32_t*>(ws + L.off_nctile);
    p.ncpre = reinterpret_cast<uint32_t*>(ws + L.off_ncpre);
    p.tbase = reinterpret_cast<uint64_t*>(ws + L.off_tbase);
    *d_err_out = p.err;
    cudaMemsetAsync(ws, 0, L.zero_bytes, s);
    if (n_out == 0) return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
    const uint8_t* in = static_cast<const uint8_t*>(d_in);
    // the kernels index the output by stream element; shift the base so that
    // element e0 lands on d_out[0] (only elements of [e0, e1) are stored)
    const uintptr_t ybase = reinterpret_cast<uintptr_t>(d_out) - W * e0;
    if (d_ref) {
        p.ref = reinterpret_cast<const void*>(reinterpret_cast<uintptr_t>(d_ref) - W * e0);
        p.qual = d_qual;
    }
    dispatch((szx_dtype_t)h->dtype, h->block_size, [&](auto tag, auto vpl) {
        using T = decltype(tag);
        constexpr int V = decltype(vpl)::value;
        // persistent, co-resident grid (index phase, grid barrier, then one
        // warp per 32-block tile): launched cooperatively, so the driver
        // either makes every CTA resident at once or rejects the launch (it
        // never hangs when fewer SMs are available, e.g. under MPS limits or
        // beside a concurrent kernel)
        auto go = [&](auto kern, const char* name) {
            const int occ = kernel_occupancy(kern, DecWCfg<T, V>::SMEM, 1);
            const uint64_t gcap = std::min<uint64_t>((uint64_t)sm_count() * occ, kMaxDecodeGrid);
            // small arrays: split each nonconstant tile into 2 or 4 work items so
            // that every decode warp of the full grid gets a few (latency hiding)
            const uint64_t want_items = (uint64_t)SZX_DITEMS * gcap * (DecWCfg<T, V>::NWARP - DecWCfg<T, V>::FILLW);
            p.split = p.nWi >= want_items ? 1u : (p.nWi * 2 >= want_items ? 2u : 4u);
            if (SZX_DSPLIT) p.split = SZX_DSPLIT;
            // dense float32 b = 128 streams: the thread-serial tile decoder (a
            // performance choice only; the device validates the stream itself)
            // (at least SZX_DTS_MINT tiles per warp of the grid: a lane-per-block tile takes
            // a warp as long as a whole tile, so few tiles per warp leave a long tail --
            // Hurricane's 6,103 tiles decode faster with the half-warp form)
            p.ts = (SZX_DTS && sizeof(T) == 4 && V == 4 && !d_ref && p.split == 1 && kb0 == 0 &&
                    kb1 == L.nB && 4 * h->n_nonconst >= 3 * L.nB &&
                    p.nWi >= (uint64_t)SZX_DTS_MINT * gcap * DecWCfg<T, V>::NWARP) ? 1u : 0u;
            uint64_t grid = cdiv(p.nWi * p.split, 8);
            if (grid > gcap) grid = gcap;
            // index CTAs: at most one per SM, and at most one 256-tile chunk each
            // (fewer arrivals at the two grid-wide prefixes)
            p.n_icta = (uint32_t)std::min<uint64_t>(std::min<uint64_t>(grid, (uint64_t)SZX_ICTA_PER_SM * sm_count()),
                                                    SZX_ICTA_CHUNK ? cdiv(p.nWi, kIndexChunk) : grid);
            launch(name, s, [&] {
                launch_coop(kern, dim3((unsigned)grid), dim3(256), DecWCfg<T, V>::SMEM, s, p, in,
                            reinterpret_cast<T*>(ybase));
            });
        };
        if (d_ref) go(k_decode_w<T, V, true>, "k_decode_q");
        else go(k_decode_w<T, V>, "k_decode");
    });
    return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
}

int read_device_bytes(const void* d_src, void* h_dst, uint64_t nbytes, cudaStream_t s) {
    if (cudaMemcpyAsync(h_dst, d_src, nbytes, cudaMemcpyDeviceToHost, s) != cudaSuccess) return SZX_ECUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) return SZX_ECUDA;
    return SZX_OK;
}

int64_t decompress_one_sync(const void* d_in, uint64_t in_bytes, const szx_header_t* h, void* d_out,
                            uint64_t cap, void* d_ws, uint64_t ws_bytes, cudaStream_t s) {
    int32_t* d_err = nullptr;
    int rc = enqueue_decompress(d_in, in_bytes, h, d_out, cap, d_ws, ws_bytes, &d_err, s);
    if (rc) return rc;
    int32_t err = 0;
    if (read_device_bytes(d_err, &err, 4, s)) return SZX_ECUDA;
    timing_resolve();
    return err ? err : (int64_t)h->n;
}

// ------------------------------------------------------------ stream sets
// An SZX1 stream is one part; an SZXC container (DESIGN.md s.4) is P parts,
// part i holding elements [first_i, first_i + n_i) of the array.
struct Part {
    szx_header_t h;
    uint64_t off, len, first;
};

int parse_parts(const void* d_in, uint64_t in_bytes, cudaStream_t s, std::vector<Part>& parts, uint64_t* total) {
    uint8_t hb[64];
    if (read_device_bytes(d_in, hb, 64, s)) return SZX_ECUDA;
    parts.clear();
    if (memcmp(hb, "SZXC", 4) == 0) {
        uint32_t P, ver;
        uint64_t total_n;
        memcpy(&ver, hb + 4, 4);
        memcpy(&P, hb + 8, 4);
        memcpy(&total_n, hb + 16, 8);
        if (ver != 1 || P == 0 || 32 + 32ull * P > in_bytes) return SZX_ECORRUPT;
        std::vector<uint8_t> tab(32ull * P);
        if (read_device_bytes(static_cast<const uint8_t*>(d_in) + 32, tab.data(), tab.size(), s)) return SZX_ECUDA;
        uint64_t expect = 0;
        for (uint32_t i = 0; i < P; i++) {
            uint64_t e[4];
            memcpy(e, tab.data() + 32ull * i, 32);
            if (e[0] != expect || e[2] % 16 || e[2] > in_bytes || e[3] > in_bytes - e[2] || e[3] < 64)
                return SZX_ECORRUPT;
            uint8_t sh[64];
            if (read_device_bytes(static_cast<const uint8_t*>(d_in) + e[2], sh, 64, s)) return SZX_ECUDA;
            Part pt;
            if (parse_header(sh, 64, &pt.h) || pt.h.n != e[1]) return SZX_ECORRUPT;
            if (!parts.empty() && pt.h.dtype != parts[0].h.dtype) return SZX_ECORRUPT;
            pt.off = e[2]; pt.len = e[3]; pt.first = e[0];
            parts.push_back(pt);
            expect += e[1];
        }
        if (expect != total_n) return SZX_ECORRUPT;
        *total = total_n;
    } else {
        Part pt;
        if (parse_header(hb, 64, &pt.h)) return SZX_ECORRUPT;
        pt.off = 0; pt.len = in_bytes; pt.first = 0;
        parts.push_back(pt);
        *total = pt.h.n;
    }
    return SZX_OK;
}

// Decode global blocks [g0, g1) of a stream or container into d_out (element
// 0 = first value of block g0).  Every part's kernel is enqueued back to back
// (each with its own workspace slice), then one synchronisation reads all
// status words.  ranged: block indices are global over the container, which
// requires every part to start on a block boundary of one common block size.
// Quality accumulators {max err bits, sse, dkey(min), ~dkey(max)} -> doubles
// {max |x - x'|, sum (x - x')^2, min finite x, max finite x}.
void qual_finish(const uint64_t* raw, double* out) {
    memcpy(&out[0], &raw[0], 8);
    memcpy(&out[1], &raw[1], 8);
    const uint64_t a = raw[2], b = ~raw[3];
    const uint64_t ba = dkey_inv(a), bb = dkey_inv(b);
    double dmn, dmx;
    memcpy(&dmn, &ba, 8);
    memcpy(&dmx, &bb, 8);
    out[2] = raw[2] == ~0ull ? INFINITY : dmn;
    out[3] = raw[3] == ~0ull ? -INFINITY : dmx;
}

int qual_init(uint64_t* d_qual, cudaStream_t s) {
    if (cudaMemsetAsync(d_qual, 0, 16, s) != cudaSuccess) return SZX_ECUDA;
    if (cudaMemsetAsync(d_qual + 2, 0xFF, 16, s) != cudaSuccess) return SZX_ECUDA;
    return SZX_OK;
}

int64_t decode_range(const void* d_in, uint64_t in_bytes, uint64_t g0, uint64_t g1, void* d_out, uint64_t cap,
                     cudaStream_t s, bool ranged, const void* d_ref = nullptr, double* h_qual = nullptr) {
    if (!d_in || in_bytes < 64) return SZX_ECORRUPT;
    if (!have_device()) return SZX_ECUDA;
    std::vector<Part> parts;
    uint64_t total = 0;
    int rc = parse_parts(d_in, in_bytes, s, parts, &total);
    if (rc) return rc;
    const uint64_t W = parts[0].h.dtype ? 8 : 4;
    const uint64_t b = parts[0].h.block_size;
    if (ranged)
        for (auto& pt : parts)
            if (pt.h.block_size != b || pt.first % b) return SZX_EINVAL;
    const uint64_t nBg = cdiv(total, b);
    if (g1 > nBg) g1 = nBg;
    if (g0 > g1) g0 = g1;  // a range starting past the end is empty
    const uint64_t e0 = ranged ? g0 * b : 0, e1 = ranged ? std::min(total, g1 * b) : total;
    const uint64_t n_out = e1 > e0 ? e1 - e0 : 0;
    if (cap < W * n_out) return SZX_ENOSPC;
    if (d_ref && (!h_qual || !aligned16(d_ref))) return SZX_EINVAL;
    if (n_out == 0) {
        if (h_qual) { const uint64_t z[4] = {0, 0, ~0ull, ~0ull}; qual_finish(z, h_qual); }
        return 0;
    }
    // per part: local block range, output position, workspace slice
    struct Job { size_t i; uint64_t kb0, kb1, out_el, ws_off; };
    std::vector<Job> jobs;
    uint64_t wsb = 0;
    for (size_t i = 0; i < parts.size(); i++) {
        const Part& pt = parts[i];
        const uint64_t pb = pt.h.block_size, nBp = cdiv(pt.h.n, pb);
        uint64_t kb0 = 0, kb1 = nBp;
        if (ranged) {
            const uint64_t f = pt.first / b;
            if (f + nBp <= g0 || f >= g1) continue;
            kb0 = g0 > f ? g0 - f : 0;
            kb1 = std::min(nBp, g1 - f);
        }
        if (pt.h.n == 0) continue;
        jobs.push_back({i, kb0, kb1, pt.first + kb0 * pb - e0, wsb});
        wsb += al16(szx_decompress_workspace_bytes(&pt.h));
    }
    void* ws = nullptr;
    keep_pool_memory();
    const uint64_t q_off = wsb;
    wsb += 32;
    if (cudaMallocAsync(&ws, std::max<uint64_t>(wsb, 16), s) != cudaSuccess) { cudaGetLastError(); return SZX_ENOMEM; }
    uint64_t* d_qual = reinterpret_cast<uint64_t*>(static_cast<uint8_t*>(ws) + q_off);
    std::vector<int32_t*> errs;
    int64_t r = 0;
    if (d_ref) r = qual_init(d_qual, s);
    for (const Job& j : jobs) {
        const Part& pt = parts[j.i];
        int32_t* d_err = nullptr;
        const uint64_t wsz = al16(szx_decompress_workspace_bytes(&pt.h));
        rc = enqueue_decompress(static_cast<const uint8_t*>(d_in) + pt.off, pt.len, &pt.h,
                                static_cast<uint8_t*>(d_out) + W * j.out_el, cap - W * j.out_el,
                                static_cast<uint8_t*>(ws) + j.ws_off, wsz, &d_err, s, j.kb0, j.kb1,
                                d_ref ? static_cast<const uint8_t*>(d_ref) + W * j.out_el : nullptr,
                                d_ref ? d_qual : nullptr);
        if (rc) { r = rc; break; }
        errs.push_back(d_err);
    }
    if (r == 0 && cudaStreamSynchronize(s) != cudaSuccess) r = SZX_ECUDA;
    for (size_t i = 0; i < errs.size() && r == 0; i++) {
        int32_t e = 0;
        if (cudaMemcpy(&e, errs[i], 4, cudaMemcpyDeviceToHost) != cudaSuccess) r = SZX_ECUDA;
        else if (e) r = e;
    }
    if (r == 0 && d_ref) {
        uint64_t raw[4];
        if (cudaMemcpy(raw, d_qual, 32, cudaMemcpyDeviceToHost) != cudaSuccess) r = SZX_ECUDA;
        else qual_finish(raw, h_qual);
    }
    timing_resolve();
    cudaFreeAsync(ws, s);
    return r < 0 ? r : (int64_t)n_out;
}

}  // namespace

// ====================================================================== C ABI
extern "C" {

uint64_t szx_compress_bound(uint64_t n, szx_dtype_t dt, uint32_t b) {
    if (b == 0) return 0;
    const uint64_t W = wbytes(dt);
    const uint64_t nB = cdiv(n, b);
    return kHeaderBytes + al16(cdiv(nB, 8)) + al16(W * nB) + al16(2 * nB) + nB + cdiv(n, 4) + nB + W * n;
}

uint64_t szx_compress_workspace_bytes(uint64_t n, szx_dtype_t dt, uint32_t b) {
    if (!block_ok(b)) return 0;
    return clayout(n, wbytes(dt), b).total;
}

uint64_t szx_decompress_workspace_bytes(const szx_header_t* h) {
    if (!h || !block_ok(h->block_size)) return 0;
    return dlayout(h->n, h->block_size).total;
}

int szx_compress_async(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                       uint32_t b, void* d_out, uint64_t cap, void* d_ws, uint64_t ws_bytes,
                       uint64_t* d_total_bytes, void* stream) {
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    uint64_t* d_tot = nullptr;
    return enqueue_compress(d_in, dt, n, mode, eb, b, d_out, cap, d_ws, ws_bytes, &d_tot, s, d_total_bytes);
}

int64_t szx_compress_ws(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                        uint32_t b, void* d_out, uint64_t cap, void* d_ws, uint64_t ws_bytes, void* stream) {
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    uint64_t* d_tot = nullptr;
    int rc = enqueue_compress(d_in, dt, n, mode, eb, b, d_out, cap, d_ws, ws_bytes, &d_tot, s);
    if (rc) return rc;
    uint64_t total = 0;
    if (finish_sync(s, d_tot, &total)) return SZX_ECUDA;
    return (int64_t)total;
}

int64_t szx_compress(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                     uint32_t b, void* d_out, uint64_t cap, void* stream) {
    int rc = check_compress_args(d_in, dt, n, mode, eb, b, d_out);
    if (rc) return rc;
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const uint64_t wsb = szx_compress_workspace_bytes(n, dt, b);
    void* ws = nullptr;
    keep_pool_memory();
    if (cudaMallocAsync(&ws, wsb, s) != cudaSuccess) { cudaGetLastError(); return SZX_ENOMEM; }
    int64_t r = szx_compress_ws(d_in, dt, n, mode, eb, b, d_out, cap, ws, wsb, stream);
    cudaFreeAsync(ws, s);
    return r;
}

int szx_read_header(const void* h_bytes, uint64_t nbytes, szx_header_t* out) {
    return parse_header(static_cast<const uint8_t*>(h_bytes), nbytes, out);
}

int szx_decompress_async(const void* d_in, uint64_t in_bytes, const szx_header_t* h, void* d_out,
                         uint64_t cap, void* d_ws, uint64_t ws_bytes, int32_t* d_status, void* stream) {
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    int32_t* d_err = nullptr;
    int rc = enqueue_decompress(d_in, in_bytes, h, d_out, cap, d_ws, ws_bytes, &d_err, s);
    if (rc) return rc;
    if (d_status && d_status != d_err)
        if (cudaMemcpyAsync(d_status, d_err, 4, cudaMemcpyDeviceToDevice, s) != cudaSuccess) return SZX_ECUDA;
    return SZX_OK;
}

int64_t szx_decompress_ws(const void* d_in, uint64_t in_bytes, void* d_out, uint64_t cap, void* d_ws,
                          uint64_t ws_bytes, void* stream) {
    if (!d_in || in_bytes < 64) return SZX_ECORRUPT;
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    uint8_t hb[64];
    if (read_device_bytes(d_in, hb, 64, s)) return SZX_ECUDA;
    szx_header_t h;
    if (parse_header(hb, 64, &h)) return SZX_ECORRUPT;
    return decompress_one_sync(d_in, in_bytes, &h, d_out, cap, d_ws, ws_bytes, s);
}

int64_t szx_decompress(const void* d_in, uint64_t in_bytes, void* d_out, uint64_t cap, void* stream) {
    return decode_range(d_in, in_bytes, 0, UINT64_MAX, d_out, cap, static_cast<cudaStream_t>(stream), false);
}

int64_t szx_decompress_quality(const void* d_in, uint64_t in_bytes, const void* d_ref, void* d_out, uint64_t cap,
                               double* h_qual, void* stream) {
    if (!d_ref || !h_qual) return SZX_EINVAL;
    return decode_range(d_in, in_bytes, 0, UINT64_MAX, d_out, cap, static_cast<cudaStream_t>(stream), false, d_ref,
                        h_qual);
}

int szx_decompress_quality_async(const void* d_in, uint64_t in_bytes, const szx_header_t* h, const void* d_ref,
                                 void* d_out, uint64_t cap, void* d_ws, uint64_t ws_bytes, uint64_t* d_qual,
                                 int32_t* d_status, void* stream) {
    if (!have_device()) return SZX_ECUDA;
    if (!d_ref || !d_qual) return SZX_EINVAL;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    int rc = qual_init(d_qual, s);
    if (rc) return rc;
    int32_t* d_err = nullptr;
    rc = enqueue_decompress(d_in, in_bytes, h, d_out, cap, d_ws, ws_bytes, &d_err, s, 0, UINT64_MAX, d_ref, d_qual);
    if (rc) return rc;
    if (d_status && d_status != d_err)
        if (cudaMemcpyAsync(d_status, d_err, 4, cudaMemcpyDeviceToDevice, s) != cudaSuccess) return SZX_ECUDA;
    return SZX_OK;
}

void szx_quality_finish(const uint64_t* raw, double* out) { qual_finish(raw, out); }

int64_t szx_decompress_blocks(const void* d_in, uint64_t in_bytes, uint64_t first_block, uint64_t n_blocks,
                              void* d_out, uint64_t cap, void* stream) {
    const uint64_t end = n_blocks > UINT64_MAX - first_block ? UINT64_MAX : first_block + n_blocks;
    return decode_range(d_in, in_bytes, first_block, end, d_out, cap, static_cast<cudaStream_t>(stream), true);
}

int64_t szx_compress_host(const void* h_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                          uint32_t b, void* h_out, uint64_t cap, void* stream) {
    if (!h_out || (n && !h_in)) return SZX_EINVAL;
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const uint64_t W = wbytes(dt), bound = szx_compress_bound(n, dt, b);
    if (!block_ok(b)) return SZX_EINVAL;
    void *d_in = nullptr, *d_out = nullptr;
    keep_pool_memory();
    if (cudaMallocAsync(&d_in, W * n + 16, s) != cudaSuccess) { cudaGetLastError(); return SZX_ENOMEM; }
    if (cudaMallocAsync(&d_out, bound, s) != cudaSuccess) { cudaGetLastError(); cudaFreeAsync(d_in, s); return SZX_ENOMEM; }
    int64_t r = SZX_ECUDA;
    if (!n || cudaMemcpyAsync(d_in, h_in, W * n, cudaMemcpyHostToDevice, s) == cudaSuccess) {
        r = szx_compress(d_in, dt, n, mode, eb, b, d_out, bound, stream);
        if (r >= 0) {
            if ((uint64_t)r > cap) r = SZX_ENOSPC;
            else if (read_device_bytes(d_out, h_out, (uint64_t)r, s)) r = SZX_ECUDA;
        }
    }
    cudaFreeAsync(d_in, s);
    cudaFreeAsync(d_out, s);
    return r;
}

int64_t szx_decompress_host(const void* h_in, uint64_t in_bytes, void* h_out, uint64_t cap, void* stream) {
    if (!h_in || in_bytes < 64) return SZX_ECORRUPT;
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    void* d_in = nullptr;
    keep_pool_memory();
    if (cudaMallocAsync(&d_in, in_bytes, s) != cudaSuccess) { cudaGetLastError(); return SZX_ENOMEM; }
    int64_t r = SZX_ECUDA;
    if (cudaMemcpyAsync(d_in, h_in, in_bytes, cudaMemcpyHostToDevice, s) == cudaSuccess) {
        // the output size comes from the header(s); decode into a device buffer
        uint64_t total = 0, W = 4;
        const uint8_t* hb = static_cast<const uint8_t*>(h_in);
        if (memcmp(hb, "SZXC", 4) == 0) {
            memcpy(&total, hb + 16, 8);
            if (in_bytes >= 32 + 32 + 64) {
                uint64_t off;
                memcpy(&off, hb + 32 + 16, 8);
                if (off <= in_bytes && in_bytes - off >= 64) W = hb[off + 5] ? 8 : 4;
            }
        } else {
            szx_header_t h;
            if (parse_header(hb, in_bytes, &h)) { cudaFreeAsync(d_in, s); return SZX_ECORRUPT; }
            total = h.n;
            W = h.dtype ? 8 : 4;
        }
        if (W * total > cap) { cudaFreeAsync(d_in, s); return SZX_ENOSPC; }
        void* d_out = nullptr;
        if (cudaMallocAsync(&d_out, W * total + 16, s) != cudaSuccess) { cudaGetLastError(); cudaFreeAsync(d_in, s); return SZX_ENOMEM; }
        r = szx_decompress(d_in, in_bytes, d_out, W * total + 16, stream);
        if (r >= 0 && read_device_bytes(d_out, h_out, W * (uint64_t)r, s)) r = SZX_ECUDA;
        cudaFreeAsync(d_out, s);
    }
    cudaFreeAsync(d_in, s);
    return r;
}

int szx_local_range(const void* d_in, szx_dtype_t dt, uint64_t n, uint32_t b, uint64_t* d_range_keys,
                    void* d_ws, uint64_t ws_bytes, void* stream) {
    if (dt != SZX_F32 && dt != SZX_F64) return SZX_EINVAL;
    if (!block_ok(b) || !d_range_keys || (n && (!d_in || !aligned16(d_in))) || n > kMaxN) return SZX_EINVAL;
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    cudaMemsetAsync(d_range_keys, 0xFF, 16, s);
    if (n == 0) return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
    // One pass over the shard: block statistics into the workspace (consumed
    // by szx_compress_shard_async) and the local finite range.
    CLayout L = clayout(n, wbytes(dt), b);
    if (!d_ws || !aligned16(d_ws) || ws_bytes < L.total) return SZX_ENOSPC;
    Plan p = make_plan(L, static_cast<uint8_t*>(d_ws), n, dt, SZX_REL, 0.0, b, d_range_keys);
    dispatch(dt, b, [&](auto tag, auto vpl) {
        using T = decltype(tag);
        enqueue_stats<T, decltype(vpl)::value>(d_in, p, 1, s);
    });
    return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
}

int szx_compress_shard_async(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                             const uint64_t* d_range_keys, uint32_t b, void* d_out, uint64_t cap,
                             void* d_ws, uint64_t ws_bytes, uint64_t* d_total_bytes, void* stream) {
    int rc = check_compress_args(d_in, dt, n, mode, eb, b, d_out);
    if (rc) return rc;
    if (mode == SZX_REL && !d_range_keys) return SZX_EINVAL;
    if (!have_device()) return SZX_ECUDA;
    if (cap < szx_compress_bound(n, dt, b)) return SZX_ENOSPC;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const int W = wbytes(dt);
    CLayout L = clayout(n, W, b);
    if (!d_ws || !aligned16(d_ws) || ws_bytes < L.total) return SZX_ENOSPC;
    uint8_t* ws = static_cast<uint8_t*>(d_ws);
    uint8_t* out = static_cast<uint8_t*>(d_out);
    Plan p = make_plan(L, ws, n, dt, mode, eb, b, mode == SZX_REL ? d_range_keys : nullptr);
    if (n == 0) {
        // REL with an empty shard still carries the global bound in its header
        launch("k_empty_header", s, [&] { k_empty_header<<<1, 1, 0, s>>>(out, dt, mode, b, eb, mode == SZX_REL ? d_range_keys : nullptr, p.total); });
    } else {
        // block statistics were produced by szx_local_range on this workspace
        cudaMemsetAsync(ws + L.off_zero, 0, L.zero_bytes, s);
        dispatch(dt, b, [&](auto tag, auto vpl) {
            using T = decltype(tag);
            enqueue_encode<T, decltype(vpl)::value>(d_in, p, L, out, s);
        });
    }
    if (d_total_bytes && cudaMemcpyAsync(d_total_bytes, p.total, 8, cudaMemcpyDeviceToDevice, s) != cudaSuccess)
        return SZX_ECUDA;
    return cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
}

}  // extern "C"

// keys [key(min), ~key(max)] -> doubles (min, max); no finite value -> (+Inf, -Inf)
__global__ void k_keys_to_minmax(const uint64_t* keys, double* mm) {
    const uint64_t a = keys[0], c = keys[1];
    mm[0] = a == ~0ull ? __longlong_as_double(0x7FF0000000000000ll) : __longlong_as_double((long long)dkey_inv(a));
    mm[1] = c == ~0ull ? __longlong_as_double((long long)0xFFF0000000000000ull)
                       : __longlong_as_double((long long)dkey_inv(~c));
}

extern "C" {

int szx_local_minmax(const void* d_in, szx_dtype_t dt, uint64_t n, double* d_minmax2, void* stream) {
    if (dt != SZX_F32 && dt != SZX_F64) return SZX_EINVAL;
    if (!d_minmax2 || (n && (!d_in || !aligned16(d_in))) || n > kMaxN) return SZX_EINVAL;
    if (!have_device()) return SZX_ECUDA;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const uint64_t wsb = std::max<uint64_t>(szx_compress_workspace_bytes(n, dt, 128), 16) + 16;
    void* ws = nullptr;
    keep_pool_memory();
    if (cudaMallocAsync(&ws, wsb, s) != cudaSuccess) { cudaGetLastError(); return SZX_ENOMEM; }
    uint64_t* keys = reinterpret_cast<uint64_t*>(static_cast<uint8_t*>(ws) + wsb - 16);
    int rc = szx_local_range(d_in, dt, n, 128, keys, ws, wsb - 16, stream);
    if (rc == SZX_OK) {
        launch("k_keys_to_minmax", s, [&] { k_keys_to_minmax<<<1, 1, 0, s>>>(keys, d_minmax2); });
        rc = cudaGetLastError() == cudaSuccess ? SZX_OK : SZX_ECUDA;
    }
    cudaFreeAsync(ws, s);
    return rc;
}

int64_t szx_compress_shard(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb_user,
                           const double* d_eb_abs, uint32_t b, void* d_out, uint64_t cap, void* stream) {
    int rc = check_compress_args(d_in, dt, n, mode, eb_user, b, d_out);
    if (rc) return rc;
    if (!d_eb_abs) return SZX_EINVAL;
    if (!have_device()) return SZX_ECUDA;
    if (cap < szx_compress_bound(n, dt, b)) return SZX_ENOSPC;
    cudaStream_t s = static_cast<cudaStream_t>(stream);
    const int W = wbytes(dt);
    CLayout L = clayout(n, W, b);
    void* wsv = nullptr;
    keep_pool_memory();
    if (cudaMallocAsync(&wsv, L.total, s) != cudaSuccess) { cudaGetLastError(); return SZX_ENOMEM; }
    uint8_t* ws = static_cast<uint8_t*>(wsv);
    uint8_t* out = static_cast<uint8_t*>(d_out);
    Plan p = make_plan(L, ws, n, dt, mode, eb_user, b, nullptr);
    p.eb_in = d_eb_abs;
    if (n == 0) {
        launch("k_empty_header", s, [&] {
            k_empty_header<<<1, 1, 0, s>>>(out, dt, mode, b, eb_user, nullptr, p.total, d_eb_abs);
        });
    } else {
        cudaMemsetAsync(ws + L.off_keys, 0xFF, 16, s);
        cudaMemsetAsync(ws + L.off_zero, 0, L.zero_bytes, s);
        dispatch(dt, b, [&](auto tag, auto vpl) {
            using T = decltype(tag);
            constexpr int V = decltype(vpl)::value;
            enqueue_stats<T, V>(d_in, p, 0, s);
            enqueue_encode<T, V>(d_in, p, L, out, s);
        });
    }
    int64_t r = SZX_ECUDA;
    uint64_t total = 0;
    if (cudaGetLastError() == cudaSuccess && finish_sync(s, p.total, &total) == SZX_OK) r = (int64_t)total;
    cudaFreeAsync(wsv, s);
    return r;
}

// ------------------------------------------------------------ dump / load
// Single-box analogue of the paper's data dumping / loading experiment
// (Fig. 16): a device array goes to host memory as an SZXC
// container of P block-range shards (DESIGN.md s.8), compression of shard
// p+1 overlapping the device-to-host copy of shard p; loading copies shard
// q+1 to the device while shard q decodes.

__global__ void k_keys_min(const uint64_t* keys, uint32_t P, uint64_t* out) {
    uint64_t a = ~0ull, c = ~0ull;
    for (uint32_t i = 0; i < P; i++) {
        a = keys[2 * i] < a ? keys[2 * i] : a;
        c = keys[2 * i + 1] < c ? keys[2 * i + 1] : c;
    }
    out[0] = a;
    out[1] = c;
}

namespace {
struct DumpRes {  // device scratch (stream-ordered pool, kept between calls) and the copy stream / events
    std::vector<void*> dev;
    std::vector<cudaEvent_t> events;
    cudaStream_t s = nullptr, s2 = nullptr;
    ~DumpRes() {
        if (s2) cudaStreamSynchronize(s2);
        for (auto p : dev) cudaFreeAsync(p, s);
        if (s) cudaStreamSynchronize(s);
        for (auto e : events) cudaEventDestroy(e);
        if (s2) cudaStreamDestroy(s2);
    }
    bool init(cudaStream_t st) {
        s = st;
        keep_pool_memory();
        return cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking) == cudaSuccess;
    }
    void* dalloc(uint64_t bytes) {
        void* p = nullptr;
        if (cudaMallocAsync(&p, bytes ? bytes : 16, s) != cudaSuccess) { cudaGetLastError(); return nullptr; }
        dev.push_back(p);
        return p;
    }
    cudaEvent_t event() {
        cudaEvent_t e = nullptr;
        if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) return nullptr;
        events.push_back(e);
        return e;
    }
};
// pinned host slots for the shard sizes (per calling thread, grown on demand, kept)
uint64_t* pinned_sizes(uint32_t P) {
    thread_local uint64_t* buf = nullptr;
    thread_local uint32_t cap = 0;
    if (P > cap) {
        if (buf) cudaFreeHost(buf);
        buf = nullptr;
        cap = 0;
        if (cudaMallocHost(&buf, 8ull * P) != cudaSuccess) return nullptr;
        cap = P;
    }
    return buf;
}
}  // namespace

int64_t szx_dump_host(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb, uint32_t b,
                      uint32_t parts, void* h_out, uint64_t h_cap, void* stream) {
    int rc = check_compress_args(d_in, dt, n, mode, eb, b, d_in);
    if (rc) return rc;
    if (!h_out || parts == 0) return SZX_EINVAL;
    if (!have_device()) return SZX_ECUDA;
    const uint64_t W = wbytes(dt), nB = cdiv(n, b);
    const uint32_t P = (uint32_t)std::max<uint64_t>(1, std::min<uint64_t>(parts, std::max<uint64_t>(nB, 1)));
    std::vector<uint64_t> e0(P), np(P);
    uint64_t nmax = 0;
    for (uint32_t q = 0; q < P; q++) {  // shard q: blocks [q nB / P, (q+1) nB / P)
        const uint64_t b0 = nB * q / P, b1 = nB * (q + 1) / P;
        e0[q] = b0 * b;
        np[q] = std::min<uint64_t>(n, b1 * b) - std::min<uint64_t>(n, b0 * b);
        nmax = std::max(nmax, np[q]);
    }
    const uint64_t head = 32 + 32ull * P;
    if (h_cap < head) return SZX_ENOSPC;
    DumpRes R;
    if (!R.init(static_cast<cudaStream_t>(stream))) return SZX_ECUDA;
    cudaStream_t s = R.s, s2 = R.s2;
    std::vector<void*> ws(P);
    std::vector<uint64_t> wsb(P);
    for (uint32_t q = 0; q < P; q++) {
        wsb[q] = std::max<uint64_t>(szx_compress_workspace_bytes(np[q], dt, b), 16);
        if (!(ws[q] = R.dalloc(wsb[q]))) return SZX_ENOMEM;
    }
    uint64_t* keys = static_cast<uint64_t*>(R.dalloc(16ull * P + 16));
    uint64_t* totals = static_cast<uint64_t*>(R.dalloc(8ull * P));
    const uint64_t cap = szx_compress_bound(nmax, dt, b);
    void* buf[2] = {R.dalloc(cap), R.dalloc(cap)};
    uint64_t* hsz = pinned_sizes(P);
    if (!hsz) return SZX_ENOMEM;
    if (!keys || !totals || !buf[0] || !buf[1]) return SZX_ENOMEM;
    const uint8_t* in = static_cast<const uint8_t*>(d_in);
    // pass 1: block statistics and the local ranges of every shard, then the global range
    for (uint32_t q = 0; q < P; q++) {
        rc = szx_local_range(in + W * e0[q], dt, np[q], b, keys + 2 * q, ws[q], wsb[q], s);
        if (rc) return rc;
    }
    uint64_t* gkeys = keys + 2 * P;
    k_keys_min<<<1, 1, 0, s>>>(keys, P, gkeys);
    // pass 2: shard q compresses on s while shard q-1 is copied out on s2
    cudaEvent_t done[2] = {R.event(), R.event()}, copied[2] = {R.event(), R.event()};
    uint8_t* ho = static_cast<uint8_t*>(h_out);
    uint64_t pos = al16(head);
    std::vector<uint64_t> off(P), sz(P);
    auto copy_out = [&](uint32_t q) -> int {
        if (cudaEventSynchronize(done[q & 1]) != cudaSuccess) return SZX_ECUDA;
        sz[q] = hsz[q];
        off[q] = pos;
        if (pos + sz[q] > h_cap) return SZX_ENOSPC;
        cudaStreamWaitEvent(s2, done[q & 1], 0);
        if (cudaMemcpyAsync(ho + pos, buf[q & 1], sz[q], cudaMemcpyDeviceToHost, s2) != cudaSuccess) return SZX_ECUDA;
        cudaEventRecord(copied[q & 1], s2);
        const uint64_t end = pos + sz[q];
        pos = q + 1 < P ? al16(end) : end;
        if (pos > h_cap) return SZX_ENOSPC;
        memset(ho + end, 0, pos - end);  // zero padding between shard streams
        return SZX_OK;
    };
    for (uint32_t q = 0; q < P; q++) {
        if (q >= 2) cudaStreamWaitEvent(s, copied[q & 1], 0);  // its buffer's previous copy is done
        rc = szx_compress_shard_async(in + W * e0[q], dt, np[q], mode, eb, gkeys, b, buf[q & 1], cap, ws[q], wsb[q],
                                      totals + q, s);
        if (rc) return rc;
        cudaMemcpyAsync(hsz + q, totals + q, 8, cudaMemcpyDeviceToHost, s);
        cudaEventRecord(done[q & 1], s);
        if (q >= 1 && (rc = copy_out(q - 1))) return rc;
    }
    if ((rc = copy_out(P - 1))) return rc;
    if (cudaStreamSynchronize(s2) != cudaSuccess) return SZX_ECUDA;
    // container header and shard table
    memset(ho, 0, al16(head));
    memcpy(ho, "SZXC", 4);
    const uint32_t ver = 1, zero = 0;
    memcpy(ho + 4, &ver, 4);
    memcpy(ho + 8, &P, 4);
    memcpy(ho + 12, &zero, 4);
    memcpy(ho + 16, &n, 8);
    for (uint32_t q = 0; q < P; q++) {
        const uint64_t e[4] = {e0[q], np[q], off[q], sz[q]};
        memcpy(ho + 32 + 32ull * q, e, 32);
    }
    timing_resolve();
    return cudaGetLastError() == cudaSuccess ? (int64_t)pos : SZX_ECUDA;
}

int64_t szx_load_host(const void* h_in, uint64_t in_bytes, void* d_out, uint64_t cap, void* stream) {
    if (!h_in || in_bytes < 64) return SZX_ECORRUPT;
    if (!have_device()) return SZX_ECUDA;
    const uint8_t* hb = static_cast<const uint8_t*>(h_in);
    std::vector<Part> parts;
    uint64_t total = 0;
    if (memcmp(hb, "SZXC", 4) == 0) {
        uint32_t P, ver;
        memcpy(&ver, hb + 4, 4);
        memcpy(&P, hb + 8, 4);
        memcpy(&total, hb + 16, 8);
        if (ver != 1 || P == 0 || 32 + 32ull * P > in_bytes) return SZX_ECORRUPT;
        uint64_t expect = 0;
        for (uint32_t i = 0; i < P; i++) {
            uint64_t e[4];
            memcpy(e, hb + 32 + 32ull * i, 32);
            if (e[0] != expect || e[2] % 16 || e[2] > in_bytes || e[3] > in_bytes - e[2] || e[3] < 64)
                return SZX_ECORRUPT;
            Part pt;
            if (parse_header(hb + e[2], e[3], &pt.h) || pt.h.n != e[1]) return SZX_ECORRUPT;
            if (!parts.empty() && pt.h.dtype != parts[0].h.dtype) return SZX_ECORRUPT;
            pt.off = e[2]; pt.len = e[3]; pt.first = e[0];
            parts.push_back(pt);
            expect += e[1];
        }
        if (expect != total) return SZX_ECORRUPT;
    } else {
        Part pt;
        if (parse_header(hb, in_bytes, &pt.h)) return SZX_ECORRUPT;
        pt.off = 0; pt.len = in_bytes; pt.first = 0;
        parts.push_back(pt);
        total = pt.h.n;
    }
    const uint64_t W = parts[0].h.dtype ? 8 : 4;
    if (cap < W * total) return SZX_ENOSPC;
    if (total && (!d_out || !aligned16(d_out))) return SZX_EINVAL;
    DumpRes R;
    if (!R.init(static_cast<cudaStream_t>(stream))) return SZX_ECUDA;
    cudaStream_t s = R.s, s2 = R.s2;
    uint64_t lmax = 16, wmax = 16;
    for (auto& pt : parts) {
        lmax = std::max(lmax, al16(pt.len));
        wmax = std::max(wmax, szx_decompress_workspace_bytes(&pt.h));
    }
    void* buf[2] = {R.dalloc(lmax), R.dalloc(lmax)};
    void* ws[2] = {R.dalloc(wmax), R.dalloc(wmax)};
    int32_t* st = static_cast<int32_t*>(R.dalloc(4ull * parts.size()));
    if (!buf[0] || !buf[1] || !ws[0] || !ws[1] || !st) return SZX_ENOMEM;
    cudaMemsetAsync(st, 0, 4ull * parts.size(), s);
    cudaEvent_t copied[2] = {R.event(), R.event()}, decoded[2] = {R.event(), R.event()};
    uint8_t* out = static_cast<uint8_t*>(d_out);
    for (size_t q = 0; q < parts.size(); q++) {
        const Part& pt = parts[q];
        if (q >= 2) cudaStreamWaitEvent(s2, decoded[q & 1], 0);  // the buffer's previous shard is decoded
        if (cudaMemcpyAsync(buf[q & 1], hb + pt.off, pt.len, cudaMemcpyHostToDevice, s2) != cudaSuccess)
            return SZX_ECUDA;
        cudaEventRecord(copied[q & 1], s2);
        cudaStreamWaitEvent(s, copied[q & 1], 0);
        if (pt.h.n) {
            int rc = szx_decompress_async(buf[q & 1], pt.len, &pt.h, out + W * pt.first, cap - W * pt.first, ws[q & 1],
                                          wmax, st + q, s);
            if (rc) return rc;
        }
        cudaEventRecord(decoded[q & 1], s);
    }
    std::vector<int32_t> hs(parts.size());
    if (cudaMemcpyAsync(hs.data(), st, 4 * hs.size(), cudaMemcpyDeviceToHost, s) != cudaSuccess) return SZX_ECUDA;
    if (cudaStreamSynchronize(s) != cudaSuccess) return SZX_ECUDA;
    timing_resolve();
    for (int32_t e : hs)
        if (e) return e;
    return (int64_t)total;
}

void szx_timing_enable(int on) {
    Timing& T = timing();
    std::lock_guard<std::mutex> g(T.mu);
    T.on = on != 0;
    g_timing_on.store(on != 0);
}
void szx_timing_reset(void) {
    Timing& T = timing();
    std::lock_guard<std::mutex> g(T.mu);
    T.resolve();
    for (auto& m : T.ms) m = 0;
    for (auto& c : T.cnt) c = 0;
}
int szx_timing_read(const char** names, double* ms_sum, uint64_t* launches, int cap) {
    Timing& T = timing();
    std::lock_guard<std::mutex> g(T.mu);
    T.resolve();
    int k = (int)T.names.size();
    for (int i = 0; i < k && i < cap; i++) {
        if (names) names[i] = T.names[i];
        if (ms_sum) ms_sum[i] = T.ms[i];
        if (launches) launches[i] = T.cnt[i];
    }
    return k;
}
uint64_t szx_launch_count(void) { return g_launches.load(); }
void szx_debug_set_r_bias(int r_bias) { g_rbias.store(r_bias); }

const char* szx_strerror(int code) {
    switch (code) {
        case SZX_OK: return "ok";
        case SZX_EINVAL: return "invalid argument";
        case SZX_ENOSPC: return "capacity too small";
        case SZX_ECORRUPT: return "corrupt stream";
        case SZX_ECUDA: return "CUDA error or no device";
        case SZX_ENOMEM: return "allocation failed";
        default: return "unknown error";
    }
}

#if SZX_TIMELINE
// diagnostic timing builds only: copy the decoder's per-warp timeline to host
int szx_debug_timeline(uint64_t* h_dst, uint64_t n) {
    const uint64_t cap = sizeof(szx::g_tl) / sizeof(uint64_t);
    return cudaMemcpyFromSymbol(h_dst, szx::g_tl, 8 * (n < cap ? n : cap)) == cudaSuccess ? SZX_OK : SZX_ECUDA;
}
// ... and the index-phase stamps of every CTA (8 x u64 per CTA)
int szx_debug_timeline_index(uint64_t* h_dst, uint64_t n) {
    const uint64_t cap = sizeof(szx::g_tli) / sizeof(uint64_t);
    return cudaMemcpyFromSymbol(h_dst, szx::g_tli, 8 * (n < cap ? n : cap)) == cudaSuccess ? SZX_OK : SZX_ECUDA;
}
#endif
#if SZX_GUARDSTAT
// diagnostic builds only: {guarded blocks, warp-tiles} counted by the fused encoder since load
int szx_debug_guardstat(uint64_t* h_dst) {
    return cudaMemcpyFromSymbol(h_dst, szx::g_guardstat, 16) == cudaSuccess ? SZX_OK : SZX_ECUDA;
}
#endif
#if SZX_ETIMELINE
// diagnostic timing builds only: the fused encoder's per-tile timeline (4 x u64 per tile)
int szx_debug_enc_timeline(uint64_t* h_dst, uint64_t n) {
    const uint64_t cap = sizeof(szx::g_etl) / sizeof(uint64_t);
    return cudaMemcpyFromSymbol(h_dst, szx::g_etl, 8 * (n < cap ? n : cap)) == cudaSuccess ? SZX_OK : SZX_ECUDA;
}
#endif
}  // extern "C"
