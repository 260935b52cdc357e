/*
 * szx.h -- C ABI of libszx_b200.so, the B200 (sm_100a) SZx block-wise
 * error-bounded lossy compressor.
 *
 * Method: Yu et al., "Ultrafast Error-Bounded Lossy Compression for
 * Scientific Datasets", HPDC'22 (cited as P:La-b = PAPER.md lines a-b).
 *   - problem statement: compress N values D under |d_i - d'_i| <= e
 *     (Formula 1); output "compressed data stream in form of
 *     bytes" (Alg. 1 I/O);
 *   - compress = Alg. 1 + Formulas 4/5 (P:L1024-1040,
 *     P:L1317-1324) + zsize_array;
 *   - decompress = Fig. 10;
 *   - REL = value-range-relative bound (footnote 1).
 * The byte layout of the stream is DESIGN.md section 4.
 *
 * Conventions (all entry points):
 *   - Pointers named d_* are DEVICE pointers, h_* are HOST pointers.
 *     Device buffers must be 16-byte aligned (torch allocations are).
 *   - The caller owns every buffer; the library keeps no pointer after the
 *     call returns.  Scratch memory is either the caller's workspace
 *     (*_ws variants, size from *_workspace_bytes) or stream-ordered
 *     cudaMallocAsync/cudaFreeAsync on `stream`.
 *   - All work is enqueued on `stream` (a cudaStream_t; NULL = legacy
 *     default stream).  Calls that return a size synchronise `stream`
 *     before returning; *_async variants never synchronise.
 *   - Errors are negative return values (SZX_E*); no call aborts, and a
 *     corrupt stream is reported as SZX_ECORRUPT without out-of-bounds
 *     accesses.  There is no CPU fallback: without a CUDA device every
 *     compute call returns SZX_ECUDA.
 *   - Supported GPU block sizes b: 32, 64, 128 and 256 (a warp per block,
 *     b / 32 values per lane; b = 128 is the paper's choice, P:L2099-2105,
 *     and the one the fast paths target; the block-size study is Sec. 5.3,
 *     P:L1748-2188).  Max elements per stream: 2^36.
 */
#ifndef SZX_B200_H
#define SZX_B200_H

#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

typedef enum { SZX_F32 = 0, SZX_F64 = 1 } szx_dtype_t;
/* SZX_ABS: eb is the absolute bound e.  SZX_REL: e = eb * (max - min) over
 * the finite values of the array (footnote 1; reading R13). */
typedef enum { SZX_ABS = 0, SZX_REL = 1 } szx_ebmode_t;

enum {
    SZX_OK = 0,
    SZX_EINVAL = -1,   /* bad argument: dtype, mode, eb < 0 / NaN / Inf, block size, null or misaligned pointer */
    SZX_ENOSPC = -2,   /* output (or workspace) capacity too small */
    SZX_ECORRUPT = -3, /* stream fails validation (magic, sizes, zsize sum, payload) */
    SZX_ECUDA = -4,    /* CUDA runtime error (or no device) */
    SZX_ENOMEM = -5    /* stream-ordered allocation failed */
};

/* Parsed 64-byte stream header. */
typedef struct {
    uint32_t version;        /* 1 */
    uint32_t dtype;          /* szx_dtype_t */
    uint32_t eb_mode;        /* szx_ebmode_t */
    uint32_t block_size;     /* b */
    uint64_t n;              /* number of values */
    double eb_user;          /* eb as passed by the caller */
    double eb_abs;           /* absolute bound actually enforced */
    uint64_t n_nonconst;     /* number of nonconstant blocks (nNC) */
    uint64_t payload_bytes;  /* sum of zsize */
    uint64_t stream_bytes;   /* total stream length implied by the header */
} szx_header_t;

/* ---------------------------------------------------------------- sizes */

/* Worst-case stream bytes for n values (every block raw):
 * 64 + al16(ceil(nB/8)) + al16(W nB) + al16(2 nB) + nB + sum ceil(len/4) + W n. */
uint64_t szx_compress_bound(uint64_t n, szx_dtype_t dt, uint32_t block_size);

/* Workspace bytes needed by szx_compress_ws / _async for n values. */
uint64_t szx_compress_workspace_bytes(uint64_t n, szx_dtype_t dt, uint32_t block_size);

/* Workspace bytes needed by szx_decompress_ws / _async to decode a stream of
 * h->n values with block size h->block_size. */
uint64_t szx_decompress_workspace_bytes(const szx_header_t* h);

/* ------------------------------------------------------------- compress */

/* Compress n values at d_in (device, dt) into d_out (device, capacity
 * out_capacity >= szx_compress_bound).  eb: absolute bound (SZX_ABS) or
 * value-range ratio (SZX_REL), finite and >= 0.  Allocates scratch with
 * cudaMallocAsync on `stream`, synchronises, and returns the stream length
 * in bytes (>= 64), or a negative SZX_E* code.  n = 0 gives a 64-byte
 * header-only stream. */
int64_t szx_compress(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                     uint32_t block_size, void* d_out, uint64_t out_capacity, void* stream);

/* As szx_compress with a caller workspace d_ws of ws_bytes
 * (>= szx_compress_workspace_bytes). */
int64_t szx_compress_ws(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                        uint32_t block_size, void* d_out, uint64_t out_capacity, void* d_ws,
                        uint64_t ws_bytes, void* stream);

/* Non-blocking compress: enqueues all kernels and writes the final stream
 * length (uint64) to d_total_bytes (device pointer).  Returns SZX_OK or a
 * negative code for argument errors detected on the host. */
int szx_compress_async(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                       uint32_t block_size, void* d_out, uint64_t out_capacity, void* d_ws,
                       uint64_t ws_bytes, uint64_t* d_total_bytes, void* stream);

/* ----------------------------------------------------------- decompress */

/* Host-side parse + validation of the 64-byte header at h_bytes (host).
 * Returns SZX_OK or SZX_ECORRUPT. */
int szx_read_header(const void* h_bytes, uint64_t nbytes, szx_header_t* out);

/* Decompress the stream (in_bytes at d_in, device) into d_out (device,
 * out_capacity_bytes >= n * W).  Accepts a bare SZX1 stream or an SZXC
 * shard container.  Reads the header(s) back to the host, synchronises,
 * and returns the number of values, or a negative SZX_E* code. */
int64_t szx_decompress(const void* d_in, uint64_t in_bytes, void* d_out,
                       uint64_t out_capacity_bytes, void* stream);

/* Decompress only blocks [first_block, first_block + n_blocks) of a stream
 * (SZX1) or container (SZXC), the "1 stream -> Q GPUs" path of SURVEY 8(e):
 * each rank decodes its own block range.  The decoder still reads the bitmap
 * and zsize sections up to the range (the paper's prefix sum over block
 * sizes; <= 0.42 % of the raw size for f32, b = 128) and
 * decodes only the tiles of the range (Fig. 10's five steps).
 *   first_block  global block index (blocks of the stream's block_size; in a
 *                container, blocks are numbered over the whole array, and
 *                every shard must start on a block boundary -- true for
 *                block-range shards -- else SZX_EINVAL);
 *   n_blocks     count, clipped to the end of the array;
 *   d_out        device, >= 16-byte aligned; receives values
 *                [first_block * b, min(n, (first_block + n_blocks) * b)),
 *                element 0 being the first value of first_block;
 *   out_capacity_bytes >= that count * W, else SZX_ENOSPC.
 * Blocking (reads headers and the status back).  Returns the number of
 * values written (0 for an empty range), or SZX_EINVAL / SZX_ECORRUPT /
 * SZX_ECUDA / SZX_ENOMEM.  Output equals the same slice of szx_decompress. */
int64_t szx_decompress_blocks(const void* d_in, uint64_t in_bytes, uint64_t first_block, uint64_t n_blocks,
                              void* d_out, uint64_t out_capacity_bytes, void* stream);

/* As szx_decompress (SZX1 only) with a caller workspace. */
int64_t szx_decompress_ws(const void* d_in, uint64_t in_bytes, void* d_out,
                          uint64_t out_capacity_bytes, void* d_ws, uint64_t ws_bytes, void* stream);

/* Non-blocking SZX1 decode.  Of the host struct h only n, dtype and
 * block_size are used (the expected shape, e.g. from an earlier
 * szx_read_header); nNC and the payload size are read from the stream header
 * in device memory and validated there, so no host round-trip is needed
 * between a compress and a decompress.  Writes 0 (ok) or SZX_ECORRUPT
 * (int32) to d_status (device).  Returns SZX_OK or a host-detected error. */
int szx_decompress_async(const void* d_in, uint64_t in_bytes, const szx_header_t* h,
                         void* d_out, uint64_t out_capacity_bytes, void* d_ws, uint64_t ws_bytes,
                         int32_t* d_status, void* stream);

/* ------------------------------------------- reconstruction quality */

/* Decompress (as szx_decompress: SZX1 or SZXC) and, fused into the same
 * kernel, compare every reconstructed value with the original d_ref (device,
 * 16-byte aligned, n values of the stream's dtype, laid out like d_out).
 * h_qual (host, 4 doubles) receives:
 *   [0] max |x - x'| -- the quantity Formula 1 bounds, in
 *       double; identical bit patterns count 0, otherwise a NaN on either
 *       side counts +Inf;
 *   [1] sum (x - x')^2 in double (MSE = [1] / n; summation order is not
 *       fixed, so it is reproducible to rounding only);
 *   [2], [3] min and max of the finite x (+Inf / -Inf if none).
 * PSNR = 20 log10(([3] - [2]) / sqrt([1] / n)) (Formula 7).
 * Blocking.  Returns n or SZX_EINVAL / SZX_ENOSPC / SZX_ECORRUPT /
 * SZX_ECUDA / SZX_ENOMEM. */
int64_t szx_decompress_quality(const void* d_in, uint64_t in_bytes, const void* d_ref, void* d_out,
                               uint64_t out_capacity_bytes, double* h_qual, void* stream);

/* Non-blocking variant for one SZX1 stream (arguments as
 * szx_decompress_async).  d_qual (device, 4 x uint64, caller-owned) is
 * initialised on the stream and receives the raw accumulators
 * {max-error bits, sum of squares (double bits), order key of the min,
 * complemented order key of the max}; szx_quality_finish converts a host
 * copy of them into the 4 doubles above. */
int szx_decompress_quality_async(const void* d_in, uint64_t in_bytes, const szx_header_t* h,
                                 const void* d_ref, void* d_out, uint64_t out_capacity_bytes,
                                 void* d_ws, uint64_t ws_bytes, uint64_t* d_qual, int32_t* d_status,
                                 void* stream);
void szx_quality_finish(const uint64_t* raw4, double* out4);

/* ------------------------------------------------ end-to-end host buffers */

/* Compress host data h_in into host buffer h_out (capacity out_capacity):
 * copies in, compresses, copies the stream back.  Pinned host memory gives
 * full PCIe/NVLink-C2C bandwidth.  Returns stream bytes or SZX_E*. */
int64_t szx_compress_host(const void* h_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                          uint32_t block_size, void* h_out, uint64_t out_capacity, void* stream);

/* Decompress a host stream into host values.  Returns n or SZX_E*. */
int64_t szx_decompress_host(const void* h_in, uint64_t in_bytes, void* h_out,
                            uint64_t out_capacity_bytes, void* stream);

/* ------------------------------------------------ dump / load through host memory */

/* Dump a device array to host memory as an SZXC container of `parts`
 * block-range shards (shard q: blocks [q nB / parts, (q+1) nB / parts),
 * clipped to >= 1 block each; DESIGN.md s.8), the single-box analogue of the
 * paper's data dumping experiment (Fig. 16).  One pass reads
 * every shard's block statistics and local range (the REL bound is global,
 * footnote 1); then shard q+1 compresses while shard q is copied
 * device -> host on a second stream.  The container is byte-identical to
 * szx_compress_shard_async of each shard with the global bound, assembled
 * as in SURVEY Appendix A.
 *   d_in   device, 16-byte aligned, n values of dt;
 *   h_out  host (pinned for overlap; pageable works, serialised), h_cap bytes;
 *   stream the compute stream (the copy stream is internal).
 * Blocking.  Returns the container bytes, or SZX_EINVAL / SZX_ENOSPC (h_cap
 * too small: the sum of the shard streams, not the bound, must fit) /
 * SZX_ECUDA / SZX_ENOMEM.  Device scratch: the shards' workspaces plus two
 * stream buffers of one shard's bound. */
int64_t szx_dump_host(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb,
                      uint32_t block_size, uint32_t parts, void* h_out, uint64_t h_cap, void* stream);

/* Load an SZX1 stream or SZXC container held in host memory (h_in, pinned
 * for overlap) into the device array d_out (16-byte aligned, >= n W bytes):
 * shard q+1 is copied host -> device while shard q decodes (Fig. 10,
 * P:L2321-2336).  Blocking.  Returns n, or SZX_ECORRUPT / SZX_ENOSPC /
 * SZX_EINVAL / SZX_ECUDA / SZX_ENOMEM. */
int64_t szx_load_host(const void* h_in, uint64_t in_bytes, void* d_out, uint64_t out_capacity_bytes,
                      void* stream);

/* ------------------------------------------------ sharded (multi-GPU) use */

/* Pass 1 of a sharded compress: one read of the local shard that writes the
 * block statistics (min/max per block of block_size values) into d_ws
 * (ws_bytes >= szx_compress_workspace_bytes) and the shard's finite-value
 * range as two order-preserving uint64 keys to d_range_keys[2] (device):
 * [key(min), ~key(max)], where
 * key(x) maps (double)x to an unsigned integer with the same total order
 * (-0 < +0).  Combine shards with an element-wise MIN (e.g. an NCCL
 * all-reduce MIN after flipping bit 63 to signed order).  A shard without
 * finite values yields [UINT64_MAX, UINT64_MAX]. */
int szx_local_range(const void* d_in, szx_dtype_t dt, uint64_t n, uint32_t block_size,
                    uint64_t* d_range_keys, void* d_ws, uint64_t ws_bytes, void* stream);

/* Pass 2 of a sharded compress: MUST follow szx_local_range on the same
 * d_in, n, block_size, d_ws and stream.  Compresses the shard as a
 * standalone SZX1 stream whose REL bound comes from the GLOBAL range keys
 * d_range_keys[2] (device; szx_local_range's keys MIN-reduced over all
 * shards); d_range_keys is ignored for SZX_ABS.
 * Writes the stream length to d_total_bytes (device) without synchronising.
 * The stream is byte-identical to the oracle's shard p of a P-shard SZXC
 * container. */
int szx_compress_shard_async(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode,
                             double eb, const uint64_t* d_range_keys, uint32_t block_size,
                             void* d_out, uint64_t out_capacity, void* d_ws, uint64_t ws_bytes,
                             uint64_t* d_total_bytes, void* stream);

/* SURVEY 8(b)'s double-valued forms of the two sharded passes (thin wrappers
 * over the key-based calls above).
 *
 * szx_local_minmax: the finite-value range of the shard, d_minmax2[0] = min,
 * d_minmax2[1] = max as doubles (exact widening of the data type; -0 and +0
 * compare as -0 < +0, reading R13); no finite value -> (+Inf, -Inf).  Combine
 * shards with an all-reduce MIN of [0] and MAX of [1]; then
 * eb_abs = REL x (max - min) in double (footnote 1).  Non-blocking
 * (stream-ordered scratch).  Returns SZX_OK / SZX_EINVAL / SZX_ECUDA /
 * SZX_ENOMEM. */
int szx_local_minmax(const void* d_in, szx_dtype_t dt, uint64_t n, double* d_minmax2, void* stream);

/* szx_compress_shard: compress the shard as a standalone SZX1 stream whose
 * absolute bound is *d_eb_abs (device double, e.g. computed from the
 * all-reduced szx_local_minmax); the header records mode and eb_user as given
 * and eb_abs.  Byte-identical to the oracle's orc_compress_shard with the same
 * eb_abs.  Blocking: returns the stream bytes, or SZX_EINVAL / SZX_ENOSPC
 * (out_capacity < szx_compress_bound) / SZX_ECUDA / SZX_ENOMEM. */
int64_t szx_compress_shard(const void* d_in, szx_dtype_t dt, uint64_t n, szx_ebmode_t mode, double eb_user,
                           const double* d_eb_abs, uint32_t block_size, void* d_out, uint64_t out_capacity,
                           void* stream);

/* ------------------------------------------------------------ diagnostics */

/* Per-kernel device timing with CUDA events recorded on the launch stream
 * around every kernel (off by default).  szx_timing_read fills up to cap
 * entries of names/ms_sum/launch counts since the last reset and returns
 * the number of kernels. */
void szx_timing_enable(int on);
void szx_timing_reset(void);
int szx_timing_read(const char** names, double* ms_sum, uint64_t* launches, int cap);

/* Total kernels launched by the library since load (the bench's
 * gpu_launches count). */
uint64_t szx_launch_count(void);

/* Test hook: start the R2 escalation search r_bias bits away from
 * Formula 4 (0 = paper behaviour; the oracle has the same hook). */
void szx_debug_set_r_bias(int r_bias);

const char* szx_strerror(int code);

#ifdef __cplusplus
}
#endif

#endif /* SZX_B200_H */
