"""SZx block-wise error-bounded lossy compression, B200-native (sm_100a).

Public API (all GPU; no CPU fallback):
    compress(x, eb, mode="rel", block_size=128) -> uint8 CUDA tensor (the stream)
    decompress(stream) -> float32/float64 CUDA tensor
    decompress_blocks(stream, first_block, n_blocks) -> the values of a block range
    decompress_quality(stream, ref) -> (values, max error / MSE / PSNR), fused into the decoder
    compress_host / decompress_host  -- end to end through host buffers
    dump_host / load_host            -- device array <-> host SZXC container, copy/compute overlapped
    Codec                            -- preallocated buffers, non-blocking calls
    local_minmax / compress_shard    -- SURVEY 8(b)'s double-valued sharded passes
    dist                             -- block-range sharding over torch.distributed (NCCL)
"""
from .szx import (ABS, F32, F64, REL, Codec, Header, SZxError, compress, compress_bound,  # noqa: F401
                  compress_host, compress_shard, decompress, decompress_blocks, decompress_host, decompress_quality, dump_host, load_host, launch_count, local_minmax, read_header,
                  set_r_bias, timing_enable, timing_read, timing_reset, workspace_bytes)

__all__ = ["compress", "decompress", "decompress_blocks", "decompress_quality", "compress_host", "decompress_host", "dump_host", "load_host", "Codec", "read_header",
           "compress_bound", "workspace_bytes", "local_minmax", "compress_shard", "SZxError", "ABS", "REL", "F32", "F64"]
