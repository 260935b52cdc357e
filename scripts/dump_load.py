"""Dump / load throughput (Fig. 16 analogue): a GPU-resident
NYX-shaped 512^3 field written to pinned host memory raw (one D2H copy) vs compressed
(szx_dump_host, P shards, compression overlapped with the copy-out), and read back raw (H2D)
vs szx_load_host.  GB/s = original bytes / wall time of the blocking call, median of 5."""
import json
import os
import statistics
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_hpdc_yudztt0c22_b200 as szx
import synth


def med(f, k=5):
    t = []
    for _ in range(k + 1):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        f()
        torch.cuda.synchronize()
        t.append(time.perf_counter() - t0)
    return statistics.median(t[1:])


for field in (0, 1):
    x = synth.nyx_like(field, n=512, device="cuda").reshape(-1).contiguous()
    nb = x.numel() * 4
    host = torch.empty(x.numel(), dtype=torch.float32, pin_memory=True)
    t_raw_out = med(lambda: host.copy_(x, non_blocking=True))
    t_raw_in = med(lambda: x.copy_(host, non_blocking=True))
    for P in (1, 4, 16):
        out = torch.empty(32 + 32 * P + nb + P * 65536, dtype=torch.uint8, pin_memory=True)
        c = szx.dump_host(x, 1e-3, "rel", 128, P, out=out)
        t_dump = med(lambda: szx.dump_host(x, 1e-3, "rel", 128, P, out=out))
        y = torch.empty_like(x)
        t_load = med(lambda: szx.load_host(c, out=y))
        assert (y.double() - x.double()).abs().max().item() <= szx.read_header(
            c[c[48:56].numpy().view("<u8")[0]:][:64].numpy().tobytes()).eb_abs
        print(json.dumps({"field": ["density", "velocity"][field], "parts": P, "bytes": nb, "container_bytes": c.numel(),
                          "cr": nb / c.numel(), "raw_d2h_gbs": nb / t_raw_out / 1e9, "dump_gbs": nb / t_dump / 1e9,
                          "raw_h2d_gbs": nb / t_raw_in / 1e9, "load_gbs": nb / t_load / 1e9,
                          "dump_speedup": t_raw_out / t_dump, "load_speedup": t_raw_in / t_load}), flush=True)
