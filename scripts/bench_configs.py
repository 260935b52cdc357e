"""Per-config throughput sweep (BASELINE.json configs 1-5 on ONE GPU): compress and
decompress GB/s (N*W / T, Formulas 2/3), compression ratio, and the
fraction of the measured HBM peak with SURVEY 8(d)'s algorithmic bytes
(compress REL: 2NW + S; decompress: S + NW).

Timing: device-resident input and output, non-blocking C-ABI calls
(szx_compress_async / szx_decompress_async), each direction captured in a CUDA
graph and replayed between CUDA events, median of --iters after 3 warm-ups.  Inputs smaller than 2x L2
(CESM, Hurricane, Miranda) get an L2 flush (a 512 MB write) before every timed
call, outside the events.  Every config is checked against Formula 1 (max error
<= eb_abs) once.  One JSON line per (config, field, eb); config 5's 34 GB box is
one 1/8 shard by default (--box-full for the whole 4096x4096x512 array).

Usage: python scripts/bench_configs.py [--iters 20] [--only nyx,hacc] > configs.jsonl
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import torch  # noqa: E402

import paper_conf_hpdc_yudztt0c22_b200 as szx  # noqa: E402
import synth  # noqa: E402


def peak():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"]
    except Exception:
        return 6650.0


def cases(box_full: bool):
    yield "cesm", "CESM-ATM-shaped 1800x3600 T-like", lambda: synth.cesm_like(0, device="cuda"), [1e-3]
    yield "cesm", "CESM-ATM-shaped 1800x3600 cloud-like", lambda: synth.cesm_like(1, device="cuda"), [1e-3]
    yield "hurricane", "Hurricane-shaped 100x500x500 U-like", lambda: synth.hurricane_like(0, device="cuda"), \
        [1e-2, 1e-3, 1e-4]
    yield "hurricane", "Hurricane-shaped 100x500x500 QSNOW-like", \
        lambda: synth.hurricane_like(1, device="cuda"), [1e-2, 1e-3, 1e-4]
    for f, nm in enumerate(("density-like", "velocity-like", "temperature-like")):
        yield "nyx", f"NYX-shaped 512^3 {nm}", (lambda f=f: synth.nyx_like(f, n=512, device="cuda")), [1e-3]
    yield "hacc", "HACC-shaped 280,953,867 velocity-like", lambda: synth.hacc_like(0, device="cuda"), [1e-3]
    yield "hacc", "HACC-shaped 280,953,867 position-like", lambda: synth.hacc_like(1, device="cuda"), [1e-3]
    shape = (512, 4096, 4096) if box_full else (64, 4096, 4096)
    yield "box", f"box-scale {'x'.join(map(str, shape))} f32 plane waves" + ("" if box_full else " (1/8 shard)"), \
        lambda: synth.box_like(shape=shape, device="cuda"), [1e-4]
    yield "box", "Miranda-like 256x384x384 f64", lambda: synth.miranda_like(device="cuda"), [1e-4]
    yield "box", "QMCPack-like 288x115x69x69 f64", lambda: synth.qmcpack_like(device="cuda"), [1e-4]


def run_case(x: torch.Tensor, eb: float, iters: int, flush: torch.Tensor | None, b: int = 128):
    x = x.reshape(-1).contiguous()
    n = x.numel()
    W = x.element_size()
    codec = szx.Codec(n, x.dtype, b, device=x.device)
    y = torch.empty_like(x)
    codec.compress_async(x, eb, "rel")
    S = codec.stream_bytes()
    h = codec.header()
    codec.decompress_async(codec.out, h, y)
    torch.cuda.synchronize()
    assert int(codec.d_status.item()) == 0
    err = (y.double() - x.double()).abs().max().item() if n <= 300_000_000 else \
        max((y[i:i + 100_000_000].double() - x[i:i + 100_000_000].double()).abs().max().item()
            for i in range(0, n, 100_000_000))
    assert err <= h.eb_abs, (err, h.eb_abs)
    # each direction captured once in a CUDA graph (the 2-memset + 4-kernel compress, the
    # memset + persistent decoder), replayed between events; the L2 flush stays outside
    gs = torch.cuda.Stream()
    with torch.cuda.stream(gs):
        codec.compress_async(x, eb, "rel")
        codec.decompress_async(codec.out, h, y)
    gs.synchronize()
    gc, gd = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
    with torch.cuda.graph(gc, stream=gs):
        codec.compress_async(x, eb, "rel")
    with torch.cuda.graph(gd, stream=gs):
        codec.decompress_async(codec.out, h, y)
    tc, td = [], []
    for i in range(3 + iters):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
        if flush is not None:
            flush.fill_(i & 0xFF)
        ev[0].record()
        gc.replay()
        ev[1].record()
        if flush is not None:
            flush.fill_((i + 1) & 0xFF)
        ev[2].record()
        gd.replay()
        ev[3].record()
        torch.cuda.synchronize()
        if i >= 3:
            tc.append(ev[0].elapsed_time(ev[1]))
            td.append(ev[2].elapsed_time(ev[3]))
    assert int(codec.d_status.item()) == 0
    # decompression with the fused quality accumulators (max error, PSNR)
    tq = []
    for i in range(3 + iters):
        ev = [torch.cuda.Event(enable_timing=True) for _ in range(2)]
        if flush is not None:
            flush.fill_(i & 0xFF)
        ev[0].record()
        codec.decompress_quality_async(codec.out, h, y, x)
        ev[1].record()
        torch.cuda.synchronize()
        if i >= 3:
            tq.append(ev[0].elapsed_time(ev[1]))
    q = codec.quality()
    assert q["max_abs_err"] == err or n > 300_000_000, (q, err)
    # per-kernel breakdown (library events around each launch; separate pass)
    szx.timing_reset()
    szx.timing_enable(True)
    for _ in range(5):
        codec.compress_async(x, eb, "rel")
        codec.decompress_async(codec.out, h, y)
    torch.cuda.synchronize()
    szx.timing_enable(False)
    kt = {k: v[0] / max(v[1], 1) for k, v in szx.timing_read().items()}
    cms, dms = statistics.median(tc), statistics.median(td)
    nb = n * W
    pk = peak()
    return {"n": n, "dtype": "f32" if W == 4 else "f64", "stream_bytes": S, "cr": nb / S,
            "nonconst_frac": h.n_nonconst / ((n + b - 1) // b), "eb_abs": h.eb_abs, "max_abs_err": err,
            "compress_ms": cms, "decompress_ms": dms,
            "compress_gbs": nb / cms / 1e6, "decompress_gbs": nb / dms / 1e6,
            "compress_hbm_frac": (2 * nb + S) / cms / 1e6 / pk, "decompress_hbm_frac": (S + nb) / dms / 1e6 / pk,
            "decompress_quality_ms": statistics.median(tq), "psnr": q["psnr"], "max_abs_err_fused": q["max_abs_err"],
            "block": b, "kernels_ms": kt, "l2_flush": flush is not None}


def oracle_gbs(x: torch.Tensor, eb: float, b: int, reps: int = 3):
    """Serial C oracle (1 host thread), best of `reps` compress+decompress (SURVEY 8(d) oracle
    timing (i)); baseline only, never a code path of the product."""
    import time

    import oracle
    arr = x.reshape(-1).cpu().numpy()
    best = float("inf")
    for _ in range(reps):
        t0 = time.perf_counter()
        s = oracle.compress(arr, eb, oracle.REL, b)
        oracle.decompress(s)
        best = min(best, time.perf_counter() - t0)
    return arr.nbytes / best / 1e9


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--iters", type=int, default=20)
    ap.add_argument("--only", default="")
    ap.add_argument("--box-full", action="store_true")
    ap.add_argument("--blocks", default="128", help="block sizes to sweep, e.g. 128,256 (SURVEY 8(f) row 2)")
    ap.add_argument("--oracle", action="store_true", help="also time the serial C oracle (configs 1-4)")
    a = ap.parse_args()
    only = set(a.only.split(",")) if a.only else None
    l2 = torch.cuda.get_device_properties(0).L2_cache_size
    flush_buf = torch.empty(512 << 20, dtype=torch.uint8, device="cuda")
    for key, name, gen, ebs in cases(a.box_full):
        if only and key not in only:
            continue
        x = gen()
        torch.cuda.synchronize()
        small = x.numel() * x.element_size() < 4 * l2
        for eb in ebs:
            for b in (int(v) for v in a.blocks.split(",")):
                r = run_case(x, eb, a.iters, flush_buf if small else None, b)
                r.update({"config": key, "workload": name, "eb_rel": eb, "peak_gbs": peak()})
                if a.oracle and key != "box":
                    g = oracle_gbs(x, eb, b)
                    r.update({"oracle_1thread_gbs": g,
                              "gpu_vs_oracle": (r["n"] * (4 if r["dtype"] == "f32" else 8)) /
                              ((r["compress_ms"] + r["decompress_ms"]) * 1e6) / g})
                print(json.dumps(r), flush=True)
        del x
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
