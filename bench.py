"""SZx B200 benchmark (one JSON line on rank 0).

Workload (BASELINE.json configs[2], the config the north_star's >=60%-of-HBM target
names): NYX-shaped 512^3 float32 synthetic field (baryon-density-like exp(2.5 g),
g a Gaussian random field with P(k) ~ k^-4), REL error bound 1e-3, block 128.
A step = compress + decompress of the rank's 512^3 array (every row of SURVEY
8(a)).  N GPUs: weak scaling, each rank owns a 512^3 shard of an N x 512^3
array; REL needs the global range (all-reduce of 16 B) and the container needs
the shard sizes (all-gather of 16 B per rank).

value = N * 512^3 * 4 bytes / (max over ranks of the device time of one step).
"""
from __future__ import annotations

import argparse
import json
import os
import platform
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

METRIC = "SZx compress+decompress throughput, N*W / (T_compress + T_decompress)"
UNIT = "GB/s"


def _args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=300)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=512, help="cube edge of the NYX-shaped field")
    ap.add_argument("--field", type=int, default=0, help="0 density, 1 velocity, 2 temperature")
    ap.add_argument("--eb", type=float, default=1e-3)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-fields", action="store_true", help="skip the other NYX fields' numbers")
    return ap.parse_args()


def _workload(a, n_total):
    names = {0: "baryon-density-like exp(2.5g)", 1: "velocity-like g", 2: "temperature-like exp(0.7g)"}
    return {"workload": f"NYX-shaped {a.n}^3 float32 synthetic GRF P(k)~k^-4, {names[a.field]}, "
                        f"REL eb {a.eb:g}, block 128 (BASELINE.json configs[2])",
            "elements_per_gpu": a.n ** 3, "global_elements": n_total, "block_size": 128,
            "eb_mode": "rel", "eb": a.eb,
            "l2": "no flush: inputs larger than L2 (537 MB field + 537 MB output per GPU > 126 MB L2)",
            "parallelism": f"block-range shards x{a.gpus} (weak)"}


class ClockSampler:
    """nvidia-smi clocks / throttle reasons sampled in the background (B200_PROFILING recipe)."""
    Q = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, index: int):
        self.rows = []
        self.index = index
        self.proc = None
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(index), f"--query-gpu={self.Q}",
                                          "--format=csv,noheader,nounits", "-lms", "50"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
        except Exception:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append((time.time(), line.strip()))

    def wait_first(self, timeout=5.0):
        t0 = time.time()
        while self.proc and not self.rows and time.time() - t0 < timeout:
            time.sleep(0.02)

    def summary(self, t0, t1):
        if self.proc:
            self.proc.terminate()
        rows = [r for (t, r) in self.rows if t0 - 0.06 <= t <= t1 + 0.06] or [r for _, r in self.rows]
        sm, mx, reasons = [], None, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in rows:
            f = [x.strip() for x in r.split(",")]
            try:
                sm.append(float(f[0]))
                mx = float(f[1])
                for nm, v in zip(names, f[4:8]):
                    if v.lower().startswith("active"):
                        reasons.add(nm)
            except (ValueError, IndexError):
                pass
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": mx,
                "reasons": sorted(reasons), "samples": len(sm)}


def _cpu_info():
    model = platform.processor() or ""
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    return model, os.cpu_count()


def _ncu_traffic(kernel: str):
    """dram__bytes_read.sum + dram__bytes_write.sum of `kernel` (one launch) from the newest
    committed ncu --set full summary under profiles/, or None."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_ncu_full_summary.json")))
    if not files:
        return None, None
    d = json.load(open(files[-1]))
    ncu_name = {"k_decode": "k_decode_w"}.get(kernel, kernel)  # timing label -> template name
    for name, v in d.items():
        if name.startswith(ncu_name + "<") or name == ncu_name:
            return v.get("dram_bytes"), os.path.basename(files[-1])
    return None, None


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"], "measured"
    except Exception:
        return 6650.0, "fallback"


def run_reference(a):
    """--impl reference: the CPU oracle as it stands (serial C, 1 thread) on a bounded
    sample of the same workload: a 128 x 512 x 512 slab of the NYX-shaped field."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import numpy as np
    import torch

    import oracle
    import synth
    x = synth.nyx_like(a.field, n=a.n, device="cpu").reshape(-1)
    slab = x[: (a.n // 4) * a.n * a.n].numpy().copy()
    del x
    times = []
    for i in range(a.warmup + a.steps):
        t0 = time.perf_counter()
        s = oracle.compress(slab, a.eb, oracle.REL, 128)
        oracle.decompress(s)
        if i >= a.warmup:
            times.append(time.perf_counter() - t0)
    ms = 1e3 * sum(times) / len(times)
    gbs = slab.nbytes / (ms / 1e3) / 1e9
    model, cores = _cpu_info()
    out = {"impl": "reference", "metric": METRIC, "value": gbs, "unit": UNIT, "n_gpus": a.gpus,
           "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms, "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": _workload(a, a.n ** 3),
           "cpu_baseline": {"value": gbs, "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": f"{slab.size} values ({a.n // 4}x{a.n}x{a.n} slab), compress+decompress",
                            "cpu": model, "host_cores": cores},
           "e2e": {"value": gbs, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
           "cr": slab.nbytes / s.size}
    print(json.dumps(out), flush=True)


def cpu_baseline(x_cpu, eb):
    """Oracle (serial C, 1 thread) timed on the host: 3 compress+decompress steps of the full field."""
    import oracle
    arr = x_cpu.numpy()
    t = []
    for _ in range(3):
        t0 = time.perf_counter()
        s = oracle.compress(arr, eb, oracle.REL, 128)
        oracle.decompress(s)
        t.append(time.perf_counter() - t0)
    sec = statistics.median(t)
    model, cores = _cpu_info()
    return {"value": arr.nbytes / sec / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"full field, {arr.size} values, median of 3 compress+decompress steps",
            "cpu": model, "host_cores": cores}, s


def cpu_baseline_all_cores(x_cpu, eb):
    """T = host-core-count serial oracles on T block-range shards
    (threads calling the C oracle release the GIL), the global REL bound from the shards' finite
    ranges: one compress+decompress of the full field, median of 3."""
    import concurrent.futures as cf

    import numpy as np

    import oracle
    from paper_conf_hpdc_yudztt0c22_b200.dist import shard_elems
    arr = x_cpu.numpy()
    T = os.cpu_count() or 1
    parts = [shard_elems(arr.size, 128, T, p) for p in range(T)]

    def rng(p):
        e0, ne = parts[p]
        v = arr[e0:e0 + ne]
        v = v[np.isfinite(v)]
        return (float(v.min()), float(v.max())) if v.size else None

    def work(p, eb_abs):
        e0, ne = parts[p]
        s = oracle.compress_shard(arr[e0:e0 + ne], eb, eb_abs, oracle.REL, 128)
        oracle.decompress(s)
        return s.size

    t = []
    with cf.ThreadPoolExecutor(T) as ex:
        for _ in range(3):
            t0 = time.perf_counter()
            r = [v for v in ex.map(rng, range(T)) if v]
            eb_abs = eb * (max(b for _, b in r) - min(a for a, _ in r)) if r else 0.0
            sizes = list(ex.map(lambda p: work(p, eb_abs), range(T)))
            t.append(time.perf_counter() - t0)
    sec = statistics.median(t)
    return {"value": arr.nbytes / sec / 1e9, "unit": UNIT, "cores": T, "kind": "oracle",
            "sample": f"full field, {arr.size} values, {T} block-range shards on {T} threads, "
                      f"median of 3 compress+decompress steps", "stream_bytes": int(sum(sizes))}


def main():
    a = _args()
    if a.impl == "reference":
        run_reference(a)
        return
    import torch
    import torch.distributed as dist

    import paper_conf_hpdc_yudztt0c22_b200 as szx
    from paper_conf_hpdc_yudztt0c22_b200 import dist as sdist
    import synth

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    group = None
    if world > 1:
        dist.init_process_group("nccl", device_id=dev)
    n_el = a.n ** 3
    x = synth.nyx_like(a.field, n=a.n, device=dev, seed_offset=rank).reshape(-1).contiguous()
    y = torch.empty_like(x)
    stream = torch.cuda.current_stream()
    sc = sdist.ShardedCompressor(n_el, torch.float32, 128, device=dev, group=group)
    codec = szx.Codec(n_el, torch.float32, 128, device=dev)

    def step():
        if world > 1:
            sc.compress(x, a.eb, "rel")
            out = sc.out
        else:
            codec.compress_async(x, a.eb, "rel")
            out = codec.out
        ev_mid.record()
        codec.decompress_async(out, hdr, y)

    # header shape for the non-blocking decoder (n, dtype, block) + first correctness check
    if world > 1:
        sc.compress(x, a.eb, "rel")
        s0 = sc.stream()
    else:
        codec.compress_async(x, a.eb, "rel")
        s0 = codec.out[: codec.stream_bytes()]
    hdr = szx.read_header(s0[:64].cpu().numpy().tobytes())
    S = s0.numel()
    if "SZX_LIB" not in os.environ:
        ref_y = szx.decompress(s0)
        err = (ref_y.double() - x.double()).abs().max().item()
        assert err <= hdr.eb_abs, (err, hdr.eb_abs)
    else:  # experiment builds (scripts/run_variants.sh) may skip work or write garbage
        err = float("nan")

    sampler = ClockSampler(local) if rank == 0 else None
    if sampler:
        sampler.wait_first()
    ev_mid = torch.cuda.Event(enable_timing=True)
    for _ in range(a.warmup):
        step()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    # ---- timed region (the contract's K steps): kernels chained with programmatic
    # dependent launch, per-phase events only (between compress and decompress)
    l0 = szx.launch_count()
    evs = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
            torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    t_wall0 = time.time()
    e_start = torch.cuda.Event(enable_timing=True)
    e_end = torch.cuda.Event(enable_timing=True)
    e_start.record()
    for i in range(a.steps):
        e0, e1, e2 = evs[i]
        e0.record()
        ev_mid = e1
        step()
        e2.record()
    e_end.record()
    torch.cuda.synchronize()
    t_wall1 = time.time()
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    launches = szx.launch_count() - l0
    total_ms = e_start.elapsed_time(e_end)
    comp_ms = statistics.median([e0.elapsed_time(e1) for e0, e1, _ in evs])
    dec_ms = statistics.median([e1.elapsed_time(e2) for _, e1, e2 in evs])
    ms_step = total_ms / a.steps
    if world > 1:
        t = torch.tensor([ms_step, comp_ms, dec_ms], device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_step, comp_ms, dec_ms = t.tolist()
    # ---- per-kernel pass: the library records CUDA events around every launch on
    # its launch stream (this serialises the launches, so it is a separate pass)
    szx.timing_reset()
    szx.timing_enable(True)
    for i in range(min(a.steps, 100)):
        step()
    torch.cuda.synchronize()
    szx.timing_enable(False)
    kt = szx.timing_read()
    clocks = sampler.summary(t_wall0, t_wall1) if sampler else None

    # ---------------- the other NYX-shaped fields (same config, same kernels): velocity and
    # temperature are dense (every block nonconstant), so they bound the ALU-heavy encode /
    # decode paths, where density's ~85% constant blocks take the fast fill path
    fields = None
    if not a.no_fields and world == 1:
        fields = {}
        peak_f, _ = _peaks()
        names = {0: "density", 1: "velocity", 2: "temperature"}
        for f in (0, 1, 2):
            if f == a.field:
                continue
            xf = synth.nyx_like(f, n=a.n, device=dev).reshape(-1).contiguous()
            cf = szx.Codec(n_el, torch.float32, 128, device=dev)
            cf.compress_async(xf, a.eb, "rel")
            Sf = cf.stream_bytes()
            hf = szx.read_header(cf.out[:64].cpu().numpy().tobytes())
            yf = torch.empty_like(xf)
            kf = max(10, min(a.steps, 50))
            ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True),
                   torch.cuda.Event(enable_timing=True)) for _ in range(kf + 3)]
            for e0, e1, e2 in ev:
                e0.record()
                cf.compress_async(xf, a.eb, "rel")
                e1.record()
                cf.decompress_async(cf.out, hf, yf)
                e2.record()
            torch.cuda.synchronize()
            cms = statistics.median([e0.elapsed_time(e1) for e0, e1, _ in ev[3:]])
            dms = statistics.median([e1.elapsed_time(e2) for _, e1, e2 in ev[3:]])
            errf = (yf.double() - xf.double()).abs().max().item()
            assert errf <= hf.eb_abs, (f, errf, hf.eb_abs)
            nb = n_el * 4
            fields[names[f]] = {"compress_gbs": nb / (cms / 1e3) / 1e9, "decompress_gbs": nb / (dms / 1e3) / 1e9,
                                "compress_hbm_frac": (2 * nb + Sf) / (cms / 1e3) / 1e9 / peak_f,
                                "decompress_hbm_frac": (Sf + nb) / (dms / 1e3) / 1e9 / peak_f,
                                "cr": nb / Sf, "nonconst_frac": hf.n_nonconst / ((n_el + 127) // 128),
                                "steps": kf, "max_abs_err_le_eb": True}
            del xf, yf, cf

    # ---------------- end to end through the C ABI host entry points (pinned host buffers)
    e2e = None
    if not a.no_e2e:
        xh = x.cpu().pin_memory()
        sh = torch.empty(szx.compress_bound(n_el, szx.F32, 128), dtype=torch.uint8, pin_memory=True)
        yh = torch.empty(n_el, dtype=torch.float32, pin_memory=True)
        ne = max(3, min(a.steps, 10))
        tt = []
        for i in range(ne + 2):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            s_h = szx.compress_host(xh, a.eb, "rel", 128, out=sh)
            szx.decompress_host(s_h, out=yh)
            tt.append(time.perf_counter() - t0)
        e2e_s = statistics.median(tt[2:])
        if world > 1:
            t = torch.tensor([e2e_s], device=dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_s = t.item()
        e2e = {"value": world * n_el * 4 / e2e_s / 1e9, "unit": UNIT,
               "h2d_bytes_per_step": n_el * 4 + S, "d2h_bytes_per_step": S + n_el * 4,
               "api": "szx_compress_host + szx_decompress_host (pinned host buffers)", "steps": ne}

    if rank == 0:
        peak, peak_kind = _peaks()
        nbytes = n_el * 4
        # per-kernel live times (library CUDA events on the launch stream, timed region only)
        kms = {k: v[0] / max(v[1], 1) for k, v in kt.items()}
        # algorithmic bytes per launch
        nnc, pb = hdr.n_nonconst, hdr.payload_bytes
        nB = (n_el + 127) // 128
        alg = {
            "k_block_stats": nbytes + nB * 8,
            "k_classify": nB * 8 + nB * 4 + nB // 8 + 9 * nnc,
            "k_enc_size": nnc * 128 * 4 + 2 * nnc + 5 * nnc,
            "k_zscan": 2 * nnc,
            "k_enc_write": nnc * 128 * 4 + 5 * nnc + pb,
            "k_decode": S + nbytes,
        }
        dom = max(kms, key=lambda k: kms[k]) if kms else None
        roof = None
        if dom:
            ach = alg.get(dom, 0) / (kms[dom] / 1e3) / 1e9
            traffic, src = _ncu_traffic(dom)
            roof = {"kernel": dom, "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
                    "frac": ach / peak, "peak_kind": peak_kind, "traffic": traffic, "traffic_source": src,
                    "alg_bytes_per_launch": alg.get(dom), "ms_per_launch": kms[dom]}
        comp_alg = 2 * nbytes + S   # REL: range pass + encode
        dec_alg = S + nbytes
        cpu = None
        if not a.no_cpu and world == 1:
            cpu, s_ref = cpu_baseline(x.cpu(), a.eb)
            cpu["stream_identical_to_gpu"] = bool(torch.equal(torch.from_numpy(s_ref), s0.cpu()))
            cpu["all_cores"] = cpu_baseline_all_cores(x.cpu(), a.eb)
        value = world * nbytes / (ms_step / 1e3) / 1e9
        out = {
            "metric": METRIC, "value": value, "unit": UNIT, "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32", "data": "synthetic", "config": _workload(a, world * n_el),
            "compress_gbs": world * nbytes / (comp_ms / 1e3) / 1e9,
            "decompress_gbs": world * nbytes / (dec_ms / 1e3) / 1e9,
            "compress_hbm_frac": comp_alg / (comp_ms / 1e3) / 1e9 / peak,
            "decompress_hbm_frac": dec_alg / (dec_ms / 1e3) / 1e9 / peak,
            "cr": nbytes / S, "stream_bytes": S, "nonconst_blocks": nnc, "blocks": nB,
            "max_abs_err": err, "eb_abs": hdr.eb_abs,
            "roofline": roof, "kernels_ms_per_launch": kms, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": launches, "clocks": clocks, "other_nyx_fields": fields,
            "timing": "value/ms_per_step: CUDA events around the K timed steps (kernels chained with PDL); "
                      "kernels_ms_per_launch/roofline: library CUDA events around each launch in a second "
                      "pass of min(K,100) steps",
            "paper_context": "cuSZx A100: 150-216 GB/s compress, 150-291 GB/s decompress (P:L3207-3220)",
        }
        print(json.dumps(out), flush=True)
    if world > 1:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
