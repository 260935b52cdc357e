"""SZx B200 benchmark (one JSON line on rank 0).

Workload (BASELINE.json configs[2], the config the north_star's >=60%-of-HBM target
names): the NYX-shaped 512^3 float32 synthetic FIELDS -- baryon-density-like
exp(2.5 g), velocity-like 1e7 g and temperature-like 1e4 exp(0.7 g), g a Gaussian
random field with P(k) ~ k^-4 -- REL error bound 1e-3,
block 128.  A step = compress + decompress of every field (every row of SURVEY
8(a)), through the non-blocking C-ABI entry points, captured in one CUDA graph.

N GPUs (torchrun): strong scaling by default -- each field is split by block
range over the N ranks, each rank compresses its shard with the
GLOBAL REL bound (NCCL all-reduce of the range keys) and all-gathers the shard
records (the container offsets), then decodes its shard; the collectives are
captured in the same CUDA graph.  --scaling weak gives every rank a whole 512^3
realisation of each field instead.

value = sum over ranks of the bytes compressed+decompressed (N*W of the fields)
        / (max over ranks of the device time of one step).
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
FIELD_NAMES = {0: "density", 1: "velocity", 2: "temperature"}
NCU_NAME = {"k_decode": "k_decode_w", "k_encode": "k_encode_fused"}  # library timing label -> kernel name
FIELD_DESC = {0: "baryon-density-like exp(2.5g)", 1: "velocity-like 1e7 g", 2: "temperature-like 1e4 exp(0.7g)"}


def _args():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=50)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--n", type=int, default=512, help="cube edge of the NYX-shaped fields")
    ap.add_argument("--fields", default="0,1,2", help="NYX fields: 0 density, 1 velocity, 2 temperature")
    ap.add_argument("--eb", type=float, default=1e-3)
    ap.add_argument("--scaling", default=None, choices=["strong", "weak"],
                    help="N>1: strong (default; every field split over the ranks) or weak")
    ap.add_argument("--no-graph", action="store_true", help="launch the step eagerly instead of a CUDA graph")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--no-kernels", action="store_true", help="skip the per-kernel timing pass")
    a = ap.parse_args()
    a.fields = [int(f) for f in a.fields.split(",") if f != ""]
    return a


def _workload(a, world, scaling):
    names = " + ".join(FIELD_DESC[f] for f in a.fields)
    return {"workload": f"NYX-shaped {a.n}^3 float32 synthetic GRF P(k)~k^-4 fields ({names}), "
                        f"REL eb {a.eb:g}, block 128 (BASELINE.json configs[2])",
            "fields": [FIELD_NAMES[f] for f in a.fields], "elements_per_field": a.n ** 3,
            "global_elements": len(a.fields) * a.n ** 3 * (world if scaling == "weak" else 1),
            "block_size": 128, "eb_mode": "rel", "eb": a.eb,
            "l2": "no flush: every field (537 MB) and its reconstruction exceed the 126 MB L2; the step "
                  "cycles through the fields",
            "parallelism": (f"block-range shards x{world} ({scaling})" if world > 1 else "1 GPU")}


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


def _ncu_summary():
    """The newest committed ncu --set full summary (profiles/r*_ncu_full_summary.json):
    {field: {kernel: {"dram_bytes": ..., "time_us": ...}}} or the older flat form."""
    import glob
    files = sorted(glob.glob(os.path.join(ROOT, "profiles", "r*_ncu_full_summary.json")))
    if not files:
        return None, None
    return json.load(open(files[-1])), os.path.basename(files[-1])


def _ncu_kernel(summ, field: str, kernel: str):
    if not summ:
        return None
    d = summ.get(field) if isinstance(summ, dict) else None  # per-field summaries only (r02+)
    if not isinstance(d, dict):
        return None
    for name, v in d.items():
        if isinstance(v, dict) and (name == kernel or name.startswith(kernel + "<")):
            return v
    return None


def _sm_count() -> int:
    try:
        import torch
        return torch.cuda.get_device_properties(0).multi_processor_count
    except Exception:  # noqa: BLE001
        return 148


def _sm_max_mhz() -> float:
    try:
        return float(json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["sm_max_mhz"])
    except Exception:  # noqa: BLE001
        return 1965.0


def _peaks():
    try:
        return json.load(open(os.path.join(ROOT, "MEASURED_PEAKS.json")))["hbm_gbs"], "measured"
    except Exception:
        return 6650.0, "fallback"


# ----------------------------------------------------------------------------- reference arm
def _slab_edge(n):
    return max(1, n // 4)


def run_reference(a):
    """--impl reference: the CPU oracle as it stands (serial C, 1 thread) on a bounded sample of
    the same workload: the first n/4 z-planes of every field, compress + decompress."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    import oracle
    import synth
    slabs = []
    for f in a.fields:
        x = synth.nyx_like(f, n=a.n, device="cpu").reshape(-1)
        slabs.append(x[: _slab_edge(a.n) * a.n * a.n].numpy().copy())
        del x
    nbytes = sum(s.nbytes for s in slabs)
    times, sbytes = [], 0
    for i in range(a.warmup + a.steps):
        t0 = time.perf_counter()
        sbytes = 0
        for sl in slabs:
            s = oracle.compress(sl, a.eb, oracle.REL, 128)
            oracle.decompress(s)
            sbytes += s.size
        if i >= a.warmup:
            times.append(time.perf_counter() - t0)
    ms = 1e3 * sum(times) / len(times)
    gbs = nbytes / (ms / 1e3) / 1e9
    model, cores = _cpu_info()
    world = a.gpus
    cfg = _workload(a, world, a.scaling or ("strong" if world > 1 else "weak"))
    cfg["sample"] = f"first {_slab_edge(a.n)} of {a.n} z-planes of each field ({sum(s.size for s in slabs)} values)"
    out = {"impl": "reference", "metric": METRIC, "value": gbs, "unit": UNIT, "n_gpus": a.gpus,
           "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms, "higher_is_better": True,
           "scaling": "strong" if world > 1 else "weak", "vs_baseline": None, "dtype": "f32",
           "data": "synthetic", "config": cfg,
           "cpu_baseline": {"value": gbs, "unit": UNIT, "cores": 1, "kind": "oracle",
                            "sample": cfg["sample"] + ", compress+decompress per step",
                            "cpu": model, "host_cores": cores},
           "e2e": {"value": gbs, "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
           "cr": nbytes / sbytes}
    print(json.dumps(out), flush=True)


# ----------------------------------------------------------------------------- host baselines
def cpu_baseline(xs_cpu, eb, n_edge):
    """Oracle (serial C, 1 thread) on the host: a bounded sample (the first n/4 z-planes of every
    field), compress+decompress, median of 3."""
    import oracle
    m = _slab_edge(n_edge) * n_edge * n_edge
    slabs = [x[:m].numpy() for x in xs_cpu]
    t = []
    for _ in range(3):
        t0 = time.perf_counter()
        for sl in slabs:
            oracle.decompress(oracle.compress(sl, eb, oracle.REL, 128))
        t.append(time.perf_counter() - t0)
    sec = statistics.median(t)
    model, cores = _cpu_info()
    nb = sum(s.nbytes for s in slabs)
    return {"value": nb / sec / 1e9, "unit": UNIT, "cores": 1, "kind": "oracle",
            "sample": f"first {_slab_edge(n_edge)} of {n_edge} z-planes of each field ({m} values x "
                      f"{len(slabs)}), median of 3 compress+decompress steps",
            "cpu": model, "host_cores": cores}


def cpu_baseline_parallel(xs_cpu, eb, n_edge):
    """the paper's OpenMP design on all host cores (oracle/szx_omp.c: parallel
    Loop 1 over blocks, zsize array, prefix sum, one stream byte-identical to the serial oracle),
    same sample as cpu_baseline."""
    import oracle
    m = _slab_edge(n_edge) * n_edge * n_edge
    slabs = [x[:m].numpy() for x in xs_cpu]
    T = os.cpu_count() or 1
    t = []
    ident = True
    for _ in range(3):
        t0 = time.perf_counter()
        outs = [oracle.omp_compress(sl, eb, oracle.REL, 128, threads=T) for sl in slabs]
        for s in outs:
            oracle.omp_decompress(s, threads=T)
        t.append(time.perf_counter() - t0)
    for sl, s in zip(slabs, outs):
        ident = ident and bool((s == oracle.compress(sl, eb, oracle.REL, 128)).all()) if s.size else ident
    sec = statistics.median(t)
    nb = sum(s.nbytes for s in slabs)
    return {"value": nb / sec / 1e9, "unit": UNIT, "cores": T, "kind": "openmp-design baseline (oracle/szx_omp.c)",
            "sample": f"same sample as cpu_baseline, {T} threads, median of 3", "stream_identical_to_oracle": ident}


# ----------------------------------------------------------------------------- our arm
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
    torchrun = "WORLD_SIZE" in os.environ
    scaling = a.scaling or ("strong" if world > 1 else "weak")
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if torchrun:
        dist.init_process_group("nccl", device_id=dev)
    n_field = a.n ** 3
    nB = (n_field + 127) // 128

    # ---- inputs: rank's part of every field (strong: its block range; weak: its own realisation)
    xs, parts = [], []
    for f in a.fields:
        if scaling == "strong":
            full = synth.nyx_like(f, n=a.n, device=dev).reshape(-1)
            e0, ne = sdist.shard_elems(n_field, 128, world, rank)
            xs.append(full[e0:e0 + ne].clone())
            parts.append((e0, ne))
            del full
        else:
            xs.append(synth.nyx_like(f, n=a.n, device=dev, seed_offset=rank).reshape(-1).contiguous())
            parts.append((0, n_field))
    torch.cuda.synchronize()
    ys = [torch.empty_like(x) for x in xs]
    # sharded path (the collectives) under torchrun, plain codec otherwise
    if torchrun:
        coders = [sdist.ShardedCompressor(x.numel(), torch.float32, 128, device=dev, force_collectives=True)
                  for x in xs]
    else:
        coders = [szx.Codec(x.numel(), torch.float32, 128, device=dev) for x in xs]
    decs = [szx.Codec(x.numel(), torch.float32, 128, device=dev) for x in xs] if torchrun else coders
    stream = torch.cuda.Stream(device=dev)

    def compress_f(i):
        if torchrun:
            coders[i].compress(xs[i], a.eb, "rel")
        else:
            coders[i].compress_async(xs[i], a.eb, "rel")

    def decompress_f(i):
        decs[i].decompress_async(coders[i].out, hdrs[i], ys[i])

    def step():
        for i in range(len(xs)):
            compress_f(i)
            decompress_f(i)

    # headers (shape of the non-blocking decoder) + a correctness check of every field
    hdrs, S, errs = [], [], []
    with torch.cuda.stream(stream):
        for i in range(len(xs)):
            compress_f(i)
    stream.synchronize()
    for i, x in enumerate(xs):
        h = szx.read_header(coders[i].out[:64].cpu().numpy().tobytes())
        hdrs.append(h)
        S.append(h.stream_bytes)
        if "SZX_LIB" not in os.environ:
            yr = szx.decompress(coders[i].out[: h.stream_bytes])
            e = (yr.double() - x.double()).abs().max().item()
            assert e <= h.eb_abs, (a.fields[i], e, h.eb_abs)
            errs.append(e)
            del yr
        else:  # experiment builds (scripts/run_variants.sh) may skip work or write garbage
            errs.append(float("nan"))

    # ---- the step as one CUDA graph (falls back to eager launches if capture is refused)
    graph = None
    with torch.cuda.stream(stream):
        for _ in range(max(1, a.warmup)):
            step()
    stream.synchronize()
    if not a.no_graph:
        try:
            g = torch.cuda.CUDAGraph()
            with torch.cuda.graph(g, stream=stream):
                step()
            graph = g
        except Exception as ex:  # noqa: BLE001
            print(f"# graph capture failed ({type(ex).__name__}: {ex}); eager launches", file=sys.stderr)
            graph = None
            torch.cuda.synchronize()

    def run_step():
        if graph is not None:
            graph.replay()
        else:
            step()

    with torch.cuda.stream(stream):
        for _ in range(a.warmup):
            run_step()
    stream.synchronize()
    if torchrun:
        dist.barrier()
    torch.cuda.synchronize()
    sampler = ClockSampler(local) if rank == 0 else None
    if sampler:
        sampler.wait_first()

    # ---- timed region: K steps, CUDA events on the launching stream
    l0 = szx.launch_count()
    e_start = torch.cuda.Event(enable_timing=True)
    e_end = torch.cuda.Event(enable_timing=True)
    t_wall0 = time.time()
    with torch.cuda.stream(stream):
        e_start.record()
        for _ in range(a.steps):
            run_step()
        e_end.record()
    torch.cuda.synchronize()
    t_wall1 = time.time()
    launches_eager = szx.launch_count() - l0
    if torchrun:
        dist.barrier()
    torch.cuda.synchronize()
    total_ms = e_start.elapsed_time(e_end)
    ms_step = total_ms / a.steps
    clocks = sampler.summary(t_wall0, t_wall1) if sampler else None
    # kernels per step: counted by the library at launch (the graph's launches were counted once, at capture)
    kern_per_step = None
    l1 = szx.launch_count()
    with torch.cuda.stream(stream):
        step()
    stream.synchronize()
    kern_per_step = szx.launch_count() - l1
    gpu_launches = kern_per_step * a.steps if graph is not None else launches_eager

    # ---- phase breakdown: each field's compress and decompress captured in their
    # own CUDA graphs (as the step runs them; eager launches with --no-graph),
    # events between the phases, median over repetitions
    kb = max(5, min(a.steps, 30))
    pg = None
    if graph is not None:
        try:
            pg = []
            for i in range(len(xs)):
                gc, gd = torch.cuda.CUDAGraph(), torch.cuda.CUDAGraph()
                with torch.cuda.graph(gc, stream=stream):
                    compress_f(i)
                with torch.cuda.graph(gd, stream=stream):
                    decompress_f(i)
                pg.append((gc, gd))
        except Exception as ex:  # noqa: BLE001
            print(f"# phase graph capture failed ({type(ex).__name__}: {ex}); eager phases", file=sys.stderr)
            pg = None
            torch.cuda.synchronize()
    ph = {i: ([], []) for i in range(len(xs))}
    with torch.cuda.stream(stream):
        for _ in range(kb):
            for i in range(len(xs)):
                e0, e1, e2 = (torch.cuda.Event(enable_timing=True) for _ in range(3))
                e0.record()
                if pg is not None:
                    pg[i][0].replay()
                else:
                    compress_f(i)
                e1.record()
                if pg is not None:
                    pg[i][1].replay()
                else:
                    decompress_f(i)
                e2.record()
                ph[i][0].append((e0, e1))
                ph[i][1].append((e1, e2))
    torch.cuda.synchronize()
    comp_ms = [statistics.median([p.elapsed_time(q) for p, q in ph[i][0]]) for i in range(len(xs))]
    dec_ms = [statistics.median([p.elapsed_time(q) for p, q in ph[i][1]]) for i in range(len(xs))]
    if torchrun and world > 1:
        t = torch.tensor([ms_step] + comp_ms + dec_ms, device=dev, dtype=torch.float64)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        v = t.tolist()
        ms_step, comp_ms, dec_ms = v[0], v[1:1 + len(xs)], v[1 + len(xs):]

    # ---- per-kernel pass, per field: the library records CUDA events around every launch on
    # its launch stream (serialises the launches: a separate pass)
    kt = {}
    if not a.no_kernels:
        for i in range(len(xs)):
            szx.timing_reset()
            szx.timing_enable(True)
            with torch.cuda.stream(stream):
                for _ in range(min(a.steps, 30)):
                    compress_f(i)
                    decompress_f(i)
            torch.cuda.synchronize()
            szx.timing_enable(False)
            kt[FIELD_NAMES[a.fields[i]]] = {k: v[0] / max(v[1], 1) for k, v in szx.timing_read().items()}

    # ---- end to end through the public host API (pinned host buffers, copies inside the timed region)
    e2e = None
    if not a.no_e2e:
        xh = [x.cpu().pin_memory() for x in xs]
        sh = [torch.empty(szx.compress_bound(x.numel(), szx.F32, 128), dtype=torch.uint8, pin_memory=True)
              for x in xs]
        yh = [torch.empty(x.numel(), dtype=torch.float32, pin_memory=True) for x in xs]
        ne = max(3, min(a.steps, 8))
        tt, h2d, d2h = [], 0, 0
        for it in range(ne + 2):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            h2d = d2h = 0
            for i in range(len(xs)):
                s_h = szx.compress_host(xh[i], a.eb, "rel", 128, out=sh[i])
                szx.decompress_host(s_h, out=yh[i])
                h2d += xh[i].numel() * 4 + s_h.numel()
                d2h += s_h.numel() + yh[i].numel() * 4
            tt.append(time.perf_counter() - t0)
        e2e_s = statistics.median(tt[2:])
        if torchrun and world > 1:
            t = torch.tensor([e2e_s], device=dev, dtype=torch.float64)
            dist.all_reduce(t, op=dist.ReduceOp.MAX)
            e2e_s = t.item()
        tot_b = sum(x.numel() for x in xs) * 4 * world
        e2e = {"value": tot_b / e2e_s / 1e9, "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "api": "szx_compress_host + szx_decompress_host per field (pinned host buffers)", "steps": ne}

    cpu = None
    if rank == 0 and not a.no_cpu:
        xc = [x.cpu() for x in xs] if world == 1 else None
        if xc is not None:
            cpu = cpu_baseline(xc, a.eb, a.n)
            try:
                cpu["all_cores"] = cpu_baseline_parallel(xc, a.eb, a.n)
            except Exception as ex:  # noqa: BLE001
                cpu["all_cores"] = {"error": f"{type(ex).__name__}: {ex}"}

    if rank == 0:
        peak, peak_kind = _peaks()
        summ, summ_src = _ncu_summary()
        local_bytes = [x.numel() * 4 for x in xs]
        per = {}
        roofs = {}
        dom_all, dom_t = None, -1.0
        for i, f in enumerate(a.fields):
            fname = FIELD_NAMES[f]
            nb, Sf, h = local_bytes[i], S[i], hdrs[i]
            nnc, pb = h.n_nonconst, h.payload_bytes
            nBl = (xs[i].numel() + 127) // 128
            alg = {  # algorithmic bytes per launch
                "k_block_stats": nb + nBl * 8,
                "k_classify": nBl * 8 + nBl * 4 + nBl // 8 + 9 * nnc,
                "k_enc_size": nnc * 128 * 4 + 2 * nnc + 5 * nnc,
                "k_zscan": 2 * nnc,
                "k_enc_write": nnc * 128 * 4 + 5 * nnc + pb,
                "k_encode": nnc * 128 * 4 + 2 * nnc + pb + 4 * nBl + nBl // 8,
                "k_decode": Sf + nb,
            }
            kms = kt.get(fname, {})
            comp_alg, dec_alg = 2 * nb + Sf, Sf + nb  # REL compress: range pass + encode
            rec = {"compress_gbs": nb / (comp_ms[i] / 1e3) / 1e9, "decompress_gbs": nb / (dec_ms[i] / 1e3) / 1e9,
                   "compress_hbm_frac": comp_alg / (comp_ms[i] / 1e3) / 1e9 / peak,
                   "decompress_hbm_frac": dec_alg / (dec_ms[i] / 1e3) / 1e9 / peak,
                   "compress_ms": comp_ms[i], "decompress_ms": dec_ms[i],
                   "cr": nb / Sf, "stream_bytes": Sf, "nonconst_blocks": nnc, "blocks": nBl,
                   "nonconst_frac": nnc / max(nBl, 1), "eb_abs": h.eb_abs, "max_abs_err": errs[i],
                   "kernels_ms_per_launch": kms}
            # bytes the kernels actually moved (ncu dram read+write of the same field, committed summary)
            moved_c = moved_d = None
            if summ:
                cks = [k for k in kms if k != "k_decode"]
                vals = [_ncu_kernel(summ, fname, NCU_NAME.get(k, k)) for k in cks]
                if cks and all(v and v.get("dram_bytes") is not None for v in vals):
                    moved_c = sum(v["dram_bytes"] for v in vals)
                vd = _ncu_kernel(summ, fname, "k_decode_w")
                if vd and vd.get("dram_bytes") is not None:
                    moved_d = vd["dram_bytes"]
            rec["compress_dram_frac"] = (moved_c / (comp_ms[i] / 1e3) / 1e9 / peak) if moved_c else None
            rec["decompress_dram_frac"] = (moved_d / (dec_ms[i] / 1e3) / 1e9 / peak) if moved_d else None
            rec["dram_source"] = summ_src if (moved_c or moved_d) else None
            if kms:
                dom = max(kms, key=lambda k: kms[k])
                ach = alg.get(dom, 0) / (kms[dom] / 1e3) / 1e9
                nv = _ncu_kernel(summ, fname, NCU_NAME.get(dom, dom))
                roofs[fname] = {"kernel": dom, "bound": "hbm", "achieved": ach, "peak": peak, "unit": "GB/s",
                                "frac": ach / peak, "peak_kind": peak_kind,
                                "traffic": nv.get("dram_bytes") if nv else None,
                                "traffic_source": summ_src if nv else None,
                                "alg_bytes_per_launch": alg.get(dom), "ms_per_launch": kms[dom]}
                if nv and nv.get("inst_executed"):
                    # the same launch against the SM issue rate (warp-instructions from the
                    # committed ncu capture of this field / live launch time; peak: 4 schedulers
                    # x SMs x max clock, one warp-instruction per scheduler per cycle)
                    ipeak = 4.0 * _sm_count() * _sm_max_mhz() * 1e6
                    iach = nv["inst_executed"] / (kms[dom] / 1e3)
                    roofs[fname]["issue"] = {"achieved": iach, "peak": ipeak, "unit": "warp-inst/s",
                                             "frac": iach / ipeak, "source": summ_src}
                tot = sum(kms.values())
                if kms[dom] > dom_t:
                    dom_all, dom_t = (fname, dom), kms[dom]
            per[fname] = rec
        # dominant kernel of the whole step: the largest per-launch time over the fields
        roof = roofs.get(dom_all[0]) if dom_all else None
        if roof:
            roof = dict(roof, field=dom_all[0])
        nbytes_step = sum(local_bytes) * world
        comp_tot, dec_tot = sum(comp_ms), sum(dec_ms)
        comp_alg_tot = sum(2 * b + s for b, s in zip(local_bytes, S))
        dec_alg_tot = sum(b + s for b, s in zip(local_bytes, S))
        out = {
            "metric": METRIC, "value": nbytes_step / (ms_step / 1e3) / 1e9, "unit": UNIT, "n_gpus": world,
            "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms_step, "higher_is_better": True,
            "scaling": scaling if world > 1 else "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
            "config": _workload(a, world, scaling),
            "compress_gbs": nbytes_step / (comp_tot / 1e3) / 1e9,
            "decompress_gbs": nbytes_step / (dec_tot / 1e3) / 1e9,
            "compress_hbm_frac": comp_alg_tot / (comp_tot / 1e3) / 1e9 / peak,
            "decompress_hbm_frac": dec_alg_tot / (dec_tot / 1e3) / 1e9 / peak,
            "cr": sum(local_bytes) / sum(S), "stream_bytes": sum(S),
            "roofline": roof, "roofline_per_field": roofs, "fields": per, "cpu_baseline": cpu, "e2e": e2e,
            "gpu_launches": gpu_launches, "kernels_per_step": kern_per_step, "graph": graph is not None,
            "clocks": clocks,
            "timing": "value/ms_per_step: CUDA events around K replays of the step's CUDA graph (eager if "
                      "graph=false); fields.*: events around each field's compress / decompress CUDA graph (eager with --no-graph), "
                      "median of the repetitions; kernels_ms_per_launch / "
                      "roofline: library CUDA events around each launch in a third pass",
            "paper_context": "cuSZx A100: 150-216 GB/s compress, 150-291 GB/s decompress (P:L3207-3220)",
        }
        print(json.dumps(out), flush=True)
    if torchrun:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
