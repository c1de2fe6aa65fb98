#!/usr/bin/env python3
"""Benchmark of the B200 decomposed in-place transpose (driver contract).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--impl ours|reference]

Workload (BASELINE.json configs[1], the metric's configuration): the paper's GPU sweep
(Table 2) -- random m, n uniform in [1000, 20000] (workloads.sweep_shapes,
seed 20140215), 4-byte (float32) and 8-byte (float64) elements, row-major.  One STEP is
one in-place transpose of every one of the S shapes in both element sizes through the C
ABI (ipt_c2r on even steps, ipt_r2c on odd steps, so both directions are timed and the
data stay meaningful).  Every call is timed alone with CUDA events on the launching
stream; L2 is flushed (a 256 MiB write, > the 126 MB L2) before every timed call, outside
the events.  Throughput per call follows Eq. 37: 2 m n s / t, GB = 1e9 B.

value   = median over all timed calls of the per-call GB/s (the paper's statistic).  With N
          ranks every rank runs the SAME S shapes (weak scaling, no collective on the data
          path); call k's time is the max over ranks and its GB/s is N x 2 m n s / that time.
moved   = the same median over the call's algorithmic bytes (4 m n s for two passes).
extras  = cfg5b (batch of 4096 4096x3000 fp32, sharded over the ranks; strong scaling),
          cfg3 (skinny AoS<->SoA, median over n) and cfg5a (~140 GB fp64) at N = 1.
e2e     = Eq. 37 bytes of a step of ipt_c2r_host calls (C ABI, pinned host buffers: H2D,
          transpose, D2H) over the step's device time, calls round-robin over 4 streams.
roofline= the dominant kernel's algorithmic bytes / its event-timed device time against
          the measured HBM copy bandwidth (MEASURED_PEAKS.json); the per-launch events run in a
          replica of two timed steps right after the timed region (--kernel-events).
cpu_baseline = the C oracle's Algorithm 1 (oracle/, single thread) on a bounded sample.

--impl reference: the reference arm of this tier is the oracle itself (the paper ships no
code): rank 0 times oracle Algorithm 1 on host cores, one sweep shape per step.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import subprocess
import sys
import tempfile
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

import workloads  # noqa: E402

METRIC = "median in-place transpose GB/s over random m×n; fraction of B200 HBM peak"
UNIT = "GB/s"
FALLBACK_HBM_GBS = 6650.0  # B200_PROFILING.md fallback, used only without MEASURED_PEAKS.json
FLUSH_BYTES = 256 << 20
REF_MAX_ELEMS = 40_000_000  # reference-arm sample: sweep shapes with m*n <= this


def parse_args():
    p = argparse.ArgumentParser()
    p.add_argument("--gpus", type=int, default=1)
    p.add_argument("--steps", type=int, default=6)
    p.add_argument("--warmup", type=int, default=3)
    p.add_argument("--impl", choices=("ours", "reference"), default="ours")
    p.add_argument("--shapes", type=int, default=200, help="sweep shapes per step (the same on every rank)")
    p.add_argument("--no-extras", action="store_true", help="skip the cfg3 / cfg5a / cfg5b keys")
    p.add_argument("--kernel-events", choices=("timed", "replica"), default="replica",
                   help="per-kernel CUDA events in a replica of 2 timed steps right after the timed region "
                        "(default) or inside the timed calls (they then add ~3.5 %% to the call times)")
    p.add_argument("--e2e-shapes", type=int, default=8)
    p.add_argument("--no-cpu-baseline", action="store_true")
    p.add_argument("--profile-only", action="store_true", help="one short untimed pass (for ncu)")
    p.add_argument("--config", choices=("sweep", "batched", "skinny"), default="sweep",
                   help="sweep: BASELINE configs[1] (the metric's workload); batched: config 5b; "
                        "skinny: config 3")
    p.add_argument("--count", type=int, default=1 << 26, help="config 3 structs")
    p.add_argument("--batch", type=int, default=4096, help="config 5b total matrices")
    p.add_argument("--chunk", type=int, default=512, help="config 5b resident matrices per call")
    return p.parse_args()


def hbm_peak():
    path = os.path.join(ROOT, "MEASURED_PEAKS.json")
    try:
        with open(path) as f:
            return float(json.load(f)["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    except Exception:
        return FALLBACK_HBM_GBS, "fallback (B200_PROFILING.md)"


def ncu_traffic():
    """Per-launch DRAM bytes of the captured kernels (profiles/ncu_summary.json), if any."""
    path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    try:
        with open(path) as f:
            return json.load(f)
    except Exception:
        return {}


class Clocks:
    """nvidia-smi sampling during the timed region (B200_PROFILING.md clocks line)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
         "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
         "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu_id: str):
        self.gpu_id = gpu_id
        self.proc = None
        self.tmp = tempfile.NamedTemporaryFile("w+", suffix=".csv", delete=False)

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "100", "-i", self.gpu_id], stdout=self.tmp,
                                         stderr=subprocess.DEVNULL)
        except Exception:
            self.proc = None

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        self.proc.wait()
        self.tmp.flush()
        rows = []
        with open(self.tmp.name) as f:
            for line in f:
                v = [x.strip() for x in line.split(",")]
                if len(v) >= 9 and v[1].isdigit():
                    rows.append(v)
        os.unlink(self.tmp.name)
        if not rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["no samples"]}
        sm = [int(r[1]) for r in rows]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in rows for k in range(4) if r[5 + k].lower().startswith("active")})
        return {"sm_mhz": statistics.median(sm), "sm_max_mhz": int(rows[0][2]), "reasons": reasons,
                "samples": len(rows), "power_w_max": max(float(r[3]) for r in rows if r[3].replace(".", "").isdigit())
                if any(r[3].replace(".", "").isdigit() for r in rows) else None}


def cpu_info():
    try:
        cores = len(os.sched_getaffinity(0))
    except Exception:
        cores = os.cpu_count()
    model = ""
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except Exception:
        pass
    return cores, model


def oracle_step(shape, eb, seed):
    """One oracle Algorithm 1 C2R on host; returns (seconds, bytes)."""
    import oracle
    m, n = shape
    host = workloads.random_words(m * n, eb, seed)
    t0 = time.perf_counter()
    oracle.c2r_alg1(host, m, n)
    dt = time.perf_counter() - t0
    return dt, 2.0 * m * n * eb


def reference_sample_shapes(k):
    out = []
    for s in workloads.sweep_shapes(4096):
        if s[0] * s[1] <= REF_MAX_ELEMS:
            out.append(s)
        if len(out) >= k:
            break
    return out


def cpu_baseline(budget_s=20.0):
    """The oracle as it stands (single-threaded C, Algorithm 1), fp32, on sweep shapes until
    ~budget_s of CPU work."""
    cores, model = cpu_info()
    shapes, t_tot, rates = [], 0.0, []
    for k, s in enumerate(workloads.sweep_shapes(64)):
        dt, by = oracle_step(s, 4, seed=k)
        shapes.append(s)
        rates.append(by / dt / 1e9)
        t_tot += dt
        if t_tot >= budget_s:
            break
    return {"value": round(statistics.median(rates), 4), "unit": UNIT, "cores": 1, "kind": "oracle",
            "host_cores_available": cores, "cpu_model": model,
            "sample": f"oracle Algorithm 1 C2R, float32, first {len(shapes)} cfg2 sweep shapes {shapes}, "
                      f"{t_tot:.1f} s CPU; median of per-shape Eq. 37 GB/s"}


def cpu_tuned(budget_s=8.0):
    """the tuned parallel CPU C2R (cpu_baseline/, OpenMP, gather form, column
    panels) on the same sweep shapes, fp32, until ~budget_s of wall time; median Eq. 37 GB/s.
    A stronger CPU reference point than the oracle; not the product and not the oracle."""
    try:
        import numpy as np
        import cpu_baseline
        rates, shapes, t_tot = [], [], 0.0
        for k, (m, n) in enumerate(workloads.sweep_shapes(64)):
            X = workloads.random_words(m * n, 4, seed=k)
            t0 = time.perf_counter()
            cpu_baseline.c2r(X, m, n)
            dt = time.perf_counter() - t0
            rates.append(2 * m * n * 4 / dt / 1e9)
            shapes.append((m, n))
            t_tot += dt
            del X
            if t_tot >= budget_s:
                break
        return {"value": round(statistics.median(rates), 3), "unit": UNIT, "cores": cpu_baseline.threads(),
                "kind": "tuned-openmp", "sample": f"cpu_baseline C2R float32, first {len(shapes)} cfg2 sweep shapes, "
                f"{t_tot:.1f} s; median of per-shape Eq. 37 GB/s"}
    except Exception as e:  # a baseline must never sink the bench line
        return {"unavailable": f"{type(e).__name__}: {e}"}


def run_reference(args, rank, world):
    if rank != 0:
        return
    shapes = reference_sample_shapes(max(1, args.steps + args.warmup))
    for k in range(args.warmup):
        oracle_step(shapes[k % len(shapes)], 4, seed=k)
    rates, secs = [], []
    for k in range(args.steps):
        s = shapes[(args.warmup + k) % len(shapes)]
        dt, by = oracle_step(s, 4, seed=100 + k)
        rates.append(by / dt / 1e9)
        secs.append(dt)
    cores, model = cpu_info()
    value = statistics.median(rates)
    sample = (f"oracle Algorithm 1 C2R (single thread), float32, one cfg2 sweep shape per step "
              f"(shapes with m*n <= {REF_MAX_ELEMS}), {sum(secs):.1f} s CPU")
    out = {"metric": METRIC, "value": round(value, 4), "unit": UNIT, "n_gpus": args.gpus, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(1e3 * statistics.mean(secs), 3), "higher_is_better": True,
           "scaling": "weak", "vs_baseline": None, "dtype": "f32", "data": "synthetic",
           "config": {"workload": "cfg2 paper sweep m,n~U[1000,20000] (reference arm: CPU oracle sample)",
                      "seed": workloads.SWEEP_SEED},
           "impl": "reference",
           "cpu_baseline": {"value": round(value, 4), "unit": UNIT, "cores": 1, "kind": "oracle", "sample": sample,
                            "host_cores_available": cores, "cpu_model": model},
           "e2e": {"value": round(value, 4), "unit": UNIT, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(out), flush=True)


def rank_shapes(rank, S):
    """Every rank transposes the SAME S sweep shapes (so that N=1 and N>1 time the same
    workload per GPU; weak scaling: the job's work grows with N, no data-path collective)."""
    return workloads.sweep_shapes(S)


def shard_batch(batch, rank, world):
    """Contiguous block of matrix indices [lo, hi) owned by `rank` (config 5b)."""
    lo = batch * rank // world
    hi = batch * (rank + 1) // world
    return lo, hi


def reduce_over_ranks(sum_vals, max_vals, world, device):
    """The bench's only collectives: SUM of sum_vals and MAX of max_vals over ranks
    (no collective ever touches the data path)."""
    if world == 1:
        return list(sum_vals), list(max_vals)
    import torch
    import torch.distributed as dist
    out = []
    for vals, op in ((sum_vals, dist.ReduceOp.SUM), (max_vals, dist.ReduceOp.MAX)):
        vals = list(vals)
        if vals:
            t = torch.tensor(vals, dtype=torch.float64, device=device)
            dist.all_reduce(t, op=op)
            vals = [float(v) for v in t]
        out.append(vals)
    return out[0], out[1]


def aggregate_calls(call_bytes, call_ms, world, device):
    """Multi-GPU semantics of the sweep metric.  Every rank runs the same calls in the same
    order; call k's job time is the MAX over ranks of its device time, and its job
    throughput is (world x its Eq. 37 bytes) / that time.  value = the median over calls
    (at world = 1: the plain per-call median, the paper's statistic).  Also returns the
    aggregate throughput = all ranks' bytes / the max over ranks of the summed device time."""
    _, t_max = reduce_over_ranks([], list(call_ms), world, device)
    per_call = [world * b / (t * 1e-3) / 1e9 for b, t in zip(call_bytes, t_max)]
    _, (tot_max,) = reduce_over_ranks([], [sum(call_ms)], world, device)
    aggregate = world * sum(call_bytes) / (tot_max * 1e-3) / 1e9
    return per_call, t_max, aggregate


def algorithmic_bytes(ipt, m, n, eb, op):
    """What the engine must move for one call: one read + one write of every
    element per pass -- 4 m n s for two passes (gcd 1, or the rotation fused), plus
    2 m n s (c - 1) / c for a separate rotation pass."""
    info = ipt.plan_info(m, n, eb) if op == "c2r" else ipt.plan_info(n, m, eb)
    c = info["c"]
    extra = 2.0 * (c - 1) / c if info["launches"] >= 3 and info["engine"] in ("c2r", "r2c") else 0.0
    return (4.0 + extra) * m * n * eb


def measure_batched(args, rank, world, local_rank, steps=2, warmup=1):
    """Config 5b: `args.batch` independent 4096 x 3000 float32 matrices (default 4096, 201 GB)
    sharded contiguously over the ranks (strong scaling); each rank transposes its shard with
    ipt_c2r_batched / ipt_r2c_batched in resident chunks of at most --chunk matrices (one GPU
    cannot hold 201 GB: the chunks reuse one 25 GB buffer).  value = total Eq. 37 bytes /
    max-over-ranks device time."""
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_catanzarokg14_b200 as ipt

    dev = torch.device("cuda", local_rank)
    m, n, eb = workloads.CONFIG5B["m"], workloads.CONFIG5B["n"], workloads.CONFIG5B["elem_bytes"]
    lo, hi = shard_batch(args.batch, rank, world)
    mine = hi - lo
    chunk = min(args.chunk, mine) if mine else 0
    buf = torch.randint(0, 255, (max(chunk, 1) * m * n * eb,), dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)
    pieces = []
    k = 0
    while k < mine:
        pieces.append(min(chunk, mine - k))
        k += chunk

    def step(record):
        for i, cnt in enumerate(pieces):
            e0 = torch.cuda.Event(enable_timing=True)
            e1 = torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            (ipt.c2r_batched if i % 2 == 0 else ipt.r2c_batched)(buf, cnt, m * n, m, n, elem_bytes=eb,
                                                                 stream=stream.cuda_stream)
            e1.record(stream)
            if record is not None:
                record.append((e0, e1))

    for _ in range(warmup):
        step(None)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    launches0 = ipt.launch_count()
    rec = []
    for _ in range(steps):
        step(rec)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    dev_ms = sum(e0.elapsed_time(e1) for e0, e1 in rec) / steps
    (total_bytes,), (t_max,) = reduce_over_ranks([2.0 * mine * m * n * eb], [dev_ms], world, dev)
    del buf
    torch.cuda.empty_cache()
    peak, _ = hbm_peak()
    value = total_bytes / (t_max * 1e-3) / 1e9
    return {"value": round(value, 2), "unit": UNIT, "metric": "Eq. 37 GB/s of the whole batch (2 m n s per matrix)",
            "n_gpus": world, "scaling": "strong", "ms_per_step": round(t_max, 3), "steps": steps,
            "workload": f"cfg5b: {args.batch} independent {m}x{n} float32 matrices, contiguous shards per rank, "
                        f"chunks of <= {args.chunk} resident matrices (c2r / r2c alternating)",
            "frac_of_hbm_peak_per_gpu": round(value / world / peak, 4),
            "moved_GBps": round(2 * value, 2), "gpu_launches": ipt.launch_count() - launches0}


def measure_skinny(args, local_rank, steps=1, warmup=1):
    """Config 3: AoS -> SoA and SoA -> AoS of args.count structs x n 4-byte fields, n = 2..32
    (ipt_aos_to_soa / ipt_soa_to_aos, the skinny engine).  value = median over all calls of
    Eq. 37 GB/s (2 * count * n * 4 / t); per-n medians; per-kernel event times."""
    import torch

    import paper_conf_ppopp_catanzarokg14_b200 as ipt

    dev = torch.device("cuda", local_rank)
    count = args.count
    ns = workloads.skinny_field_counts()
    buf = torch.randint(0, 255, (count * max(ns) * 4,), dtype=torch.uint8, device=dev)
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)

    def one(n, op, rec):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        op(buf, count, n, field_bytes=4, stream=stream.cuda_stream)
        e1.record(stream)
        if rec is not None:
            rec.append((n, op.__name__, e0, e1))

    for _ in range(warmup):
        for n in ns:
            one(n, ipt.aos_to_soa, None)
            one(n, ipt.soa_to_aos, None)
    torch.cuda.synchronize()
    launches0 = ipt.launch_count()
    ipt.profile_enable(True)
    ipt.profile_read()
    rec = []
    for _ in range(steps):
        for n in ns:
            one(n, ipt.aos_to_soa, rec)
            one(n, ipt.soa_to_aos, rec)
    torch.cuda.synchronize()
    ipt.profile_enable(False)
    kern = ipt.profile_read()
    rates, per_n, dev_ms = [], {}, 0.0
    for n, name, e0, e1 in rec:
        ms = e0.elapsed_time(e1)
        dev_ms += ms
        g = 2.0 * count * n * 4 / (ms * 1e-3) / 1e9
        rates.append(g)
        per_n.setdefault(f"{name}_n{n}", []).append(g)
    del buf, flush
    torch.cuda.empty_cache()
    peak, _ = hbm_peak()
    value = statistics.median(rates)
    return {"value": round(value, 2), "unit": UNIT, "metric": "median in-place AoS<->SoA GB/s (Eq. 37) over n = 2..32",
            "workload": f"cfg3 skinny: {count} structs x n 4-byte fields, n = 2..32, ipt_aos_to_soa then "
                        "ipt_soa_to_aos, L2 flushed before every call",
            "frac_of_hbm_peak": round(value / peak, 4), "max_GBps": round(max(rates), 2),
            "ceiling_note": "(2 + 1/n) passes for odd n, 3 for even n: eff <= copy / (2 + 1/n) or copy / 3",
            "per_n": {k: round(statistics.median(v), 1) for k, v in per_n.items()},
            "kernels": {k: {"launches": v[0], "ms": round(v[1], 3), "GBps": round(v[2] / (v[1] * 1e-3) / 1e9, 1)}
                        for k, v in kern.items()},
            "ms_per_step": round(dev_ms / steps, 3), "gpu_launches": ipt.launch_count() - launches0}


def measure_huge(local_rank, shapes=((120011, 145820), (125000, 140000)), eb=8):
    """Config 5a: in-place transpose of ~140 GB float64 matrices on one GPU (c2r then r2c,
    one warm-up pair, one timed pair per shape).  Skipped when the device lacks the memory."""
    import torch

    import paper_conf_ppopp_catanzarokg14_b200 as ipt

    dev = torch.device("cuda", local_rank)
    torch.cuda.empty_cache()
    out = {}
    stream = torch.cuda.current_stream(dev)
    for (m, n) in shapes:
        free, _ = torch.cuda.mem_get_info(dev)
        need = m * n * eb
        key = f"{m}x{n}"
        if free < need + (3 << 30):
            out[key] = {"skipped": f"needs {need / 1e9:.1f} GB, {free / 1e9:.1f} GB free"}
            continue
        x = torch.empty(need, dtype=torch.uint8, device=dev)
        ipt.c2r(x, m, n, elem_bytes=eb)
        ipt.r2c(x, m, n, elem_bytes=eb)
        torch.cuda.synchronize()
        ipt.profile_enable(True)
        ipt.profile_read()
        res = {}
        for op in ("c2r", "r2c"):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record(stream)
            getattr(ipt, op)(x, m, n, elem_bytes=eb, stream=stream.cuda_stream)
            e1.record(stream)
            e1.synchronize()
            ms = e0.elapsed_time(e1)
            res[op + "_GBps"] = round(2.0 * m * n * eb / (ms * 1e-3) / 1e9, 1)
            res[op + "_ms"] = round(ms, 2)
        ipt.profile_enable(False)
        kern = ipt.profile_read()
        info = ipt.plan_info(m, n, eb)
        res.update({"bytes": need, "gcd": info["c"], "engine": info["engine"], "row_cluster_K": info["row_cluster"],
                    "launches": info["launches"], "scratch_bytes": info["scratch_bytes"],
                    "kernels": {k: {"launches": v[0], "ms": round(v[1], 3),
                                    "GBps": round(v[2] / (v[1] * 1e-3) / 1e9, 1)} for k, v in kern.items()}})
        out[key] = res
        del x
        torch.cuda.empty_cache()
    return {"workload": "cfg5a: 120011x145820 (gcd 1) and 125000x140000 (gcd 5000) float64, ~140 GB each, "
                        "one GPU; Eq. 37 GB/s per call (device events)", "shapes": out}


def run_batched(args, rank, world, local_rank):
    import torch
    torch.cuda.set_device(local_rank)
    res = measure_batched(args, rank, world, local_rank, steps=args.steps, warmup=args.warmup)
    if rank == 0:
        print(json.dumps({"metric": METRIC, "value": res["value"], "unit": UNIT, "n_gpus": world,
                          "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
                          "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "f32",
                          "data": "synthetic", "config": {"workload": res["workload"]}, "impl": "ours",
                          "frac_of_hbm_peak_per_gpu": res["frac_of_hbm_peak_per_gpu"],
                          "gpu_launches": res["gpu_launches"]}), flush=True)


def run_skinny(args, rank, world, local_rank):
    import torch
    torch.cuda.set_device(local_rank)
    res = measure_skinny(args, local_rank, steps=args.steps, warmup=args.warmup)
    if rank == 0:
        print(json.dumps({"metric": res["metric"], "value": res["value"], "unit": UNIT, "n_gpus": world,
                          "steps": args.steps, "warmup": args.warmup, "ms_per_step": res["ms_per_step"],
                          "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "f32",
                          "data": "synthetic", "config": {"workload": res["workload"]}, "impl": "ours",
                          **{k: v for k, v in res.items() if k not in ("value", "metric", "workload", "ms_per_step")}}),
              flush=True)


def run_ours(args, rank, world, local_rank):
    import torch
    import torch.distributed as dist

    import paper_conf_ppopp_catanzarokg14_b200 as ipt

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    S = args.shapes
    shapes = rank_shapes(rank, S)
    ebs = (4, 8)
    maxel = max(m * n for m, n in shapes)
    bufs = {eb: torch.randint(0, 255, (maxel * eb,), dtype=torch.uint8, device=dev) for eb in ebs}
    flush = torch.empty(FLUSH_BYTES, dtype=torch.uint8, device=dev)
    stream = torch.cuda.current_stream(dev)
    alg = {}
    for (m, n) in shapes:
        for eb in ebs:
            for op in ("c2r", "r2c"):
                alg[(m, n, eb, op)] = algorithmic_bytes(ipt, m, n, eb, op)

    def one_step(step, record):
        opn = "c2r" if step % 2 == 0 else "r2c"
        op = getattr(ipt, opn)
        for (m, n) in shapes:
            for eb in ebs:
                flush.zero_()
                if record is not None:
                    e0 = torch.cuda.Event(enable_timing=True)
                    e1 = torch.cuda.Event(enable_timing=True)
                    e0.record(stream)
                op(bufs[eb], m, n, elem_bytes=eb, stream=stream.cuda_stream)
                if record is not None:
                    e1.record(stream)
                    record.append((m, n, eb, opn, e0, e1))

    if args.profile_only:
        one_step(0, None)
        torch.cuda.synchronize()
        return

    for w in range(args.warmup):
        one_step(w, None)
    torch.cuda.synchronize()

    gpu_id = "GPU-" + str(torch.cuda.get_device_properties(dev).uuid) if hasattr(
        torch.cuda.get_device_properties(dev), "uuid") else str(local_rank)
    clocks = Clocks(gpu_id)
    if world > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    time.sleep(0.3)
    launches0 = ipt.launch_count()
    profiled = args.kernel_events == "timed"
    ipt.profile_enable(profiled)
    ipt.profile_read()
    rec = []
    t_wall = time.perf_counter()
    for k in range(args.steps):
        one_step(args.warmup + k, rec)
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    t_wall = time.perf_counter() - t_wall
    ipt.profile_enable(False)
    kern = ipt.profile_read()
    launches = ipt.launch_count() - launches0
    clk = clocks.stop()
    if not profiled:
        # per-kernel attribution from a replica of two timed steps (one c2r, one r2c), so that
        # the per-launch event records do not sit inside the timed calls
        ipt.profile_enable(True)
        ipt.profile_read()
        for k in range(2):
            one_step(args.warmup + k, None)
        torch.cuda.synchronize()
        ipt.profile_enable(False)
        kern = ipt.profile_read()

    call_ms = [e0.elapsed_time(e1) for (_, _, _, _, e0, e1) in rec]
    call_bytes = [2.0 * m * n * eb for (m, n, eb, _, _, _) in rec]
    per_call, t_max, aggregate = aggregate_calls(call_bytes, call_ms, world, dev)
    moved = [world * alg[(m, n, eb, op)] / (t * 1e-3) / 1e9 for (m, n, eb, op, _, _), t in zip(rec, t_max)]
    by_eb = {eb: [g for g, r in zip(per_call, rec) if r[2] == eb] for eb in ebs}
    value = statistics.median(per_call)
    ms_step = sum(t_max) / args.steps

    # ---- e2e through the public API with host buffers --------------------------------
    # ipt_c2r_host (host -> device, transpose, device -> host, stream-ordered) on every e2e
    # shape, consecutive calls round-robin over NS streams and device buffers, so that one
    # call's device->host copy overlaps the next calls' host->device copies (the two directions
    # of the host link).  E = all Eq. 37 bytes of the step / the step's device time (first
    # copy in to last copy out); median of 3 steps after one warm-up step.
    e2e_shapes = [(m, n, eb) for eb in ebs for (m, n) in shapes[:args.e2e_shapes]]
    big = max(m * n * eb for m, n, eb in e2e_shapes)
    # calls in flight (tools/e2e_streams.py: 1 / 2 / 3 / 4 streams -> 54 / 71 / 81 / 84 GB/s); 2 per
    # rank at N > 1, so that the pinned host buffers (NS x the largest matrix) stay modest per node
    NS = 4 if world == 1 else 2
    hosts = [torch.empty(big, dtype=torch.uint8, pin_memory=True).random_(0, 255) for _ in range(NS)]
    devs = [torch.empty(big, dtype=torch.uint8, device=dev) for _ in range(NS)]
    sts = [stream] + [torch.cuda.Stream(device=dev) for _ in range(NS - 1)]
    e2e_rates = []
    step_bytes = sum(2.0 * m * n * eb for m, n, eb in e2e_shapes)
    h2d = sum(m * n * eb for m, n, eb in e2e_shapes)
    for rep in range(4):
        torch.cuda.synchronize()
        e0, e1 = (torch.cuda.Event(enable_timing=True) for _ in range(2))
        e0.record(sts[0])
        for st_ in sts[1:]:
            st_.wait_event(e0)
        for k, (m, n, eb) in enumerate(e2e_shapes):
            # call k + NS reuses call k's buffers on the same stream, after its D2H
            ipt.c2r_host(hosts[k % NS][:m * n * eb], devs[k % NS], m, n, elem_bytes=eb, stream=sts[k % NS].cuda_stream)
        for st_ in sts[1:]:
            ev = torch.cuda.Event()
            ev.record(st_)
            sts[0].wait_event(ev)
        e1.record(sts[0])
        e1.synchronize()
        if rep > 0:
            e2e_rates.append(step_bytes / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    e2e_med = statistics.median(e2e_rates)
    (e2e_sum,), _ = reduce_over_ranks([e2e_med], [], world, dev)
    e2e = {"value": round(e2e_sum, 2), "unit": UNIT, "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": h2d,
           "statistic": "all Eq. 37 bytes of the step / its device time (first H2D to last D2H), median of 3 steps, "
                        "summed over ranks",
           "note": f"ipt_c2r_host on pinned host buffers (C ABI: H2D, transpose, D2H), {len(e2e_shapes)} calls per step "
                   f"(first {args.e2e_shapes} sweep shapes x {'/'.join('fp%d' % (8 * e) for e in ebs)}), round-robin over "
                   f"{NS} streams and device buffers so D2H of one call overlaps H2D of the next; bound by the host link "
                   "(H2D 38, D2H 52 GB/s alone)"}
    del hosts, devs
    del bufs, flush
    torch.cuda.empty_cache()

    # ---- the other BASELINE configs, folded into the same line ------------------------
    extras = {}
    if not args.no_extras:
        extras["cfg5b_batched"] = measure_batched(args, rank, world, local_rank)
        if world == 1:
            extras["cfg3_skinny"] = measure_skinny(args, local_rank)
            extras["cfg5a_huge"] = measure_huge(local_rank)
    if rank != 0:
        return

    peak, peak_src = hbm_peak()
    dom = max(kern.items(), key=lambda kv: kv[1][1]) if kern else None
    roof = None
    if dom:
        name, (nl, ms, by) = dom
        achieved = by / (ms * 1e-3) / 1e9
        tr = ncu_traffic().get(name)
        roof = {"bound": "hbm", "kernel": name, "achieved": round(achieved, 1), "peak": peak, "unit": "GB/s",
                "frac": round(achieved / peak, 4), "peak_source": peak_src,
                "traffic": tr.get("dram_bytes_per_launch") if tr else None,
                "traffic_algorithmic": tr.get("algorithmic_bytes_per_launch") if tr else None,
                "traffic_source": tr.get("source") if tr else None,
                "launches": nl, "share_of_device_time": round(ms / sum(v[1] for v in kern.values()), 3)}
    kernels = {k: {"launches": v[0], "ms": round(v[1], 3), "GBps": round(v[2] / (v[1] * 1e-3) / 1e9, 1),
                   "frac_of_hbm_peak": round(v[2] / (v[1] * 1e-3) / 1e9 / peak, 4)}
               for k, v in kern.items()}
    moved_med = statistics.median(moved)
    out = {"metric": METRIC, "value": round(value, 2), "unit": UNIT, "n_gpus": world, "steps": args.steps,
           "warmup": args.warmup, "ms_per_step": round(ms_step, 3), "higher_is_better": True, "scaling": "weak",
           "vs_baseline": None, "dtype": "f32+f64", "data": "synthetic",
           "config": {"workload": "cfg2 paper sweep: m,n ~ U[1000,20000] (seed 20140215), row-major, "
                                  "float32+float64, ipt_c2r/ipt_r2c alternating steps",
                      "shapes_per_rank": S, "elem_bytes": list(ebs), "calls_per_step": S * len(ebs),
                      "l2": "flushed before every timed call (256 MiB write > 126 MB L2)",
                      "parallelism": f"replicas x{world}: every rank runs the same shapes; per call the max over "
                                     "ranks of its device time (no data-path collective)",
                      "engine": "paper heuristic PAPER.md:959 (C2R if m > n else R2C)",
                      "kernel_events": ("inside the timed calls" if args.kernel_events == "timed" else
                                        "CUDA events around every launch (on its stream) in a replica of 2 of the "
                                        "timed steps, same calls and order, run right after the timed region; the "
                                        "timed calls carry no per-kernel events (they would add ~3.5 % to the call "
                                        "times: 2367 vs 2455 GB/s, gpurun_out r02x)")},
           "impl": "ours",
           "statistic": "median over calls of Eq. 37 GB/s = world x 2 m n s / max-over-ranks call time "
                        "(PAPER.md:789-795, GB = 1e9 B)",
           "median_GBps_fp32": round(statistics.median(by_eb[4]), 2),
           "median_GBps_fp64": round(statistics.median(by_eb[8]), 2),
           "p10_GBps": round(sorted(per_call)[len(per_call) // 10], 2),
           "p90_GBps": round(sorted(per_call)[(9 * len(per_call)) // 10], 2),
           "aggregate_GBps": round(aggregate, 2),
           "frac_of_hbm_peak": round(value / world / peak, 4),
           "frac_of_spec_8TBps": round(value / world / 8000.0, 4),
           "moved_GBps": round(moved_med, 2),
           "moved_frac_of_hbm_peak": round(moved_med / world / peak, 4),
           "moved_frac_of_spec_8TBps": round(moved_med / world / 8000.0, 4),
           "moved_note": "algorithmic bytes of the call's passes (4 m n s, + 2 m n s (c-1)/c for a separate "
                         "rotation) / call time, median over calls; 2-pass ceiling of Eq. 37 = 50% of copy",
           "paper_context": {"K20c_median_GBps_fp64": 19.53, "K20c_median_GBps_fp32": 14.23,
                             "source": "PAPER.md:1027-1033 Table 2 (other hardware; context only)"},
           "roofline": roof, "kernels": kernels, "gpu_launches": launches, "e2e": e2e, "clocks": clk,
           "wall_s_timed_region": round(t_wall, 3)}
    out.update(extras)
    if world == 1 and not args.no_cpu_baseline:
        out["cpu_baseline"] = cpu_baseline()
        out["cpu_tuned"] = cpu_tuned()
    print(json.dumps(out), flush=True)


def main():
    args = parse_args()
    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if world > 1:
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
    try:
        if args.config == "batched":
            run_batched(args, rank, world, local_rank)
        elif args.config == "skinny":
            run_skinny(args, rank, world, local_rank)
        else:
            run_ours(args, rank, world, local_rank)
    finally:
        if world > 1:
            import torch.distributed as dist
            dist.destroy_process_group()


if __name__ == "__main__":
    main()
