"""A/B per-call comparison of library variants selected by environment knobs (development
tool, not the benchmark).

    python tools/ab_calls.py --variant A "" --variant B "IPT_ROW_PIPE=0" [--shapes 48] [--eb 4 8]

For every sweep shape, element size and direction, each variant's call is timed (CUDA
events, L2 flushed, median of --reps) with per-kernel-kind event times.  Prints one JSON
line per call and a summary per class (gcd 1 / fused rotation / separate rotation) of the
row-pass, column-pass and whole-call GB/s medians of each variant.
"""
import argparse
import json
import math
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402
import workloads  # noqa: E402


def set_env(spec):
    for kv in filter(None, spec.split(",")):
        k, v = kv.split("=")
        os.environ[k] = v


def clear_env(spec):
    for kv in filter(None, spec.split(",")):
        os.environ.pop(kv.split("=")[0], None)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--variant", nargs=2, action="append", metavar=("NAME", "ENV"), required=True)
    p.add_argument("--shapes", type=int, default=48)
    p.add_argument("--eb", type=int, nargs="+", default=[4, 8])
    p.add_argument("--reps", type=int, default=3)
    p.add_argument("--quiet", action="store_true")
    p.add_argument("--no-kernels", action="store_true", help="no per-kernel events (they separate the launches)")
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    summary = {}
    for (m, n) in workloads.sweep_shapes(a.shapes):
        for eb in a.eb:
            x = torch.empty(m * n * eb, dtype=torch.uint8, device="cuda")
            for opn in ("c2r", "r2c"):
                op = getattr(ipt, opn)
                info = ipt.plan_info(m, n, eb) if opn == "c2r" else ipt.plan_info(n, m, eb)
                cls = "gcd1" if info["c"] == 1 else ("fused" if info["launches"] == 2 else "rot")
                rec = {"m": m, "n": n, "eb": eb, "op": opn, "gcd": math.gcd(m, n), "class": cls,
                       "row_bytes": info["N"] * eb}
                for name, env in a.variant:
                    set_env(env)
                    op(x, m, n, elem_bytes=eb)
                    torch.cuda.synchronize()
                    ipt.profile_enable(not a.no_kernels)
                    ipt.profile_read()
                    ts = []
                    for _ in range(a.reps):
                        flush.zero_()
                        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                        e0.record()
                        op(x, m, n, elem_bytes=eb)
                        e1.record()
                        torch.cuda.synchronize()
                        ts.append(e0.elapsed_time(e1))
                    prof = ipt.profile_read()
                    ipt.profile_enable(False)
                    clear_env(env)
                    med = statistics.median(ts)
                    kern = {k: round(v[2] / v[1] / 1e6, 1) for k, v in prof.items() if v[0] and v[1]}
                    rec[name] = {"GBps": round(2 * m * n * eb / med / 1e6, 1), **kern}
                    for key, val in [("call", rec[name]["GBps"])] + list(kern.items()):
                        summary.setdefault((cls, name, key), []).append(val)
                        summary.setdefault(("all", name, key), []).append(val)
                if not a.quiet:
                    print(json.dumps(rec), flush=True)
            del x
            torch.cuda.empty_cache()
    for (cls, name, key), v in sorted(summary.items()):
        print(f"SUMMARY {cls:6s} {name:10s} {key:12s} n={len(v):4d} median={statistics.median(v):8.1f}", flush=True)


if __name__ == "__main__":
    main()
