"""Per-call Eq. 37 GB/s of the bench sweep shapes (development tool, not the benchmark).

    python tools/sweep_calls.py [--shapes 48] [--eb 4 8] [--reps 3]

One JSON line per (shape, eb, op): gcd, plan summary, median Eq. 37 GB/s (CUDA events, L2
flushed before each call) and per-kernel-kind device time.
"""
import argparse
import json
import math
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402
import workloads  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--shapes", type=int, default=48)
    p.add_argument("--eb", type=int, nargs="+", default=[4, 8])
    p.add_argument("--reps", type=int, default=3)
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for (m, n) in workloads.sweep_shapes(a.shapes):
        for eb in a.eb:
            x = torch.empty(m * n * eb, dtype=torch.uint8, device="cuda")
            for opn in ("c2r", "r2c"):
                op = getattr(ipt, opn)
                op(x, m, n, elem_bytes=eb)
                torch.cuda.synchronize()
                ipt.profile_enable(True)
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
                ts.sort()
                med = ts[len(ts) // 2]
                kern = {k: round(v[2] / v[1] / 1e6, 1) for k, v in prof.items() if v[0] and v[1]}
                print(json.dumps({"m": m, "n": n, "eb": eb, "op": opn, "gcd": math.gcd(m, n),
                                  "GBps": round(2 * m * n * eb / med / 1e6, 1), "kernels": kern}), flush=True)
            del x
            torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
