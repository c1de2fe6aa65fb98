"""Per-pass device times of ipt_c2r on one shape (development tool, not the benchmark).

    python tools/time_passes.py --shape 17226x6052 --shape 30011x40009 --eb 8 --reps 5

Prints, per shape, the plan and each kernel kind's GB/s (algorithmic bytes / device time
from ipt_profile_read), plus the whole call's Eq. 37 GB/s (CUDA events, L2 flushed).
"""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--shape", action="append", required=True)
    p.add_argument("--eb", type=int, default=4)
    p.add_argument("--reps", type=int, default=5)
    p.add_argument("--op", default="c2r")
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for sh in a.shape:
        m, n = (int(v) for v in sh.split("x"))
        x = torch.empty(m * n * a.eb, dtype=torch.uint8, device="cuda")
        op = getattr(ipt, a.op)
        op(x, m, n, elem_bytes=a.eb)
        torch.cuda.synchronize()
        ipt.profile_enable(True)
        ipt.profile_read()
        ts = []
        for _ in range(a.reps):
            flush.zero_()
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            e0.record()
            op(x, m, n, elem_bytes=a.eb)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        prof = ipt.profile_read()
        ipt.profile_enable(False)
        ts.sort()
        med = ts[len(ts) // 2]
        out = {"shape": sh, "eb": a.eb, "plan": ipt.plan_info(m, n, a.eb),
               "eq37_GBps": round(2 * m * n * a.eb / med / 1e6, 1), "ms": round(med, 3),
               "kernels": {k: {"launches": v[0], "ms": round(v[1], 3),
                               "GBps": round(v[2] / v[1] / 1e6, 1) if v[1] else None}
                           for k, v in prof.items() if v[0]}}
        print(json.dumps(out), flush=True)
        del x
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
