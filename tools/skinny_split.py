"""Per-kernel-kind breakdown of the skinny engine per direction (development tool).

    python tools/skinny_split.py [--count 67108864] [--n 8 9 24 25]
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--count", type=int, default=1 << 26)
    p.add_argument("--n", type=int, nargs="+", default=[2, 3, 8, 9, 16, 24, 25, 32])
    p.add_argument("--reps", type=int, default=3)
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    x = torch.empty(a.count * max(a.n) * 4, dtype=torch.uint8, device="cuda")
    for n in a.n:
        nb = a.count * n * 4
        for op in ("aos_to_soa", "soa_to_aos"):
            f = getattr(ipt, op)
            f(x[:nb], a.count, n, field_bytes=4)
            ts = []
            ipt.profile_enable(True)
            ipt.profile_read()
            for _ in range(a.reps):
                flush.zero_()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                f(x[:nb], a.count, n, field_bytes=4)
                e1.record()
                e1.synchronize()
                ts.append(e0.elapsed_time(e1))
            prof = ipt.profile_read()
            ipt.profile_enable(False)
            kern = {k: "%d x %.1f GB/s (%.2f ms)" % (v[0] // a.reps, v[2] / (v[1] * 1e-3) / 1e9, v[1] / a.reps)
                    for k, v in prof.items() if v[0]}
            ms = statistics.median(ts)
            print(f"n={n:2d} {op:10s} {2 * nb / ms / 1e6:7.1f} GB/s  {ms:6.2f} ms  plan={ipt.plan_info(a.count, n, 4)['c']} {kern}",
                  flush=True)


if __name__ == "__main__":
    main()
