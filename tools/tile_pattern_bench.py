"""Microbenchmark of the column-tile access pattern (identity mode of the column kernel).

Times ipt_debug_tile_copy over tile widths, cluster sizes and with/without the cluster
barrier, next to torch's contiguous copy_, on the engine view of a sweep shape.  Prints
one JSON line per configuration: GB/s = (bytes read + written) / device time.
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def timed(fn, flush, reps=5):
    ts = []
    for _ in range(reps + 1):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        fn()
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return statistics.median(ts[1:])


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--M", type=int, default=17226)
    p.add_argument("--N", type=int, default=6052)
    p.add_argument("--eb", type=int, default=4)
    a = p.parse_args()
    nb = a.M * a.N * a.eb
    x = torch.randint(0, 255, (nb,), dtype=torch.uint8, device="cuda")
    y = torch.empty_like(x)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    t = timed(lambda: y.copy_(x), flush)
    print(json.dumps({"what": "torch copy_", "GBps": round(2 * nb / t / 1e6, 1)}), flush=True)
    for twb in (64, 128):
        for K in (16, 32, 48, 64, 96, 128):
            for bar in (0, 1):
                try:
                    t = timed(lambda: ipt.debug_tile_copy(x, a.M, a.N, a.eb, twb, K, bar), flush)
                except ipt.IptError as e:
                    print(json.dumps({"twb": twb, "K": K, "barrier": bar, "err": str(e)}), flush=True)
                    break
                print(json.dumps({"twb": twb, "K": K, "barrier": bar, "GBps": round(2 * nb / t / 1e6, 1)}),
                      flush=True)


if __name__ == "__main__":
    main()
