"""BASELINE config 4 / PAPER.md Fig. 8: unit-stride AoS store and copy bandwidth of the
three consumer-kernel variants (Direct, Vector, Coalesced = coalesced_ptr<T>) over 2**26
structs of S = 1..16 four-byte words.  GB/s = bytes read + written / device time (events,
L2 flushed before every timed call).  Prints one JSON line per (S, op, variant) and a
summary line.

    python tools/aos_bench.py [--count 67108864] [--reps 5]
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402

NAMES = {ipt.AOS_DIRECT: "direct", ipt.AOS_VECTOR: "vector", ipt.AOS_COALESCED: "coalesced"}


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--count", type=int, default=1 << 26)
    p.add_argument("--reps", type=int, default=5)
    p.add_argument("--max-words", type=int, default=16)
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    rows = []
    for S in range(1, a.max_words + 1):
        src = torch.randint(0, 2**31 - 1, (a.count * S,), dtype=torch.int32, device="cuda")
        dst = torch.empty_like(src)
        for op in ("copy", "store"):
            for v in (ipt.AOS_DIRECT, ipt.AOS_VECTOR, ipt.AOS_COALESCED):
                ts = []
                for r in range(a.reps + 1):
                    flush.zero_()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    if op == "copy":
                        ipt.aos_copy(src, dst, a.count, S, v)
                    else:
                        ipt.aos_fill(dst, a.count, S, v)
                    e1.record()
                    e1.synchronize()
                    if r:
                        ts.append(e0.elapsed_time(e1))
                by = a.count * S * 4 * (2 if op == "copy" else 1)
                g = by / (statistics.median(ts) * 1e-3) / 1e9
                row = {"S": S, "struct_bytes": 4 * S, "op": op, "variant": NAMES[v], "GBps": round(g, 1)}
                rows.append(row)
                print(json.dumps(row), flush=True)
        del src, dst
    summ = {}
    for op in ("copy", "store"):
        for v in NAMES.values():
            gs = [r["GBps"] for r in rows if r["op"] == op and r["variant"] == v]
            summ[f"{op}_{v}_median"] = round(statistics.median(gs), 1)
            summ[f"{op}_{v}_min"] = round(min(gs), 1)
    speed = [next(r["GBps"] for r in rows if r["op"] == o and r["S"] == s and r["variant"] == "coalesced") /
             next(r["GBps"] for r in rows if r["op"] == o and r["S"] == s and r["variant"] == "direct")
             for o in ("copy", "store") for s in range(1, a.max_words + 1)]
    summ["max_speedup_coalesced_vs_direct"] = round(max(speed), 2)
    print(json.dumps({"summary": summ, "count": a.count}), flush=True)


if __name__ == "__main__":
    main()
