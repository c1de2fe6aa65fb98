"""SURVEY §8 row f1 / PAPER.md Fig. 9: random-access AoS gather (dst[k] = src[idx[k]]) and
scatter (dst[idx[k]] = src[k], idx a permutation) bandwidth of the consumer-kernel variants
(Direct, Vector, Coalesced = warp_gather_aos / warp_scatter_aos) over `count` structs of
S = 1..16 four-byte words.  GB/s = struct bytes read + written / device time (events, L2
flushed before every timed call; the index reads are not counted).  One JSON line per
(S, op, variant), then a summary line.

    python tools/aos_random_bench.py [--count 16777216] [--reps 3]
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
    p.add_argument("--count", type=int, default=1 << 24)
    p.add_argument("--reps", type=int, default=3)
    p.add_argument("--max-words", type=int, default=16)
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    g = torch.Generator(device="cuda")
    g.manual_seed(9)
    perm = torch.randperm(a.count, device="cuda", generator=g).to(torch.int32)
    rows = []
    for S in range(1, a.max_words + 1):
        src = torch.randint(0, 2**31 - 1, (a.count * S,), dtype=torch.int32, device="cuda")
        dst = torch.empty_like(src)
        for op in ("gather", "scatter"):
            for v in (ipt.AOS_DIRECT, ipt.AOS_VECTOR, ipt.AOS_COALESCED):
                ts = []
                for r in range(a.reps + 1):
                    flush.zero_()
                    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                    e0.record()
                    if op == "gather":
                        ipt.aos_gather(src, perm, dst, a.count, S, v)
                    else:
                        ipt.aos_scatter(src, perm, dst, a.count, S, v)
                    e1.record()
                    e1.synchronize()
                    if r:
                        ts.append(e0.elapsed_time(e1))
                gbps = a.count * S * 4 * 2 / (statistics.median(ts) * 1e-3) / 1e9
                row = {"S": S, "struct_bytes": 4 * S, "op": op, "variant": NAMES[v], "GBps": round(gbps, 1)}
                rows.append(row)
                print(json.dumps(row), flush=True)
        del src, dst
    summ = {}
    for op in ("gather", "scatter"):
        for v in NAMES.values():
            gs = [r["GBps"] for r in rows if r["op"] == op and r["variant"] == v]
            summ[f"{op}_{v}_median"] = round(statistics.median(gs), 1)
    print(json.dumps({"summary": summ, "count": a.count}), flush=True)


if __name__ == "__main__":
    main()
