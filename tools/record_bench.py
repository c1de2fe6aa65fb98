"""Throughput of multi-word records and 1/2-byte elements against single-word calls of the same bytes.

For each (m, n, record bytes) it times ipt_c2r on the record matrix and, for comparison, the
single-word call that moves the same buffer as one 16-byte-word (or 4-byte) transpose
P_{m, n*k}.  Effective GB/s = 2*m*n*s / t (Eq. 37).  Inputs larger than L2
(126 MB) except the config-1 shape, which is preceded by an L2 flush.  CUDA events on the
current stream, median of --reps.

    python tools/record_bench.py --reps 10 > gpurun_out/records.jsonl
"""
import argparse
import json
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402

SHAPES = [(1200, 1800, 12), (1200, 1800, 32), (14414, 6565, 12), (14414, 6565, 24), (14414, 6565, 32),
          (6565, 14414, 64), (4096, 3000, 48), (17226, 6052, 20),
          (14414, 6565, 2), (6565, 14414, 2), (14412, 6565, 1), (14414, 6566, 2), (14412, 6564, 1),
          (1200, 1800, 2), (1200, 1800, 1), (1 << 24, 5, 12), (1 << 25, 3, 2), (1 << 24, 4, 1)]


def time_op(fn, reps, flush):
    ts = []
    for _ in range(reps):
        flush.zero_()
        a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        a.record()
        fn()
        b.record()
        torch.cuda.synchronize()
        ts.append(a.elapsed_time(b) / 1e3)
    return statistics.median(ts)


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--reps", type=int, default=10)
    a = p.parse_args()
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for m, n, eb in SHAPES:
        x = torch.randint(0, 255, (m * n * eb,), dtype=torch.uint8, device="cuda")
        w = 16 if eb % 16 == 0 else 8 if eb % 8 == 0 else 4
        k = eb // w
        # the single-word call over the same bytes: P_{m, n*k}; sub-word: packed 4-byte words
        wm, wn = (m, n * k) if eb >= 4 else ((m, n * eb // 4) if n * eb % 4 == 0 else (m * eb // 4, n))
        ipt.c2r(x, m, n, elem_bytes=eb)  # warm-up (plans, pools)
        ipt.c2r(x, wm, wn, elem_bytes=w)
        t_rec = time_op(lambda: ipt.c2r(x, m, n, elem_bytes=eb), a.reps, flush)
        t_word = time_op(lambda: ipt.c2r(x, wm, wn, elem_bytes=w), a.reps, flush)
        by = 2 * m * n * eb
        print(json.dumps({"m": m, "n": n, "record_bytes": eb, "word_bytes": w, "k": k,
                          "record_gbs": round(by / t_rec / 1e9, 1), "record_ms": round(t_rec * 1e3, 3),
                          "one_word_step_gbs": round(by / t_word / 1e9, 1),
                          "plan": ipt.plan_info(m, n, eb)}), flush=True)
        del x
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
