"""Engine landscapes (SURVEY row f2; Figs. 4-5, :871-959) and the B200 check of the
paper's engine heuristic (:959, "if m > n, use the C2R algorithm, otherwise use the R2C").

    python tools/landscape.py --shapes 2000 --eb 4 8 --out profiles/r02_landscape

For `--shapes` random (m, n) uniform in [1000, 25000] (seed 959) and each element size, the
row-major transpose P_{m,n} is timed with each engine forced (IPT_FORCE_ENGINE=c2r: C2R(M=m,
N=n), rows of n on chip; =r2c: R2C(M=n, N=m), rows of m on chip), CUDA events around the
whole call, L2 flushed before every call, median of --reps.  Writes one JSON line per shape
to <out>_eb<s>.jsonl and prints a summary: Eq. 37 medians of each fixed rule, of the
paper's rule and of the per-shape best, win rates per class (gcd 1 / 2..32 / > 32, and
whether the shorter row fits two shared-memory buffers), and a binned landscape table.
"""
import argparse
import json
import math
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def timed(op, x, m, n, eb, flush, reps):
    op(x, m, n, elem_bytes=eb)  # plan + warm-up
    ts = []
    for _ in range(reps):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        op(x, m, n, elem_bytes=eb)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    return 2.0 * m * n * eb / (statistics.median(ts) * 1e-3) / 1e9


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--shapes", type=int, default=2000)
    p.add_argument("--eb", type=int, nargs="+", default=[4, 8])
    p.add_argument("--reps", type=int, default=3)
    p.add_argument("--lo", type=int, default=1000)
    p.add_argument("--hi", type=int, default=25000)
    p.add_argument("--out", default="gpurun_out/landscape")
    a = p.parse_args()
    rng = np.random.default_rng(959)
    shapes = [(int(u), int(v)) for u, v in rng.integers(a.lo, a.hi + 1, size=(a.shapes, 2))]
    flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
    for eb in a.eb:
        x = torch.empty(a.hi * a.hi * eb, dtype=torch.uint8, device="cuda")
        rows = []
        with open(f"{a.out}_eb{eb}.jsonl", "w") as f:
            for (m, n) in shapes:
                rec = {"m": m, "n": n, "eb": eb, "gcd": math.gcd(m, n)}
                for eng in ("c2r", "r2c"):
                    os.environ["IPT_FORCE_ENGINE"] = eng
                    rec[eng] = round(timed(ipt.c2r, x, m, n, eb, flush, a.reps), 1)
                os.environ.pop("IPT_FORCE_ENGINE", None)
                rec["paper"] = rec["c2r"] if m > n else rec["r2c"]
                f.write(json.dumps(rec) + "\n")
                rows.append(rec)
        del x
        torch.cuda.empty_cache()
        summarize(rows, eb)


def summarize(rows, eb):
    def med(key, sel=lambda r: True):
        v = [r[key] if isinstance(key, str) else key(r) for r in rows if sel(r)]
        return round(statistics.median(v), 1) if v else None

    best = lambda r: max(r["c2r"], r["r2c"])
    flipped = lambda r: r["r2c"] if r["m"] > r["n"] else r["c2r"]
    print(f"eb={eb} n={len(rows)} medians: paper {med('paper')} flipped {med(flipped)} always-c2r {med('c2r')} "
          f"always-r2c {med('r2c')} per-shape-best {med(best)}", flush=True)
    classes = {
        "gcd1": lambda r: r["gcd"] == 1,
        "gcd2-32": lambda r: 1 < r["gcd"] <= 32,
        "gcd>32": lambda r: r["gcd"] > 32,
        "minrow<=56KB": lambda r: min(r["m"], r["n"]) * eb <= 56 * 1024,
        "minrow>56KB": lambda r: min(r["m"], r["n"]) * eb > 56 * 1024,
    }
    for name, sel in classes.items():
        sub = [r for r in rows if sel(r)]
        if not sub:
            continue
        paper_wins = sum(1 for r in sub if r["paper"] >= max(r["c2r"], r["r2c"]) * 0.999)
        print(f"  {name:13s} n={len(sub):5d} paper-rule picks the faster engine {100 * paper_wins / len(sub):5.1f}% | "
              f"medians paper {med('paper', sel)} flipped {med(flipped, sel)} best {med(best, sel)}", flush=True)
    # binned landscape (Fig. 4/5 analogue): median GB/s per (m, n) bin for each engine
    edges = list(range(1000, 26001, 4000))
    for eng in ("c2r", "r2c"):
        print(f"  landscape {eng} (rows: m bins, cols: n bins {edges[:-1]})")
        for i in range(len(edges) - 1):
            line = []
            for j in range(len(edges) - 1):
                v = [r[eng] for r in rows if edges[i] <= r["m"] < edges[i + 1] and edges[j] <= r["n"] < edges[j + 1]]
                line.append(f"{statistics.median(v):6.0f}" if v else "     -")
            print(f"    m {edges[i]:5d}-{edges[i + 1]:5d} " + " ".join(line))


if __name__ == "__main__":
    main()
