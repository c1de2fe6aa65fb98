"""Pass-by-pass sampled check of ipt_c2r on index data (development tool).

    python tools/dbg_huge.py --shape 120011x145820 --eb 8

The buffer carries its own element index.  After each pass (IPT_DEBUG_PASSES=k) sampled
outputs are compared with the source index the oracle's per-pass gather forms give
(R2C: Eqs. 34-35 then Eq. 24; C2R: Eq. 23, Eq. 31, Eq. 26).
"""
import argparse
import os
import random
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import numpy as np  # noqa: E402
import torch  # noqa: E402

import oracle  # noqa: E402
import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--shape", action="append", required=True)
    p.add_argument("--eb", type=int, default=8)
    p.add_argument("--samples", type=int, default=4000)
    a = p.parse_args()
    for sh in a.shape:
        m, n = (int(v) for v in sh.split("x"))
        info = ipt.plan_info(m, n, a.eb)
        M, N, eng = info["M"], info["N"], info["engine"]
        print(sh, info, flush=True)
        rng = random.Random(1)
        pos = [(rng.randrange(M), rng.randrange(N)) for _ in range(a.samples)]
        if eng == "r2c":   # pass 1: gather q^{-1}((i-j) mod M) (Eq. 34 o Eq. 35); pass 2: d'_i (Eq. 24)
            p1 = lambda i, j: (oracle.eq34_qinv(M, N, (i - j) % M), j)
            p2 = lambda i, j: (i, oracle.eq24_dp(M, N, i, j))
            passes = [p1, p2]
            if info["c"] > 1:
                passes.append(lambda i, j: (oracle.eq36_rinv(M, N, i, j), j))
        else:
            passes = []
            if info["c"] > 1:
                passes.append(lambda i, j: (oracle.eq23_r(M, N, i, j), j))
            passes.append(lambda i, j: (i, oracle.eq31_dpinv(M, N, i, j)))
            passes.append(lambda i, j: (oracle.eq26_sp(M, N, i, j), j))
        # after k passes, element (i, j) came from f1(f2(...fk(i, j)))
        for k in range(1, len(passes) + 1):
            x = torch.empty(M * N, dtype=torch.int32 if a.eb == 4 else torch.int64, device="cuda")
            for s in range(0, M * N, 1 << 28):  # one arange over > 2^32 elements leaves the tail zero
                e = min(M * N, s + (1 << 28))
                x[s:e] = torch.arange(s, e, dtype=torch.int64, device="cuda").to(x.dtype)
            os.environ["IPT_DEBUG_PASSES"] = str(k)
            ipt.c2r(x, m, n, elem_bytes=a.eb)
            torch.cuda.synchronize()
            bad = 0
            idx, exp = [], []
            for (i, j) in pos:
                ii, jj = i, j
                for f in reversed(passes[:k]):
                    ii, jj = f(ii, jj)
                idx.append(i * N + j)
                exp.append(ii * N + jj)
            got = x[torch.tensor(idx, device="cuda")].cpu().numpy().astype(np.int64)
            e = np.array(exp, dtype=np.int64)
            if a.eb == 4:
                e = e.astype(np.int32).astype(np.int64)
            bad = np.nonzero(got != e)[0]
            print(f"  after pass {k}: {len(bad)} / {len(pos)} wrong", flush=True)
            for b in bad[:5]:
                i, j = divmod(idx[b], N)
                g = int(got[b])
                print(f"    (i={i}, j={j}) got src ({g // N}, {g % N}) want ({exp[b] // N}, {exp[b] % N})")
            del x
            torch.cuda.empty_cache()
        os.environ.pop("IPT_DEBUG_PASSES", None)


if __name__ == "__main__":
    main()
