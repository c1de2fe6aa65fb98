"""Run ipt_c2r / ipt_r2c on one shape a few times (for ncu captures; not a benchmark).

    python tools/one_shape.py --m 17226 --n 6052 --eb 4 --reps 3 [--op c2r]
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def main():
    p = argparse.ArgumentParser()
    p.add_argument("--m", type=int, default=17226)
    p.add_argument("--n", type=int, default=6052)
    p.add_argument("--eb", type=int, default=4)
    p.add_argument("--reps", type=int, default=3)
    p.add_argument("--op", default="c2r")
    a = p.parse_args()
    x = torch.randint(0, 255, (a.m * a.n * a.eb,), dtype=torch.uint8, device="cuda")
    op = getattr(ipt, a.op)
    for _ in range(a.reps):
        op(x, a.m, a.n, elem_bytes=a.eb)
    torch.cuda.synchronize()
    print(ipt.plan_info(a.m, a.n, a.eb))


if __name__ == "__main__":
    main()
