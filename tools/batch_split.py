"""Per-kernel breakdown of a batched call (config 5b shape by default; development tool).

    python tools/batch_split.py [--m 4096 --n 3000 --batch 512]
"""
import argparse
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402

p = argparse.ArgumentParser()
p.add_argument("--m", type=int, default=4096)
p.add_argument("--n", type=int, default=3000)
p.add_argument("--batch", type=int, default=512)
a = p.parse_args()
x = torch.empty(a.batch * a.m * a.n * 4, dtype=torch.uint8, device="cuda")
S = a.batch * a.m * a.n * 4
for op in ("c2r_batched", "r2c_batched"):
    f = getattr(ipt, op)
    f(x, a.batch, a.m * a.n, a.m, a.n, elem_bytes=4)
    ts = []
    ipt.profile_enable(True)
    ipt.profile_read()
    for _ in range(3):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        f(x, a.batch, a.m * a.n, a.m, a.n, elem_bytes=4)
        e1.record()
        e1.synchronize()
        ts.append(e0.elapsed_time(e1))
    prof = ipt.profile_read()
    ipt.profile_enable(False)
    kern = {k: "%.0f GB/s" % (v[2] / (v[1] * 1e-3) / 1e9) for k, v in prof.items() if v[0]}
    print(f"{op}: {2 * S / statistics.median(ts) / 1e6:.0f} GB/s {kern} env={os.environ.get('IPT_ROW_CHUNK_K', '')}", flush=True)
