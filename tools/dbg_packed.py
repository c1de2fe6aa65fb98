"""Debug: the degenerate-shape packed run, one call at a time (CUDA_LAUNCH_BLOCKING=1)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ppopp_catanzarokg14_b200 as ipt
import workloads
shapes = [(1, 1), (1, 500), (500, 1), (2, 2), (97, 97), (256, 256), (1000, 10), (10, 1000),
          (4096, 64), (64, 4096), (2, 3000), (3000, 2), (6, 4), (4, 6), (1024, 1023), (1023, 1024)]
for eb in (4, 8, 16):
    offs, tot = [], 0
    for m, n in shapes:
        offs.append(tot)
        tot += m * n + 3
    host = workloads.random_words(tot, eb, 100 + eb)
    buf = torch.from_numpy(np.ascontiguousarray(host).view(np.uint8).reshape(-1).copy()).cuda()
    for (m, n), o in zip(shapes, offs):
        print(eb, m, n, "base mod 16 =", (buf.data_ptr() + o * eb) % 16, ipt.plan_info(m, n, eb), flush=True)
        ipt.c2r(buf.data_ptr() + o * eb, m, n, elem_bytes=eb)
        torch.cuda.synchronize()
print("all ok")
