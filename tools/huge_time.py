"""Time one c2r / r2c pair on a config-5a matrix with per-kernel kinds (development tool)."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402

m, n, eb = (int(v) for v in (sys.argv[1:4] if len(sys.argv) > 3 else (120011, 145820, 8)))
x = torch.empty(m * n * eb, dtype=torch.uint8, device="cuda")
ipt.c2r(x, m, n, elem_bytes=eb)
ipt.r2c(x, m, n, elem_bytes=eb)
torch.cuda.synchronize()
ipt.profile_enable(True)
ipt.profile_read()
for op in ("c2r", "r2c"):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    getattr(ipt, op)(x, m, n, elem_bytes=eb)
    e1.record()
    e1.synchronize()
    print(op, round(2 * m * n * eb / (e0.elapsed_time(e1) * 1e-3) / 1e9, 1), "GB/s", flush=True)
prof = ipt.profile_read()
print({k: round(v[2] / (v[1] * 1e-3) / 1e9, 1) for k, v in prof.items() if v[0]}, ipt.plan_info(m, n, eb)["row_cluster"],
      os.environ.get("IPT_ROW_CLUSTER_K"), os.environ.get("IPT_ROW_CLUSTER_MODE"), flush=True)
