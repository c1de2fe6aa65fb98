"""e2e throughput of ipt_c2r_host over the first sweep shapes with k streams / buffers in
flight (development tool): all Eq. 37 bytes / device time, first H2D to last D2H."""
import os
import statistics
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402
import workloads  # noqa: E402

shapes = [(m, n, eb) for eb in (4, 8) for (m, n) in workloads.sweep_shapes(8)]
big = max(m * n * eb for m, n, eb in shapes)
for k in (1, 2, 3, 4):
    hosts = [torch.empty(big, dtype=torch.uint8, pin_memory=True) for _ in range(k)]
    devs = [torch.empty(big, dtype=torch.uint8, device="cuda") for _ in range(k)]
    sts = [torch.cuda.Stream() for _ in range(k)]
    rates = []
    for rep in range(3):
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(sts[0])
        for s in sts[1:]:
            s.wait_event(e0)
        for i, (m, n, eb) in enumerate(shapes):
            ipt.c2r_host(hosts[i % k][:m * n * eb], devs[i % k], m, n, elem_bytes=eb, stream=sts[i % k].cuda_stream)
        for s in sts[1:]:
            ev = torch.cuda.Event()
            ev.record(s)
            sts[0].wait_event(ev)
        e1.record(sts[0])
        e1.synchronize()
        rates.append(sum(2.0 * m * n * eb for m, n, eb in shapes) / (e0.elapsed_time(e1) * 1e-3) / 1e9)
    # pure copy rates for reference
    print(f"streams={k}: e2e {statistics.median(rates[1:]):.1f} GB/s", flush=True)
    del hosts, devs
h = torch.empty(1 << 30, dtype=torch.uint8, pin_memory=True)
d = torch.empty(1 << 30, dtype=torch.uint8, device="cuda")
for name, fn in (("H2D", lambda: d.copy_(h, non_blocking=True)), ("D2H", lambda: h.copy_(d, non_blocking=True))):
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    fn()
    e1.record()
    e1.synchronize()
    print(f"{name} 1 GiB: {(1 << 30) / (e0.elapsed_time(e1) * 1e-3) / 1e9:.1f} GB/s", flush=True)
