"""Time the column kernel's identity pass (ipt_debug_tile_copy) -- the access pattern alone.

    python tools/tilecopy_time.py M N eb [twb]    (prints GB/s for barrier 0/1, G from the band)
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402

M, N, eb = (int(v) for v in sys.argv[1:4])
twb = int(sys.argv[4]) if len(sys.argv) > 4 else 128
x = torch.zeros(M * N * eb, dtype=torch.uint8, device="cuda")
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
B = 46 * 1024 // (twb + 8)
G = (M + B - 1) // B
for bar in (0, 1):
    ts = []
    for k in range(6):
        flush.zero_()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        ipt.debug_tile_copy(x, M, N, eb, twb, G, bar)
        e1.record()
        torch.cuda.synchronize()
        if k:
            ts.append(e0.elapsed_time(e1))
    ts.sort()
    print(f"tilecopy M={M} N={N} eb={eb} twb={twb} G={G} barrier={bar} pipe={os.environ.get('IPT_COL_PIPE', '1')}: "
          f"{2 * M * N * eb / ts[len(ts) // 2] / 1e6:.1f} GB/s")
