"""One identity column-tile pass (for ncu).  python tools/one_tilecopy.py M N eb twb groupsize barrier"""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ppopp_catanzarokg14_b200 as ipt
M, N, eb, twb, G, bar = (int(v) for v in sys.argv[1:7])
x = torch.zeros(M * N * eb, dtype=torch.uint8, device="cuda")
for _ in range(2):
    ipt.debug_tile_copy(x, M, N, eb, twb, G, bar)
torch.cuda.synchronize()
