import sys, torch
sys.path.insert(0, '.')
import paper_conf_ppopp_catanzarokg14_b200 as ipt
n = int(sys.argv[1]); op = sys.argv[2]; cnt = 1 << 26
x = torch.empty(cnt * n * 4, dtype=torch.uint8, device='cuda')
for _ in range(2):
    getattr(ipt, op)(x, cnt, n, field_bytes=4)
torch.cuda.synchronize()
