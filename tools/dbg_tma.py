import os, sys
sys.path.insert(0, '/root/repo')
import torch, numpy as np
import paper_conf_ppopp_catanzarokg14_b200 as ipt
import oracle
for (m, n) in [(8, 8), (12, 20), (33, 64), (64, 64), (1200, 1800), (2000, 3000), (3000, 2000), (4096, 3000)]:
    for eb in (4, 8, 16):
        x = torch.randint(0, 2**31 - 1, (m * n * eb // 4,), dtype=torch.int32, device="cuda")
        h = x.cpu().numpy().copy()
        try:
            ipt.c2r(x, m, n, elem_bytes=eb)
            torch.cuda.synchronize()
            want = oracle.transpose(h.view(np.dtype((np.void, eb))), m, n)
            ok = x.cpu().numpy().tobytes() == want.tobytes()
            print(m, n, eb, "ok" if ok else "MISMATCH", ipt.plan_info(m, n, eb), flush=True)
        except Exception as e:
            print(m, n, eb, "ERR", e, flush=True)
            try:
                torch.cuda.synchronize()
            except Exception as e2:
                print("sync:", e2)
            sys.exit(1)
# degenerate / tiny shapes (TMA maps smaller than a box must fall back)
for (m, n) in [(1000, 10), (10, 1000), (2, 3000), (3000, 2), (4096, 64), (64, 4096), (1023, 1024), (1000, 12), (12, 1000)]:
    for eb in (4, 8, 16):
        x = torch.randint(0, 2**31 - 1, (m * n * eb // 4,), dtype=torch.int32, device="cuda")
        h = x.cpu().numpy().copy()
        ipt.c2r(x, m, n, elem_bytes=eb)
        torch.cuda.synchronize()
        want = oracle.transpose(h.view(np.dtype((np.void, eb))), m, n)
        print(m, n, eb, "ok" if x.cpu().numpy().tobytes() == want.tobytes() else "MISMATCH", flush=True)
