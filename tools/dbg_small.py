import torch, numpy as np, time, sys
sys.path.insert(0,'.')
import paper_conf_ppopp_catanzarokg14_b200 as ipt, oracle
for (m,n) in [(37,53),(300,451),(1200,1800),(17226,6052)]:
    print(m,n, ipt.plan_info(m,n,4), flush=True)
    h = np.random.default_rng(0).integers(0,2**32,m*n,dtype=np.uint32)
    x = torch.from_numpy(h.view(np.uint8).copy()).cuda()
    ipt.c2r(x,m,n,elem_bytes=4); torch.cuda.synchronize()
    ok = x.cpu().numpy().tobytes()==oracle.transpose(h,m,n).tobytes()
    t0=time.perf_counter(); 
    for _ in range(3): ipt.c2r(x,m,n,elem_bytes=4)
    torch.cuda.synchronize(); print("ok",ok, (time.perf_counter()-t0)/3*1e3,"ms", flush=True)
