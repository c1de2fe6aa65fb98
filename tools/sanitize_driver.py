"""Small calls of every kernel variant, for compute-sanitizer (memcheck / racecheck /
synccheck / initcheck).  Not a test: the parity tests check values; this only exercises
each kernel family on shapes small enough for the sanitizers, and checks round trips.

    compute-sanitizer --tool memcheck python tools/sanitize_driver.py
"""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))

import torch  # noqa: E402

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def env(**kv):
    for k, v in kv.items():
        if v is None:
            os.environ.pop(k, None)
        else:
            os.environ[k] = str(v)


def roundtrip(m, n, eb, tag):
    x = torch.randint(0, 2**31 - 1, (m * n * eb // 4,), dtype=torch.int32, device="cuda")
    y = x.clone()
    ipt.c2r(x, m, n, elem_bytes=eb)
    ipt.r2c(x, m, n, elem_bytes=eb)
    torch.cuda.synchronize()
    ok = torch.equal(x, y)
    print(f"{tag:40s} {m}x{n} eb{eb}: {'ok' if ok else 'MISMATCH'}", flush=True)
    if not ok:
        sys.exit(1)


def main():
    # row pass (pipelined, gcd 1; lagged layouts), column shuffle (both engines)
    for eng in ("c2r", "r2c"):
        env(IPT_FORCE_ENGINE=eng)
        roundtrip(301, 517, 4, f"gcd1 {eng}")
        roundtrip(517, 301, 8, f"gcd1 {eng}")
        roundtrip(97, 64, 16, f"gcd1 {eng}")
        # fused rotation: chunked pass (auto for small c) and the flag-based row_rot_kernel
        env(IPT_ROW_CHUNK=1)
        roundtrip(2 * 301, 2 * 517, 4, f"fused chunked {eng}")
        roundtrip(6 * 101, 6 * 77, 8, f"fused chunked {eng}")
        env(IPT_ROW_CHUNK=0)
        roundtrip(2 * 301, 2 * 517, 4, f"fused flags {eng}")
        roundtrip(6 * 101, 6 * 77, 8, f"fused flags {eng}")
        env(IPT_ROW_CHUNK=None)
        # c = 5..8: chunked pass chosen automatically; single-buffered rows (L2 prefetch)
        roundtrip(6 * 101, 6 * 77, 4, f"fused c=6 auto {eng}")
        env(IPT_ROW_DB_MAX=1024)
        roundtrip(6 * 101, 6 * 77, 4, f"fused c=6 single-buffered {eng}")
        env(IPT_ROW_DB_MAX=None)
        # legacy row kernel
        env(IPT_ROW_PIPE=0)
        roundtrip(301, 517, 4, f"row legacy {eng}")
        env(IPT_ROW_PIPE=None)
        # separate rotation pass (COL_ROT)
        env(IPT_FUSE_ROT=0)
        roundtrip(40 * 13, 40 * 17, 4, f"separate rotation {eng}")
        env(IPT_FUSE_ROT=None)
        # cluster row pass (rows forced onto clusters)
        env(IPT_ROW_CLUSTER_MIN=1, IPT_ROW_CLUSTER_K=4)
        roundtrip(203, 307, 8, f"cluster rows {eng}")
        env(IPT_ROW_CLUSTER_MIN=None, IPT_ROW_CLUSTER_K=None)
    env(IPT_FORCE_ENGINE=None)
    # batched
    x = torch.randint(0, 2**31 - 1, (3 * 120 * 77,), dtype=torch.int32, device="cuda")
    y = x.clone()
    ipt.c2r_batched(x, 3, 120 * 77, 120, 77, elem_bytes=4)
    ipt.r2c_batched(x, 3, 120 * 77, 120, 77, elem_bytes=4)
    torch.cuda.synchronize()
    print("batched:", "ok" if torch.equal(x, y) else "MISMATCH", flush=True)
    # host-buffer entry point on two streams
    hs = [torch.randint(0, 2**31 - 1, (301 * 517,), dtype=torch.int32).pin_memory() for _ in range(2)]
    ref = [h.clone() for h in hs]
    ds = [torch.empty(301 * 517, dtype=torch.int32, device="cuda") for _ in range(2)]
    sts = [torch.cuda.Stream(), torch.cuda.Stream()]
    for k in range(2):
        ipt.c2r_host(hs[k], ds[k], 301, 517, elem_bytes=4, stream=sts[k])
    torch.cuda.synchronize()
    for k in range(2):
        ipt.r2c_host(hs[k], ds[k], 301, 517, elem_bytes=4, stream=sts[k])
    torch.cuda.synchronize()
    print("host API:", "ok" if all(torch.equal(hs[k], ref[k]) for k in range(2)) else "MISMATCH", flush=True)
    # skinny engine (register and shared-memory row kernels, folded rotation)
    for n, eb in ((3, 4), (8, 4), (5, 8)):
        cnt = 65536 + 96
        x = torch.randint(0, 2**31 - 1, (cnt * n * eb // 4,), dtype=torch.int32, device="cuda")
        y = x.clone()
        ipt.aos_to_soa(x, cnt, n, field_bytes=eb)
        ipt.soa_to_aos(x, cnt, n, field_bytes=eb)
        torch.cuda.synchronize()
        print(f"skinny n={n} eb={eb}:", "ok" if torch.equal(x, y) else "MISMATCH", flush=True)
    # records and sub-word elements
    for (m, n, eb) in ((60, 70, 12), (33, 21, 48), (64, 50, 2), (64, 52, 1)):
        nb = m * n * eb
        x = torch.randint(0, 255, (nb,), dtype=torch.uint8, device="cuda")
        y = x.clone()
        ipt.c2r(x, m, n, elem_bytes=eb)
        ipt.r2c(x, m, n, elem_bytes=eb)
        torch.cuda.synchronize()
        print(f"records {m}x{n} eb{eb}:", "ok" if torch.equal(x, y) else "MISMATCH", flush=True)
    # AoS helpers: consumer kernels, warp load/store, random gather/scatter
    for S in (1, 3, 4, 7, 16):
        cnt = 32 * 40 + 5
        src = torch.randint(0, 2**31 - 1, (cnt * S,), dtype=torch.int32, device="cuda")
        for v in (ipt.AOS_DIRECT, ipt.AOS_VECTOR, ipt.AOS_COALESCED):
            dst = torch.zeros_like(src)
            ipt.aos_copy(src, dst, cnt, S, v)
            idx = torch.randperm(cnt, device="cuda").to(torch.int32)
            ipt.aos_gather(src, idx, dst, cnt, S, v)
            ipt.aos_scatter(src, idx, dst, cnt, S, v)
            ipt.aos_fill(dst, cnt, S, v)
        torch.cuda.synchronize()
        print(f"aos S={S}: ok", flush=True)


if __name__ == "__main__":
    main()
