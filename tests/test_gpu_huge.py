"""GPU parity of the huge-shape realisation: rows longer than one CTA's
shared memory go through the cluster row pass (K CTAs per row, distributed shared memory).

* Small and medium shapes with the cluster pass forced (IPT_ROW_CLUSTER_MIN=1,
  IPT_ROW_CLUSTER_K = 2, 4, 8, 16) are compared with the oracle in full, both engines,
  4/8/16-byte elements, gcd 1 and gcd > 1 (the f2 tail rows of Eq. 24 / Eq. 31).
* Shapes whose rows really exceed 227 KB, up to BASELINE config 5a (120011 x 145820 fp64,
  140 GB, 64-bit offsets), carry their own index as data (the "index_words" recipe of
  DESIGN.md) and are checked on sampled outputs one by one with the oracle's Eqs. 7-8,
  then round-tripped and compared in full on the device.
"""
import os
import random

import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402

DEV = torch.device("cuda:0")


class env:
    def __init__(self, **kv):
        self.kv = {k: str(v) for k, v in kv.items() if v is not None}

    def __enter__(self):
        self.old = {k: os.environ.get(k) for k in self.kv}
        os.environ.update(self.kv)

    def __exit__(self, *a):
        for k, v in self.old.items():
            if v is None:
                os.environ.pop(k, None)
            else:
                os.environ[k] = v


def vwords(host, eb):
    return np.ascontiguousarray(host).view(np.dtype((np.void, eb))).reshape(-1)


def to_dev(host):
    return torch.from_numpy(np.ascontiguousarray(host).view(np.uint8).reshape(-1).copy()).to(DEV)


SMALL = [(2, 3), (3, 2), (5, 7), (33, 31), (31, 33), (64, 48), (48, 64), (97, 130), (130, 97),
         (40, 512), (512, 40), (600, 400), (400, 600), (1000, 1), (129, 1025)]


@pytest.mark.parametrize("K", [2, 4, 8, 16])
@pytest.mark.parametrize("engine", ["c2r", "r2c"])
def test_cluster_rows_forced_small(K, engine):
    for eb in (4, 8, 16):
        for m, n in SMALL:
            host = workloads.random_words(m * n, eb, seed=m * 7 + n + K)
            hv = vwords(host, eb)
            with env(IPT_ROW_CLUSTER_MIN=1, IPT_ROW_CLUSTER_K=K, IPT_FORCE_ENGINE=engine):
                info = ipt.plan_info(m, n, eb)
                if min(m, n) > 1:
                    assert info["row_cluster"] == K, info
                x = to_dev(host)
                ipt.c2r(x, m, n, elem_bytes=eb)
                got = vwords(x.cpu().numpy(), eb)
                assert got.tobytes() == oracle.transpose(hv, m, n).tobytes(), (m, n, eb, K, engine)
                ipt.r2c(x, m, n, elem_bytes=eb)
                assert x.cpu().numpy().tobytes() == np.ascontiguousarray(host).tobytes(), (m, n, eb, K)


@pytest.mark.parametrize("K", [2, 4, 8, 16])
@pytest.mark.parametrize("engine", ["c2r", "r2c"])
def test_cluster_rows_forced_medium(K, engine):
    """Config 1 (gcd 600) and ragged gcd-1 shapes with several warps per segment."""
    for (m, n), eb in [((1200, 1800), 4), ((4099, 3001), 4), ((3001, 4099), 8), ((2048, 6144), 8),
                       ((1500, 2000), 16)]:
        host = workloads.random_words(m * n, eb, seed=K + m)
        hv = vwords(host, eb)
        with env(IPT_ROW_CLUSTER_MIN=1, IPT_ROW_CLUSTER_K=K, IPT_FORCE_ENGINE=engine):
            assert ipt.plan_info(m, n, eb)["row_cluster"] == K
            x = to_dev(host)
            ipt.c2r(x, m, n, elem_bytes=eb)
            assert vwords(x.cpu().numpy(), eb).tobytes() == oracle.transpose(hv, m, n).tobytes(), (m, n, K)
            ipt.r2c(x, m, n, elem_bytes=eb)
            assert x.cpu().numpy().tobytes() == np.ascontiguousarray(host).tobytes()


@pytest.mark.parametrize("mode,sync", [(0, 0), (0, 1), (0, 2), (1, 1)])
def test_cluster_variants(mode, sync):
    """IPT_ROW_CLUSTER_MODE (0: DSMEM gather, 1: L2 gather) and IPT_ROW_CLUSTER_SYNC
    (release/acquire barriers or CTA-scope fences), every K, both engines."""
    for (m, n), eb in [((3001, 4099), 4), ((1200, 1800), 8), ((517, 300), 16)]:
        host = workloads.random_words(m * n, eb, seed=sync + 3 * mode)
        for K in (2, 4, 8, 16):
            for engine in ("c2r", "r2c"):
                with env(IPT_ROW_CLUSTER_MIN=1, IPT_ROW_CLUSTER_SYNC=sync, IPT_ROW_CLUSTER_MODE=mode,
                         IPT_ROW_CLUSTER_K=K, IPT_FORCE_ENGINE=engine):
                    x = to_dev(host)
                    for _ in range(2):
                        ipt.c2r(x, m, n, elem_bytes=eb)
                        ipt.r2c(x, m, n, elem_bytes=eb)
                    ipt.c2r(x, m, n, elem_bytes=eb)
                    got = vwords(x.cpu().numpy(), eb)
                    assert got.tobytes() == oracle.transpose(vwords(host, eb), m, n).tobytes(), (m, n, K, engine)


def index_tensor(total, eb, chunk=1 << 28):
    """Element k carries k (8-byte words; 16-byte words carry (k, ~k)); 4-byte words k mod 2^32.
    Filled in chunks: one torch.arange over more than 2^32 elements leaves the tail zero."""
    x = torch.empty(total * (2 if eb == 16 else 1), dtype=torch.int32 if eb == 4 else torch.int64, device=DEV)
    for s in range(0, total, chunk):
        e = min(total, s + chunk)
        k = torch.arange(s, e, dtype=torch.int64, device=DEV)
        if eb == 16:
            x.view(-1, 2)[s:e] = torch.stack([k, ~k], dim=1)
        else:
            x[s:e] = k.to(x.dtype)
    return x


def check_index_transpose(x, m, n, eb, samples, seed):
    """x holds ipt_c2r(m, n) of index_tensor: output l must carry input s*n + c (Eqs. 7-8)."""
    rng = random.Random(seed)
    ls = [rng.randrange(m * n) for _ in range(samples)]
    want = []
    for l in ls:
        i, j = divmod(l, n)
        si, sj = oracle.c2r_source(m, n, i, j)
        want.append(si * n + sj)
    idx = torch.tensor(ls, dtype=torch.int64, device=DEV)
    if eb == 16:
        got = x.view(-1, 2)[idx].cpu().numpy()
        assert np.array_equal(got[:, 0], np.array(want, dtype=np.int64))
        assert np.array_equal(got[:, 1], ~np.array(want, dtype=np.int64))
    else:
        got = x[idx].cpu().numpy().astype(np.int64)
        w = np.array(want, dtype=np.int64)
        if eb == 4:
            w = w.astype(np.int32).astype(np.int64)
        assert np.array_equal(got, w), (m, n, eb)


def check_identity_chunked(x, total, eb, chunk=1 << 28):
    per = 2 if eb == 16 else 1
    flat = x.view(-1)
    for s in range(0, total, chunk):
        e = min(total, s + chunk)
        k = torch.arange(s, e, dtype=torch.int64, device=DEV)
        if eb == 16:
            want = torch.stack([k, ~k], dim=1).reshape(-1)
        else:
            want = k.to(flat.dtype)
        assert torch.equal(flat[s * per:e * per], want), (s, e)


def need_bytes(nbytes):
    torch.cuda.empty_cache()
    free, _ = torch.cuda.mem_get_info()
    if free < nbytes + (4 << 30):
        pytest.skip(f"needs {nbytes / 1e9:.1f} GB free on the device, {free / 1e9:.1f} GB available")


@pytest.mark.parametrize("m,n,eb", [(30011, 40009, 8), (40009, 30011, 8), (30000, 45000, 8),
                                    (60013, 60001, 4), (15013, 20011, 16)])
def test_rows_beyond_one_cta(m, n, eb):
    """min(m, n) * eb > 227 KB: the planner must pick the cluster row pass by itself."""
    need_bytes(m * n * eb)
    info = ipt.plan_info(m, n, eb)
    assert info["row_cluster"] >= 2, info
    x = index_tensor(m * n, eb)
    ipt.c2r(x, m, n, elem_bytes=eb)
    check_index_transpose(x, m, n, eb, 20000, seed=m + n)
    ipt.r2c(x, m, n, elem_bytes=eb)
    check_identity_chunked(x, m * n, eb)
    del x


def test_config5a_full_size():
    """BASELINE config 5a: m = 120011, n = 145820, fp64 (140 GB), gcd 1; M N > 2^32."""
    m, n, eb = 120011, 145820, 8
    need_bytes(m * n * eb)
    info = ipt.plan_info(m, n, eb)
    assert info["engine"] == "r2c" and info["c"] == 1 and info["row_cluster"] >= 2, info
    x = index_tensor(m * n, eb)
    ipt.c2r(x, m, n, elem_bytes=eb)
    check_index_transpose(x, m, n, eb, 20000, seed=5)
    ipt.r2c(x, m, n, elem_bytes=eb)
    check_identity_chunked(x, m * n, eb)
    del x
    torch.cuda.empty_cache()


def test_config5a_prime_gcd_5000():
    """BASELINE config 5a, second shape: m = 125000, n = 140000 fp64 (140 GB), gcd 5000 > 32:
    cluster row pass + the separate rotation pass (Eq. 36) over 140000-row column tiles +
    the column shuffle.  10^6 sampled outputs checked one by one with the oracle's Eqs. 7-8,
    then the full round trip r2c(c2r(x)) == x compared on the device."""
    m, n, eb = 125000, 140000, 8
    need_bytes(m * n * eb)
    info = ipt.plan_info(m, n, eb)
    assert info["c"] == 5000 and info["row_cluster"] >= 2 and info["launches"] == 3, info
    x = index_tensor(m * n, eb)
    ipt.c2r(x, m, n, elem_bytes=eb)
    check_index_transpose(x, m, n, eb, 1_000_000, seed=7)
    ipt.r2c(x, m, n, elem_bytes=eb)
    check_identity_chunked(x, m * n, eb)
    del x
    torch.cuda.empty_cache()
