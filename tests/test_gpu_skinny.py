"""GPU parity of the skinny AoS <-> SoA engine (§6.1).

The engine (rolling long rows + one tmp row, n-row column tiles) is forced onto small
counts with IPT_SKINNY_MIN so that every fields count n in 2..32 is compared with the
oracle in full; BASELINE config 3 sizes (2**26 structs) are checked on sampled outputs
one by one with the oracle's Eqs. 7-8.
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


def to_dev(host):
    return torch.from_numpy(np.ascontiguousarray(host).view(np.uint8).reshape(-1).copy()).cuda()


class skinny_min:
    def __init__(self, v):
        self.v = v

    def __enter__(self):
        os.environ["IPT_SKINNY_MIN"] = str(self.v)

    def __exit__(self, *a):
        os.environ.pop("IPT_SKINNY_MIN", None)


class fuse_rot:
    def __init__(self, v):
        self.v = v

    def __enter__(self):
        os.environ["IPT_FUSE_ROT"] = self.v

    def __exit__(self, *a):
        os.environ.pop("IPT_FUSE_ROT", None)


@pytest.mark.parametrize("fold", ["1", "0"])
@pytest.mark.parametrize("count", [4099, 4096, 6000])
@pytest.mark.parametrize("eb", [4, 8])
def test_all_field_counts_both_directions(count, eb, fold):
    """fold=1: for gcd(n, count) > 1 the rotation is folded into the rolling-row locations
    (no rotation pass); fold=0: the separate rotation pass."""
    with skinny_min(1000), fuse_rot(fold):
        for n in range(2, 33):
            assert ipt.plan_info(count, n, eb)["engine"] == "skinny"
            host = workloads.random_words(count * n, eb, seed=count + n)
            x = to_dev(host)
            ipt.aos_to_soa(x, count, n, field_bytes=eb)
            soa = x.cpu().numpy().view(host.dtype)
            assert soa.tobytes() == oracle.aos_to_soa(host, count, n).tobytes(), (count, n, eb)
            ipt.soa_to_aos(x, count, n, field_bytes=eb)
            assert x.cpu().numpy().tobytes() == host.tobytes(), (count, n, eb)


def test_sixteen_byte_fields_and_c2r_export():
    """16-byte fields, and the same engine reached through ipt_c2r / ipt_r2c."""
    with skinny_min(1000):
        for n in (2, 3, 7, 16, 32):
            count = 3001
            host = workloads.random_words(count * n, 16, seed=n)
            hv = np.ascontiguousarray(host).view(np.dtype((np.void, 16))).reshape(-1)
            x = to_dev(host)
            ipt.c2r(x, count, n, elem_bytes=16)
            got = x.cpu().numpy().view(np.dtype((np.void, 16)))
            assert got.tobytes() == oracle.transpose(hv, count, n).tobytes(), n
            ipt.r2c(x, count, n, elem_bytes=16)
            assert x.cpu().numpy().tobytes() == np.ascontiguousarray(host).tobytes()


@pytest.mark.parametrize("n", [2, 3, 8])
def test_config3_full_size_sampled(n):
    """BASELINE config 3: 2**26 structs of n 4-byte fields (default engine selection)."""
    count = 1 << 26
    assert ipt.plan_info(count, n, 4)["engine"] == "skinny"
    host = workloads.random_words(count * n, 4, seed=n)
    x = to_dev(host)
    ipt.aos_to_soa(x, count, n, field_bytes=4)
    got = x.cpu().numpy().view(np.uint32)
    rng = random.Random(n)
    for _ in range(20000):  # P_{count,n} = C2R(count, n): output l holds input s*n + c (Eqs. 7-8)
        l = rng.randrange(count * n)
        i, j = divmod(l, n)
        si, sj = oracle.c2r_source(count, n, i, j)
        assert got[l] == host[si * n + sj]
    ipt.soa_to_aos(x, count, n, field_bytes=4)
    assert torch.equal(x, to_dev(host))


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.parametrize("fold", ["1", "0"])
def test_batched_one_launch_per_pass(eb, fold):
    """Skinny engine on a batch (ipt_c2r_batched / ipt_r2c_batched with a skinny shape): every
    pass is ONE launch over the batch (gridDim.y = matrix, a tmp row per matrix), packed and
    gapped strides, odd and even field counts (rotation folded or separate), compared in full;
    the launch count is that of one matrix."""
    with skinny_min(1000), fuse_rot(fold):
        for (count, n) in [(4099, 3), (4096, 6), (3001, 8)]:
            for gap in (0, 5):
                batch, stride = 4, count * n + gap
                host = workloads.random_words(batch * stride, eb, seed=count + n + gap)
                hv = np.ascontiguousarray(host).view(np.dtype((np.void, eb))).reshape(-1)
                x = to_dev(host)
                assert ipt.plan_info(count, n, eb)["engine"] == "skinny"
                l0 = ipt.launch_count()
                ipt.c2r_batched(x, batch, stride, count, n, elem_bytes=eb)
                torch.cuda.synchronize()
                launches = ipt.launch_count() - l0
                assert launches == ipt.plan_info(count, n, eb)["launches"], launches
                got = x.cpu().numpy().view(np.uint8).view(np.dtype((np.void, eb))).reshape(-1)
                for k in range(batch):
                    o = k * stride
                    assert got[o:o + count * n].tobytes() == oracle.transpose(hv[o:o + count * n], count, n).tobytes()
                    assert got[o + count * n:o + stride].tobytes() == hv[o + count * n:o + stride].tobytes()
                ipt.r2c_batched(x, batch, stride, count, n, elem_bytes=eb)
                assert x.cpu().numpy().tobytes() == np.ascontiguousarray(host).tobytes()


@pytest.mark.timeout(900)
def test_config3_all_field_counts_sampled():
    """Every call the bench's cfg3 key times: 2**26 structs x n = 2..32 4-byte fields,
    aos_to_soa then soa_to_aos. Index pattern (word l holds l mod 2^32); 2^17 sampled
    destinations plus the first and last 4096 checked against the oracle's Eqs. 7-8
    (oracle.source_many, P_{count,n} = C2R(count, n)), the whole output checked to be a
    permutation (sum and sum of squares), and the inverse checked to restore the input."""
    count = 1 << 26
    rng = np.random.default_rng(3)
    base = torch.arange(count * 32, dtype=torch.int64, device="cuda")
    for n in range(2, 33):
        total = count * n
        x = base[:total].to(torch.int32)
        u = x.to(torch.int64) & 0xffffffff
        s1, s2 = u.sum().item(), (u * u).sum().item()
        ipt.aos_to_soa(x, count, n, field_bytes=4)
        pos = np.concatenate([np.arange(4096), np.arange(total - 4096, total),
                              rng.integers(0, total, size=1 << 17)]).astype(np.int64)
        got = (x[torch.from_numpy(pos).cuda()].to(torch.int64) & 0xffffffff).cpu().numpy()
        want = oracle.source_many("c2r", count, n, pos)
        bad = np.nonzero(got != want)[0]
        assert bad.size == 0, (n, int(pos[bad[0]]), int(got[bad[0]]), int(want[bad[0]]))
        u = x.to(torch.int64) & 0xffffffff
        assert u.sum().item() == s1 and (u * u).sum().item() == s2, n
        ipt.soa_to_aos(x, count, n, field_bytes=4)
        assert torch.equal(x, base[:total].to(torch.int32)), n


def test_large_batch_of_small_skinny_matrices():
    """A batch of more skinny matrices than co-resident CTAs: the one-launch row shuffles
    (cooperative, grid barrier) fall back to one launch per row; every matrix compared in full."""
    count, n, batch = 1024, 3, 3000
    with skinny_min(1000):
        assert ipt.plan_info(count, n, 4)["engine"] == "skinny"
        host = workloads.random_words(batch * count * n, 4, seed=77)
        x = to_dev(host)
        ipt.c2r_batched(x, batch, count * n, count, n, elem_bytes=4)
        got = x.cpu().numpy().view(np.uint32)
        for k in (0, 1, batch // 2, batch - 1):
            o = k * count * n
            assert got[o:o + count * n].tobytes() == oracle.transpose(host[o:o + count * n], count, n).tobytes(), k
        ipt.r2c_batched(x, batch, count * n, count, n, elem_bytes=4)
        assert x.cpu().numpy().tobytes() == host.tobytes()
