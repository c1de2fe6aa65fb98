"""GPU parity of the warp-cooperative AoS helpers (include/ipt/aos.cuh; §6.2).

After warp_load_aos<S>, lane l's register k must hold chunk word l*S + k (reading C16, the
oracle's warp_load_aos_registers); warp_store_aos is the exact inverse; the three consumer
kernel variants (direct, vector, coalesced_ptr) must produce bit-identical outputs.
"""
import numpy as np
import pytest

import oracle
import workloads

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():  # pragma: no cover
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_ppopp_catanzarokg14_b200 as ipt  # noqa: E402


def dev(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


@pytest.mark.parametrize("S", list(range(1, 33)))
def test_warp_load_registers_match_oracle(S):
    nchunks = 7
    words = workloads.random_words(nchunks * 32 * S, 4, seed=S)
    src = dev(words)
    dump = torch.zeros_like(src)
    ipt.warp_load_dump(src, dump, nchunks, S)
    got = dump.cpu().numpy().reshape(nchunks, 32, S)  # [chunk][lane][register]
    for c in range(nchunks):
        R = oracle.warp_load_aos_registers(words[c * 32 * S:(c + 1) * 32 * S], S)  # [register][lane]
        assert np.array_equal(got[c], R.T), (S, c)


@pytest.mark.parametrize("S", list(range(1, 33)))
def test_warp_store_is_inverse(S):
    nchunks = 5
    regs = workloads.random_words(nchunks * 32 * S, 4, seed=100 + S)
    dst = torch.zeros(nchunks * 32 * S, dtype=torch.uint32, device="cuda")
    ipt.warp_store(dev(regs), dst, nchunks, S)
    assert np.array_equal(dst.cpu().numpy(), regs), S


@pytest.mark.parametrize("S", [1, 2, 3, 4, 5, 7, 8, 12, 16, 31, 32])
@pytest.mark.parametrize("count", [32 * 1000, 32 * 1000 + 13, 5])
def test_consumer_variants_agree(S, count):
    src_h = workloads.random_words(count * S, 4, seed=S * 7 + count)
    src = dev(src_h)
    ref_fill = np.arange(count * S, dtype=np.uint32)
    for variant in (ipt.AOS_DIRECT, ipt.AOS_VECTOR, ipt.AOS_COALESCED):
        dst = torch.zeros_like(src)
        ipt.aos_copy(src, dst, count, S, variant)
        assert np.array_equal(dst.cpu().numpy(), src_h), (S, count, variant)
        dst.zero_()
        ipt.aos_fill(dst, count, S, variant)
        assert np.array_equal(dst.cpu().numpy(), ref_fill), (S, count, variant)


@pytest.mark.parametrize("S", [1, 2, 3, 4, 5, 7, 8, 12, 16, 24, 31, 32])
@pytest.mark.parametrize("count", [32 * 500, 32 * 500 + 7, 9])
def test_random_access_gather_scatter(S, count):
    """warp_gather_aos / warp_scatter_aos (row f1, PAPER.md :1087, :1099): gather with a
    random index vector (repeats allowed) and scatter through a random permutation equal
    the oracle's struct-by-struct definitions (oracle.aos_gather / aos_scatter, pinned to
    numpy in test_oracle.py), bit for bit; direct, vector and cooperative variants all
    match; partial tail warps take the per-lane path."""
    rng = np.random.default_rng(S * 1000 + count)
    nsrc = count + 37
    src_h = workloads.random_words(nsrc * S, 4, seed=S + count).reshape(nsrc, S)
    idx_h = rng.integers(0, nsrc, size=count, dtype=np.uint32)
    want = oracle.aos_gather(src_h, idx_h, S).reshape(count, S)       # plain loops (oracle)
    perm = rng.permutation(count).astype(np.uint32)
    want_sc = oracle.aos_scatter(src_h[:count], perm, S).reshape(count, S)
    src, idx, pidx = dev(src_h.reshape(-1)), dev(idx_h), dev(perm)
    for variant in (ipt.AOS_DIRECT, ipt.AOS_VECTOR, ipt.AOS_COALESCED):
        dst = torch.zeros(count * S, dtype=torch.uint32, device="cuda")
        ipt.aos_gather(src, idx, dst, count, S, variant)
        assert np.array_equal(dst.cpu().numpy().reshape(count, S), want), (S, count, variant)
        dst.zero_()
        ipt.aos_scatter(src, pidx, dst, count, S, variant)
        assert np.array_equal(dst.cpu().numpy().reshape(count, S), want_sc), (S, count, variant)
