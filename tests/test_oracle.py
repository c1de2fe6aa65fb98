"""Pins for the CPU oracle (runs without a GPU).

Every oracle function is checked against something other than itself: the paper's
printed figures (tests/golden, typed from PAPER.md), numpy's out-of-place transpose (a
library routine), the paper's theorems as invariants, inverse pairs, and brute force over
every small shape.  A dropped term, a wrong sign, a swapped index or a transposed operand
anywhere in oracle/ipt_oracle.c breaks at least one of these.
"""
import itertools

import numpy as np
import pytest

import oracle
import workloads


def words(count, eb, seed=0):
    w = workloads.random_words(count, eb, seed)
    if w.ndim == 2:  # 16-byte elements and multi-word records as opaque eb-byte elements
        return np.ascontiguousarray(w).view(np.dtype((np.void, eb))).reshape(-1)
    return w


def same(a, b):
    a = np.ascontiguousarray(a)
    b = np.ascontiguousarray(b)
    return a.shape == b.shape and a.tobytes() == b.tobytes()


def np_P(X, x, y):
    """numpy's out-of-place transpose of the row-major x-by-y buffer X."""
    return np.ascontiguousarray(np.asarray(X).reshape(x, y).T).reshape(-1)


# ---------------------------------------------------------------------------------------
# Paper fixtures
# ---------------------------------------------------------------------------------------
def test_fig1_direction_and_element16(golden):
    """PAPER.md:69-79 (Fig. 1) and :147-155: R2C maps left -> right, C2R right -> left;
    element 16 at (2, 0) lands at (1, 5) under R2C (Eq. 14)."""
    g = golden("fig1_m3_n8.txt")
    left = np.array(g["left"], dtype=np.uint32).ravel()
    right = np.array(g["right"], dtype=np.uint32).ravel()
    assert same(oracle.r2c_definition(left, 3, 8), right)
    assert same(oracle.c2r_definition(right, 3, 8), left)
    assert same(oracle.c2r_alg1(right, 3, 8), left)
    assert same(oracle.r2c_alg1(left, 3, 8), right)
    # Eq. 14: A_R2C[s(i,j), c(i,j)] = A[i,j]; the paper computes s(2,0)=1, c(2,0)=5.
    assert oracle.c2r_source(3, 8, 2, 0) == (1, 5)
    assert right.reshape(3, 8)[1, 5] == 16 == left.reshape(3, 8)[2, 0]


def test_fig2_algorithm1_intermediate_states(golden):
    """PAPER.md:607-621 (Fig. 2): the 4 x 8 C2R after each outer loop of Algorithm 1."""
    g = golden("fig2_m4_n8.txt")
    A = np.array(g["input"], dtype=np.uint32).ravel()
    out, snaps = oracle.c2r_alg1(A, 4, 8, snapshots=True)
    assert same(snaps[0], np.array(g["column_rotate"], dtype=np.uint32).ravel())
    assert same(snaps[1], np.array(g["row_shuffle"], dtype=np.uint32).ravel())
    assert same(snaps[2], np.array(g["column_shuffle"], dtype=np.uint32).ravel())
    assert same(out, np.array(g["column_shuffle"], dtype=np.uint32).ravel())
    # §4.2 gather forms: step 1 is the same Eq. 23 gather; steps 3+4 equal Eq. 26's shuffle.
    out2, s2 = oracle.c2r_gather_forms(A, 4, 8, snapshots=True)
    assert same(s2[0], np.array(g["column_rotate"], dtype=np.uint32).ravel())
    assert same(out2, np.array(g["column_shuffle"], dtype=np.uint32).ravel())
    # the inverse walks the figure backwards
    back, rs = oracle.r2c_alg1(out, 4, 8, snapshots=True)
    assert same(rs[0], np.array(g["row_shuffle"], dtype=np.uint32).ravel())
    assert same(rs[1], np.array(g["column_rotate"], dtype=np.uint32).ravel())
    assert same(back, A)


# ---------------------------------------------------------------------------------------
# Plain definitions vs numpy (Theorem 1 / 2)
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("eb", [1, 2, 4, 8, 16, 12, 24, 64])
def test_definitions_equal_numpy_transpose(eb):
    for m, n in [(1, 1), (1, 7), (7, 1), (3, 8), (8, 3), (5, 5), (12, 18), (17, 13), (64, 40)]:
        X = words(m * n, eb, seed=m * 100 + n)
        assert same(oracle.transpose(X, m, n), np_P(X, m, n))
        assert same(oracle.c2r_definition(X, m, n), np_P(X, m, n))       # C2R(m,n) = P_{m,n}
        assert same(oracle.r2c_definition(X, m, n), np_P(X, n, m))       # R2C(m,n) = P_{n,m}


def test_square_reduces_to_textbook_swap():
    """m = n: the transpose is A[i,j] <-> A[j,i]; C2R and R2C coincide."""
    for m in (1, 2, 5, 16, 33):
        X = words(m * m, 4, seed=m)
        ref = X.reshape(m, m).copy()
        for i in range(m):
            for j in range(i + 1, m):
                ref[i, j], ref[j, i] = ref[j, i], ref[i, j]
        assert same(oracle.c2r_alg1(X, m, m), ref.ravel())
        assert same(oracle.r2c_alg1(X, m, m), ref.ravel())


def test_theorem2_swapped_dimensions_transpose_column_major():
    """Theorem 2: C2R with m,n swapped transposes a column-major m x n array."""
    m, n = 6, 10
    A = words(m * n, 4, seed=5).reshape(m, n)
    colmajor = np.ascontiguousarray(A.T).ravel()            # A stored column-major
    out = oracle.c2r_alg1(colmajor, n, m)                   # swap m and n
    assert same(out, A.ravel())                             # = A^T stored column-major


# ---------------------------------------------------------------------------------------
# Brute force: Algorithm 1, its inverse, and the §4 gather forms on every small shape
# ---------------------------------------------------------------------------------------
def test_bruteforce_alg1_and_gather_forms_eb4():
    """Every m, n <= 64 (north_star: brute force over all m, n <= 64, coprime and not)."""
    for m, n in workloads.small_shapes(64):
        X = words(m * n, 4, seed=m * 1000 + n)
        ref = np_P(X, m, n)
        y = oracle.c2r_alg1(X, m, n)
        assert same(y, ref), (m, n)
        assert same(oracle.c2r_gather_forms(X, m, n), ref), (m, n)
        assert same(oracle.r2c_alg1(y, m, n), X), (m, n)
        assert same(oracle.r2c_gather_forms(y, m, n), X), (m, n)


@pytest.mark.parametrize("eb", [1, 2, 8, 16, 12])
def test_bruteforce_other_element_sizes(eb):
    """Every m, n <= 64 for the other element sizes as well (the words are opaque)."""
    for m, n in workloads.small_shapes(64):
        X = words(m * n, eb, seed=m * 1000 + n)
        ref = np_P(X, m, n)
        assert same(oracle.c2r_alg1(X, m, n), ref), (m, n)
        assert same(oracle.r2c_alg1(ref, m, n), X), (m, n)
        assert same(oracle.c2r_gather_forms(X, m, n), ref), (m, n)
        assert same(oracle.r2c_gather_forms(ref, m, n), X), (m, n)


def test_intermediate_states_of_alg1_and_gather_forms_agree():
    """Both C2R pipelines share step 1 (Eq. 23) and the row state (Eq. 24 scatter ==
    Eq. 31 gather); their last two gathers compose to Eq. 26 (p_j o q = s'_j, :715)."""
    for m, n in [(4, 8), (6, 9), (12, 18), (10, 25), (7, 5), (30, 12)]:
        X = words(m * n, 4, seed=m + n)
        _, a = oracle.c2r_alg1(X, m, n, snapshots=True)
        _, g = oracle.c2r_gather_forms(X, m, n, snapshots=True)
        if oracle.gcd(m, n) > 1:
            assert same(a[0], g[0])
        assert same(a[1], g[1])
        assert same(a[2], g[3])
        _, ra = oracle.r2c_alg1(np_P(X, m, n), m, n, snapshots=True)
        _, rg = oracle.r2c_gather_forms(np_P(X, m, n), m, n, snapshots=True)
        assert same(ra[0], rg[1])          # after the inverse column shuffle
        assert same(ra[1], rg[2])          # after the row gather by d'


# ---------------------------------------------------------------------------------------
# Theorems and lemmas as invariants
# ---------------------------------------------------------------------------------------
SMALL = [(m, n) for m in range(1, 25) for n in range(1, 25)]


def test_lemma1_periodicity_and_coprime_case():
    for m, n in SMALL:
        c = oracle.gcd(m, n)
        b = n // c
        for i in range(m):
            for j in range(n):
                assert oracle.eq22_d(m, n, i, j) == oracle.eq22_d(m, n, i, j + b)   # Lemma 1
                if c == 1:                                                          # :471-477
                    assert oracle.eq23_r(m, n, i, j) == i
                    assert oracle.eq24_dp(m, n, i, j) == oracle.eq22_d(m, n, i, j)


def test_theorem3_row_scatter_is_bijection():
    for m, n in SMALL:
        for i in range(m):
            assert sorted(oracle.eq24_dp(m, n, i, j) for j in range(n)) == list(range(n)), (m, n, i)


def test_gather_forms_are_inverses_and_compositions():
    for m, n in SMALL:
        for i in range(m):
            for j in range(n):
                # Eq. 31 inverts Eq. 24 (row shuffle)
                assert oracle.eq31_dpinv(m, n, i, oracle.eq24_dp(m, n, i, j)) == j
                assert oracle.eq24_dp(m, n, i, oracle.eq31_dpinv(m, n, i, j)) == j
        for i in range(m):
            assert oracle.eq34_qinv(m, n, oracle.eq33_q(m, n, i)) == i          # Eq. 34 o Eq. 33
            for j in range(n):
                assert oracle.eq32_p(m, n, oracle.eq33_q(m, n, i), j) == oracle.eq26_sp(m, n, i, j)
                assert oracle.eq35_pinv(m, n, oracle.eq32_p(m, n, i, j), j) == i  # Eq. 35
                assert oracle.eq36_rinv(m, n, oracle.eq23_r(m, n, i, j), j) == i  # Eq. 36


def test_mmi():
    for x, y in itertools.product(range(1, 60), range(1, 60)):
        if oracle.gcd(x, y) == 1:
            v = oracle.mmi(x, y)
            assert 0 <= v < y and (x * v) % y == 1 % y
    assert oracle.mmi(7, 1) == 0     # reading C4


@pytest.mark.parametrize("m,n", [(4, 8), (3, 8), (12, 18), (7, 13), (40, 24), (1, 9)])
def test_theorem6_reads_and_writes_per_element(m, n):
    """Theorem 6 proof: each element is read and written at most 6 times."""
    X = words(m * n, 4, seed=1)
    for fn in (oracle.c2r_alg1, oracle.r2c_alg1):
        _, (ar, aw, tr, tw) = fn(X, m, n, counts=True)
        steps = 3 if oracle.gcd(m, n) > 1 else 2
        assert (ar, aw, tr, tw) == (steps * m * n,) * 4
        assert ar + tr <= 6 * m * n and aw + tw <= 6 * m * n


def test_theorem7_linearization_independent():
    """Theorem 7: C2R/R2C with column-major indexing induce the same
    buffer permutation as with row-major indexing."""
    for m, n in [(3, 8), (4, 8), (6, 10), (9, 6), (11, 7), (16, 24), (25, 15)]:
        X = words(m * n, 4, seed=m * n)
        assert same(oracle.c2r_alg1(X, m, n, linearization="col"), oracle.c2r_alg1(X, m, n))
        assert same(oracle.r2c_alg1(X, m, n, linearization="col"), oracle.r2c_alg1(X, m, n))


# ---------------------------------------------------------------------------------------
# Export-level semantics (include/ipt.h) and AoS register mapping
# ---------------------------------------------------------------------------------------
def test_export_semantics_against_numpy():
    m, n = 5, 7
    A = words(m * n, 8, seed=3).reshape(m, n)
    row = A.ravel()
    col = np.ascontiguousarray(A.T).ravel()
    # c2r: the m x n input in `layout` becomes its n x m transpose in the same layout
    assert same(oracle.ipt_c2r(row, m, n, oracle.ROW_MAJOR), np.ascontiguousarray(A.T).ravel())
    assert same(oracle.ipt_c2r(col, m, n, oracle.COL_MAJOR), A.ravel())
    # r2c with the same arguments inverts c2r
    for lay, X in ((oracle.ROW_MAJOR, row), (oracle.COL_MAJOR, col)):
        assert same(oracle.ipt_r2c(oracle.ipt_c2r(X, m, n, lay), m, n, lay), X)
    # AoS <-> SoA (§6.1): struct k field f at k*fields+f  ->  field f of struct k at f*count+k
    cnt, f = 9, 3
    aos = words(cnt * f, 4, seed=9)
    soa = oracle.aos_to_soa(aos, cnt, f)
    for k in range(cnt):
        for fi in range(f):
            assert soa[fi * cnt + k] == aos[k * f + fi]
    assert same(oracle.soa_to_aos(soa, cnt, f), aos)


def test_warp_register_mapping():
    """§6.2 reading C16: lane l register k holds word l*S + k."""
    for S in (1, 2, 3, 5, 16):
        w = np.arange(32 * S, dtype=np.uint32)
        R = oracle.warp_load_aos_registers(w, S)
        assert R.shape == (S, 32)
        assert all(R[k, lane] == lane * S + k for k in range(S) for lane in range(32))
        # the register array is the R2C(S, 32) of the loaded chunk: chunk word k*32+l (the
        # coalesced load order, Eq. 4 column-major view) ... equals numpy's P_{32,S}.
        assert same(R.ravel(), np_P(w, 32, S))


@pytest.mark.parametrize("S", [1, 2, 3, 5, 16, 32])
def test_aos_gather_scatter_against_numpy(S):
    """Pins oracle.aos_gather / aos_scatter (Fig. 9 random-access AoS)
    to numpy fancy indexing of the struct array, an independent implementation; plus the
    invariants: gathering through a permutation and scattering back through the same
    permutation is the identity, and a gather with the identity index is a copy."""
    rng = np.random.default_rng(S)
    nsrc, count = 301, 257
    src = rng.integers(0, 2**32, size=(nsrc, S), dtype=np.uint32)
    idx = rng.integers(0, nsrc, size=count, dtype=np.uint32)          # repeats allowed
    assert same(oracle.aos_gather(src, idx, S), src[idx].reshape(-1))
    perm = rng.permutation(count).astype(np.uint32)
    want = np.zeros((count, S), dtype=np.uint32)
    want[perm] = src[:count]
    got = oracle.aos_scatter(src[:count], perm, S)
    assert same(got, want.reshape(-1))
    assert same(oracle.aos_scatter(oracle.aos_gather(src[:count], perm, S), perm, S), src[:count].reshape(-1))
    ident = np.arange(nsrc, dtype=np.uint32)
    assert same(oracle.aos_gather(src, ident, S), src.reshape(-1))
    assert oracle.aos_gather(src, idx[:0], S).size == 0


@pytest.mark.parametrize("m,n", [(1, 1), (1, 9), (9, 1), (6, 4), (7, 11), (12, 18), (64, 40), (1200, 1800)])
def test_source_many_against_numpy(m, n):
    """oracle.source_many (Eqs. 7-10, used by the full-size sampled GPU checks) names the
    element numpy's out-of-place transpose puts at each destination: c2r(m, n) = P_{m,n},
    r2c(m, n) = P_{n,m} (Theorem 1 buffer form)."""
    pos = np.arange(m * n, dtype=np.int64)
    idx = np.arange(m * n, dtype=np.int64)
    assert same(oracle.source_many("c2r", m, n, pos), np_P(idx, m, n))
    assert same(oracle.source_many("r2c", m, n, pos), np_P(idx, n, m))
    rng = np.random.default_rng(m * 31 + n)
    sub = rng.integers(0, m * n, size=min(500, m * n))
    assert same(oracle.source_many("c2r", m, n, sub), np_P(idx, m, n)[sub])
