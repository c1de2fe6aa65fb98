"""GPU parity: the CUDA path (through the C ABI) against the CPU oracle, bit-exact.

Tolerance is zero: the transpose moves opaque words (north_star: "bit-exact against the
oracle for every element type, including floats").  Inputs are random bit patterns from
workloads.py (NaN payloads, -0.0 and subnormals included when viewed as floats).
"""
import math
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


def vwords(host, eb):
    """numpy view of host words as opaque eb-byte elements."""
    return np.ascontiguousarray(host).view(np.dtype((np.void, eb))).reshape(-1)


def to_dev(host):
    return torch.from_numpy(np.ascontiguousarray(host).view(np.uint8).reshape(-1).copy()).to(DEV)


def dev_bytes(t):
    return t.cpu().numpy().tobytes()


class forced_engine:
    def __init__(self, eng):
        self.eng = eng

    def __enter__(self):
        self.old = os.environ.get("IPT_FORCE_ENGINE")
        if self.eng:
            os.environ["IPT_FORCE_ENGINE"] = self.eng
        else:
            os.environ.pop("IPT_FORCE_ENGINE", None)

    def __exit__(self, *a):
        if self.old is None:
            os.environ.pop("IPT_FORCE_ENGINE", None)
        else:
            os.environ["IPT_FORCE_ENGINE"] = self.old


class debug_passes:
    def __init__(self, k):
        self.k = k

    def __enter__(self):
        os.environ["IPT_DEBUG_PASSES"] = str(self.k)

    def __exit__(self, *a):
        os.environ.pop("IPT_DEBUG_PASSES", None)


def run_packed(shapes, eb, op, layout, engine, seed):
    """Pack every shape into one device buffer, run `op` on each slice, compare each slice
    with the oracle, then run the inverse and compare with the input."""
    offs, tot = [], 0
    for m, n in shapes:
        offs.append(tot)
        tot += m * n + 3  # gaps between matrices must stay untouched
    host = workloads.random_words(tot, eb, seed)
    hv = vwords(host, eb)
    buf = to_dev(host)
    base = buf.data_ptr()
    inv = ipt.r2c if op is ipt.c2r else ipt.c2r
    with forced_engine(engine):
        for (m, n), o in zip(shapes, offs):
            op(base + o * eb, m, n, elem_bytes=eb, layout=layout)
        got = vwords(buf.cpu().numpy(), eb)
        oc = oracle.ipt_c2r if op is ipt.c2r else oracle.ipt_r2c
        for (m, n), o in zip(shapes, offs):
            want = oc(hv[o:o + m * n], m, n, {"row": oracle.ROW_MAJOR, "col": oracle.COL_MAJOR}[layout])
            assert got[o:o + m * n].tobytes() == want.tobytes(), (m, n, eb, layout, engine)
            assert got[o + m * n:o + m * n + 3].tobytes() == hv[o + m * n:o + m * n + 3].tobytes()
        for (m, n), o in zip(shapes, offs):
            inv(base + o * eb, m, n, elem_bytes=eb, layout=layout)
    torch.cuda.synchronize()
    assert dev_bytes(buf) == np.ascontiguousarray(host).tobytes()


class env_var:
    def __init__(self, name, value):
        self.name, self.value = name, value

    def __enter__(self):
        self.old = os.environ.get(self.name)
        os.environ[self.name] = self.value

    def __exit__(self, *a):
        if self.old is None:
            os.environ.pop(self.name, None)
        else:
            os.environ[self.name] = self.old


@pytest.mark.parametrize("fuse", ["1", "0"])
@pytest.mark.parametrize("engine", [None, "c2r", "r2c"])
def test_bruteforce_all_shapes_to_64_fp32(engine, fuse):
    """fuse=1: gcd <= 32 takes the fused rotation + row pass; fuse=0: the separate
    column-rotation pass for every gcd > 1."""
    shapes = workloads.small_shapes(64)
    with env_var("IPT_FUSE_ROT", fuse):
        run_packed(shapes, 4, ipt.c2r, "row", engine, seed=11)


@pytest.mark.parametrize("fuse", ["1", "0"])
@pytest.mark.parametrize("eb", [8, 16])
@pytest.mark.parametrize("engine", ["c2r", "r2c"])
def test_bruteforce_shapes_to_64_wide_elements(eb, engine, fuse):
    """Every m, n <= 64 for 8- and 16-byte elements too, both engines, fused rotation on and off."""
    with env_var("IPT_FUSE_ROT", fuse):
        run_packed(workloads.small_shapes(64), eb, ipt.c2r, "row", engine, seed=eb)


@pytest.mark.parametrize("shape", [(1200, 1816), (1816, 1200), (4096, 3000), (96, 40), (640, 32 * 33)])
@pytest.mark.parametrize("engine", ["c2r", "r2c"])
def test_fused_rotation_each_pass(shape, engine):
    """gcd in 2..32: the rotation folds into the row pass (Eq. 23 + Eq. 31 for
    C2R, Eq. 24 + Eq. 36 for R2C).  Each of the two passes is compared with the oracle's
    gather-form snapshot after the same steps."""
    m, n = shape
    eb = 4
    assert 1 < math.gcd(m, n) <= 32
    host = workloads.random_words(m * n, eb, seed=m ^ n)
    with forced_engine(engine):
        x = to_dev(host)
        ipt.c2r(x, m, n, elem_bytes=eb)
        assert dev_bytes(x) == oracle.transpose(host, m, n).tobytes()
        ipt.r2c(x, m, n, elem_bytes=eb)
        assert dev_bytes(x) == host.tobytes()
        if engine == "c2r":       # C2R(M=m, N=n): [r_j + d'^{-1}], p_j o q
            _, snaps = oracle.c2r_gather_forms(host, m, n, snapshots=True)
            expect = [snaps[1], snaps[3]]
        else:                     # R2C(M=n, N=m): q^{-1} o p^{-1}, [d' + r^{-1}]
            _, snaps = oracle.r2c_gather_forms(host, n, m, snapshots=True)
            expect = [snaps[1], snaps[3]]
        for k, e in enumerate(expect, start=1):
            x = to_dev(host)
            with debug_passes(k):
                ipt.c2r(x, m, n, elem_bytes=eb)
            assert dev_bytes(x) == e.tobytes(), f"pass {k}"
        info = ipt.plan_info(m, n, eb)
        assert info["launches"] == 2, info


@pytest.mark.parametrize("layout", ["row", "col"])
@pytest.mark.parametrize("op", ["c2r", "r2c"])
def test_layouts_and_directions(layout, op):
    shapes = [(m, n) for m in (1, 2, 3, 7, 16, 33, 64, 100) for n in (1, 2, 5, 8, 31, 64, 97)]
    run_packed(shapes, 4, getattr(ipt, op), layout, None, seed=3)
    run_packed(shapes, 8, getattr(ipt, op), layout, None, seed=4)


@pytest.mark.parametrize("engine", ["c2r", "r2c"])
def test_config1_matches_algorithm1_and_each_pass(engine):
    """BASELINE config 1: m=1200, n=1800, 4-byte elements, gcd 600 (pre-rotation)."""
    m, n, eb = 1200, 1800, 4
    host = workloads.random_words(m * n, eb, seed=1)
    want = oracle.c2r_alg1(host, m, n)                       # Algorithm 1
    assert want.tobytes() == oracle.transpose(host, m, n).tobytes()
    with forced_engine(engine):
        x = to_dev(host)
        ipt.c2r(x, m, n, elem_bytes=eb)
        assert dev_bytes(x) == want.tobytes()
        ipt.r2c(x, m, n, elem_bytes=eb)
        assert dev_bytes(x) == host.tobytes()
        # per-pass parity against the oracle's §4.2 / §4.3 gather-form snapshots
        if engine == "c2r":       # C2R(M=1200, N=1800): [r_j], d'^{-1}, p_j o q
            _, snaps = oracle.c2r_gather_forms(host, m, n, snapshots=True)
            expect = [snaps[0], snaps[1], snaps[3]]
        else:                     # R2C(M=1800, N=1200): q^{-1} o p^{-1}, d', [r^{-1}]
            _, snaps = oracle.r2c_gather_forms(host, n, m, snapshots=True)
            expect = [snaps[1], snaps[2], snaps[3]]
        for k, e in enumerate(expect, start=1):
            x = to_dev(host)
            with debug_passes(k):
                ipt.c2r(x, m, n, elem_bytes=eb)
            assert dev_bytes(x) == e.tobytes(), f"pass {k}"


def test_misaligned_base_and_batched_with_gaps():
    m, n = 37, 91
    for eb in (4, 8):
        for shift in (1, 2, 3):  # base not 16-byte aligned
            batch, stride = 5, m * n + 7
            tot = shift + batch * stride
            host = workloads.random_words(tot, eb, seed=shift)
            hv = vwords(host, eb)
            x = to_dev(host)
            ipt.c2r_batched(x.data_ptr() + shift * eb, batch, stride, m, n, elem_bytes=eb)
            got = vwords(x.cpu().numpy(), eb)
            want = hv.copy()
            for k in range(batch):
                o = shift + k * stride
                want[o:o + m * n] = oracle.ipt_c2r(hv[o:o + m * n], m, n)
            assert got.tobytes() == want.tobytes()
            ipt.r2c_batched(x.data_ptr() + shift * eb, batch, stride, m, n, elem_bytes=eb)
            assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()


def test_two_streams_disjoint_buffers():
    shapes = [(300, 451), (512, 384)]
    hosts = [workloads.random_words(m * n, 4, seed=i) for i, (m, n) in enumerate(shapes)]
    xs = [to_dev(h) for h in hosts]
    torch.cuda.synchronize()  # the H2D copies ran on the default stream
    ss = [torch.cuda.Stream(), torch.cuda.Stream()]
    for rep in range(4):
        for (m, n), x, s in zip(shapes, xs, ss):
            with torch.cuda.stream(s):
                ipt.c2r(x, m, n, elem_bytes=4, stream=s)
                if rep < 3:
                    ipt.r2c(x, m, n, elem_bytes=4, stream=s)
    torch.cuda.synchronize()
    for (m, n), x, h in zip(shapes, xs, hosts):
        assert dev_bytes(x) == oracle.transpose(h, m, n).tobytes()


def test_degenerate_shapes():
    """m or n = 1: identity; m = n: textbook swap; n | m (b = 1) and m | n (a = 1)."""
    shapes = [(1, 1), (1, 500), (500, 1), (2, 2), (97, 97), (256, 256), (1000, 10), (10, 1000),
              (4096, 64), (64, 4096), (2, 3000), (3000, 2), (6, 4), (4, 6), (1024, 1023), (1023, 1024)]
    for eb in (4, 8, 16):
        run_packed(shapes, eb, ipt.c2r, "row", None, seed=eb + 100)


def _sampled_check(got_words, host_words, m, n, samples, rng):
    """Check sampled outputs one by one with the oracle's Eqs. 7-8 source function:
    ipt_c2r(m, n, ROW) is the C2R of the m x n buffer (Theorem 1), so output element
    l = i*n + j (Eq. 1) holds input element s(i,j)*n + c(i,j) (Eq. 11)."""
    for _ in range(samples):
        l = rng.randrange(m * n)
        i, j = divmod(l, n)                 # C2R output position on the m x n view
        si, sj = oracle.c2r_source(m, n, i, j)
        assert got_words[l] == host_words[si * n + sj], (m, n, l)


@pytest.mark.parametrize("eb", [4, 8])
def test_sweep_shapes_full_size(eb):
    """Config-2 shapes at full size (the bench workload): full comparison with the oracle's
    plain transpose for the first shapes, sampled one-by-one checks for the rest."""
    rng = random.Random(eb)
    for k, (m, n) in enumerate(workloads.sweep_shapes(6)):
        host = workloads.random_words(m * n, eb, seed=k)
        x = to_dev(host)
        ipt.c2r(x, m, n, elem_bytes=eb)
        got = x.cpu().numpy().view(host.dtype)
        if k < 2:
            assert got.tobytes() == oracle.transpose(host, m, n).tobytes(), (m, n)
        else:
            _sampled_check(got, host, m, n, 20000, rng)
        ipt.r2c(x, m, n, elem_bytes=eb)
        assert torch.equal(x, to_dev(host)), (m, n)


def test_config5b_batch_shape_sampled():
    """Config 5b matrices (4096 x 3000 float32, gcd 8) in a batch: whole-matrix comparison
    of the first, sampled one-by-one checks (oracle Eqs. 7-8) of the others."""
    m, n, batch = 4096, 3000, 6
    host = workloads.random_words(batch * m * n, 4, seed=55)
    x = to_dev(host)
    ipt.c2r_batched(x, batch, m * n, m, n, elem_bytes=4)
    got = x.cpu().numpy().view(np.uint32)
    assert got[:m * n].tobytes() == oracle.transpose(host[:m * n], m, n).tobytes()
    rng = random.Random(5)
    for k in range(1, batch):
        _sampled_check(got[k * m * n:(k + 1) * m * n], host[k * m * n:(k + 1) * m * n], m, n, 5000, rng)
    ipt.r2c_batched(x, batch, m * n, m, n, elem_bytes=4)
    assert torch.equal(x, to_dev(host))


@pytest.mark.parametrize("twb", ["128", "256", "512"])
@pytest.mark.parametrize("pipe", ["1", "0"])
def test_column_tile_widths_and_small_bands(twb, pipe):
    """Column-pass geometry: every tile width (16-byte hull staging, 16-byte vector stores
    with element stores at misaligned segment ends), tiny bands (IPT_COL_SMEM small, so a
    tile spans many group members and the halo crosses band edges), pipelined and one-unit
    kernels; the separate rotation pass (IPT_FUSE_ROT=0) exercises COL_ROT.  Shapes mix
    coprime / gcd > 1, ragged right tiles and rows misaligned to 16 bytes."""
    shapes = [(1200, 1800), (97, 1031), (1031, 97), (513, 700), (700, 513), (64, 4096), (2003, 129),
              (384, 640), (129, 2003)]
    with env_var("IPT_TILE_BYTES", twb), env_var("IPT_COL_PIPE", pipe), env_var("IPT_COL_SMEM", "12000"), \
            env_var("IPT_FUSE_ROT", "0"):
        for eb in (4, 8, 16):
            for engine in ("c2r", "r2c"):
                run_packed(shapes, eb, ipt.c2r, "row", engine, seed=int(twb) + eb)


@pytest.mark.parametrize("stage", ["1", "16384", "200000"])
@pytest.mark.parametrize("fuse", ["1", "0"])
def test_row_groups(stage, fuse):
    """Row pass in groups of R rows per CTA stage (IPT_ROW_STAGE bytes: R = 1, the default,
    and the largest R); groups that straddle the last rows (f2 = 1 tails, C2R wrap rows of
    the fused rotation), partial last groups, M < R, and batches whose groups must not
    cross matrix boundaries."""
    shapes = [(1200, 1800), (1114, 5285), (5285, 1114), (1026, 19126 // 7), (333, 999), (7, 300), (300, 7),
              (64, 96), (96, 64), (130, 2050), (2050, 130)]
    with env_var("IPT_ROW_STAGE", stage), env_var("IPT_FUSE_ROT", fuse):
        for eb in (4, 8):
            for engine in ("c2r", "r2c"):
                run_packed(shapes, eb, ipt.c2r, "row", engine, seed=len(stage) + eb)
        m, n, batch = 130, 2050, 3
        host = workloads.random_words(batch * m * n, 4, seed=9)
        x = to_dev(host)
        ipt.c2r_batched(x, batch, m * n, m, n, elem_bytes=4)
        got = x.cpu().numpy().view(np.uint32)
        for k in range(batch):
            assert got[k * m * n:(k + 1) * m * n].tobytes() == oracle.transpose(host[k * m * n:(k + 1) * m * n], m, n).tobytes()


@pytest.mark.parametrize("lagd", ["1", "3", "1000"])
def test_lagged_tile_layouts(lagd):
    """Shuffle pass with lagged tile layouts (D = IPT_COL_LAGD tiles, clamped to ntiles - 1):
    tiles t < D go through the side block, the rest D tiles to the left; the row pass reads
    (R2C) / writes (C2R) that layout.  Both engines, fused and separate rotation, ragged last
    tiles, rows misaligned to 16 bytes, batches (the side block of each matrix aligned like
    its rows), and IPT_COL_LAG=0 (per-tile barrier) for comparison."""
    shapes = [(1200, 1800), (1031, 97), (97, 1031), (513, 700), (700, 513), (2003, 129), (129, 2003), (333, 4099)]
    for lag in ("1", "0"):
        with env_var("IPT_COL_LAGD", lagd), env_var("IPT_COL_LAG", lag):
            for fuse in ("1", "0"):
                with env_var("IPT_FUSE_ROT", fuse):
                    for eb in (4, 8, 16):
                        for engine in ("c2r", "r2c"):
                            run_packed(shapes, eb, ipt.c2r, "row", engine, seed=eb + len(lagd))
            m, n, batch = 300, 1001, 4
            for eb in (4, 8):
                host = workloads.random_words(1 + batch * (m * n + 5), eb, seed=77)
                hv = vwords(host, eb)
                x = to_dev(host)
                ipt.c2r_batched(x.data_ptr() + eb, batch, m * n + 5, m, n, elem_bytes=eb)
                got = vwords(x.cpu().numpy(), eb)
                for k in range(batch):
                    o = 1 + k * (m * n + 5)
                    assert got[o:o + m * n].tobytes() == oracle.ipt_c2r(hv[o:o + m * n], m, n).tobytes()
                ipt.r2c_batched(x.data_ptr() + eb, batch, m * n + 5, m, n, elem_bytes=eb)
                assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()


@pytest.mark.parametrize("vec", ["1", "0"])
def test_fused_rotation_vector_gather(vec):
    """Fused C2R rotation + row pass, rows with f2 = 0 gathered in 16-byte output chunks of
    the row's aligned chunk grid (IPT_ROW_VEC=1: stepped walk, vector stores, element stores
    at the row ends and at a chunk straddling the lagged split) vs the per-element walk
    (IPT_ROW_VEC=0): gcd 2..32, misaligned rows, row groups, every element size, both lag
    settings."""
    shapes = [(1200, 1816), (1816, 1200), (96, 40), (640, 32 * 33), (2 * 1009, 2 * 1013), (30 * 37, 30 * 41),
              (4 * 999, 4 * 250), (2 * 3001, 2 * 2203), (6 * 301, 6 * 77)]
    for lag in ("1", "0"):
        with env_var("IPT_ROW_VEC", vec), env_var("IPT_COL_LAG", lag):
            for eb in (4, 8, 16):
                run_packed(shapes, eb, ipt.c2r, "row", "c2r", seed=eb * 7 + len(vec))


# ---------------------------------------------------------------------------------------
# Multi-word elements (records): elem_bytes = k*w, run as P_{x,y*k} then
# P_{k,x} on w-byte words (include/ipt.h).  The oracle moves eb-byte records directly.
# ---------------------------------------------------------------------------------------
@pytest.mark.parametrize("eb", [12, 20, 24, 32, 48, 64, 96])
def test_multiword_small_shapes_bit_exact(eb):
    shapes = [(m, n) for m, n in workloads.small_shapes(24) if (m * 7 + n) % 5 == 0]
    run_packed(shapes, eb, ipt.c2r, "row", None, seed=eb)
    run_packed(shapes[::3], eb, ipt.r2c, "col", None, seed=eb + 1)


@pytest.mark.parametrize("m,n,eb", [(1200, 1800, 12), (1800, 1200, 24), (333, 4097, 32), (4096, 3000 // 8, 64),
                                    (5000, 7, 12), (3, 20000, 48), (2000, 2100, 128), (2100, 2000, 128)])
def test_multiword_config_shapes(m, n, eb):
    host = workloads.random_words(m * n, eb, seed=m + n + eb)
    x = to_dev(host)
    ipt.c2r(x, m, n, elem_bytes=eb)
    assert dev_bytes(x) == oracle.transpose(vwords(host, eb), m, n).tobytes()
    ipt.r2c(x, m, n, elem_bytes=eb)
    assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()


@pytest.mark.parametrize("offset", [4, 8, 12])
def test_multiword_base_alignment(offset):
    """Bases aligned to 4 or 8 bytes only pick narrower words (the result is the same)."""
    m, n, eb = 37, 91, 32
    host = workloads.random_words(m * n + 4, eb, seed=offset)
    buf = to_dev(host)
    ipt.c2r(buf.data_ptr() + offset, m, n, elem_bytes=eb)
    raw = np.ascontiguousarray(host).view(np.uint8).reshape(-1)
    body = raw[offset:offset + m * n * eb].copy()
    want = oracle.transpose(body.view(np.dtype((np.void, eb))), m, n).tobytes()
    got = dev_bytes(buf)
    assert got[offset:offset + m * n * eb] == want
    assert got[:offset] == raw[:offset].tobytes() and got[offset + m * n * eb:] == raw[offset + m * n * eb:].tobytes()


@pytest.mark.parametrize("packed", [True, False])
@pytest.mark.parametrize("B,m,n,eb", [(5, 61, 45, 24), (5, 45, 61, 24), (2, 900, 950, 256)])
def test_multiword_batched(packed, B, m, n, eb):
    """Small blocks go through the shared-memory record pass; 900 x 256 B blocks (> 220 KiB)
    are staged in global scratch slots."""
    stride = m * n + (0 if packed else 7)
    host = workloads.random_words(B * stride, eb, seed=B + stride)
    hv = vwords(host, eb)
    buf = to_dev(host)
    ipt.c2r_batched(buf, B, stride, m, n, elem_bytes=eb)
    got = vwords(buf.cpu().numpy(), eb)
    for k in range(B):
        o = k * stride
        assert got[o:o + m * n].tobytes() == oracle.transpose(hv[o:o + m * n], m, n).tobytes()
        assert got[o + m * n:o + stride].tobytes() == hv[o + m * n:o + stride].tobytes()
    ipt.r2c_batched(buf, B, stride, m, n, elem_bytes=eb)
    assert dev_bytes(buf) == np.ascontiguousarray(host).tobytes()


@pytest.mark.parametrize("B,m,n,eb,stride", [(1, 300, 257, 24, None), (3, 97, 130, 32, 97 * 130),
                                             (3, 130, 97, 12, 130 * 97 + 5)])
def test_multiword_engine_fallback(B, m, n, eb, stride):
    """IPT_RECORD_ENGINE=1: both word-level steps on the engine (the path for blocks beyond
    the record pass's scratch cap), packed and gapped batches."""
    stride = stride or m * n
    host = workloads.random_words(B * stride, eb, seed=m * n + eb)
    hv = vwords(host, eb)
    buf = to_dev(host)
    with env_var("IPT_RECORD_ENGINE", "1"):
        ipt.c2r_batched(buf, B, stride, m, n, elem_bytes=eb)
        got = vwords(buf.cpu().numpy(), eb)
        for k in range(B):
            o = k * stride
            assert got[o:o + m * n].tobytes() == oracle.transpose(hv[o:o + m * n], m, n).tobytes()
            assert got[o + m * n:o + stride].tobytes() == hv[o + m * n:o + stride].tobytes()
        ipt.r2c_batched(buf, B, stride, m, n, elem_bytes=eb)
    assert dev_bytes(buf) == np.ascontiguousarray(host).tobytes()


def test_multiword_aos_soa_records():
    """Skinny entry point with 12-byte fields: count structs of `fields` 12-byte records."""
    count, fields, eb = 100003, 5, 12
    host = workloads.random_words(count * fields, eb, seed=3)
    x = to_dev(host)
    ipt.aos_to_soa(x, count, fields, field_bytes=eb)
    assert dev_bytes(x) == oracle.aos_to_soa(vwords(host, eb), count, fields).tobytes()
    ipt.soa_to_aos(x, count, fields, field_bytes=eb)
    assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()


def test_multiword_scratch_and_plan():
    """The plan of a record call reports the first word-level step and both steps' launches."""
    g12, o12 = ipt.scratch_bytes(1200, 1800, 12)
    g4, o4 = ipt.scratch_bytes(1200, 1800 * 3, 4)
    assert g12 >= g4 and o12 >= o4
    info = ipt.plan_info(1200, 1800, 32)  # 32 B = two 16-byte words
    ref = ipt.plan_info(1200, 3600, 16)
    assert all(info[k] == ref[k] for k in ("engine", "M", "N", "c"))
    assert info["launches"] > ref["launches"]
    with pytest.raises(ipt.IptError):
        ipt.scratch_bytes(10, 10, 6)
    # sub-word: the packed-word engine step (y % g == 0: P_{x,y/g}; else P_{x/g,y}) + 1 launch
    sub = ipt.plan_info(1200, 1800, 2)  # both sides even, x <= y: split
    ref = ipt.plan_info(1200, 900, 4)
    assert all(sub[k] == ref[k] for k in ("engine", "M", "N", "c"))
    assert sub["launches"] == ref["launches"] + 1
    sub = ipt.plan_info(1200, 1801, 1)
    ref = ipt.plan_info(300, 1801, 4)
    assert all(sub[k] == ref[k] for k in ("engine", "M", "N", "c"))
    with pytest.raises(ipt.IptError):
        ipt.plan_info(7, 9, 2)


# ---------------------------------------------------------------------------------------
# Sub-word elements (1 and 2 bytes): 4 / eb elements per engine word plus
# the record-block split/merge pass (include/ipt.h).  Every buffer starts 4-byte aligned.
# ---------------------------------------------------------------------------------------
def _subword_roundtrip(m, n, eb, layout="row", seed=0):
    host = workloads.random_words(m * n, eb, seed)
    x = to_dev(host)
    lay = {"row": oracle.ROW_MAJOR, "col": oracle.COL_MAJOR}[layout]
    ipt.c2r(x, m, n, elem_bytes=eb, layout=layout)
    assert dev_bytes(x) == oracle.ipt_c2r(host, m, n, lay).tobytes(), (m, n, eb, layout)
    ipt.r2c(x, m, n, elem_bytes=eb, layout=layout)
    assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()


@pytest.mark.parametrize("eb", [1, 2])
def test_subword_small_shapes_bit_exact(eb):
    g = 4 // eb
    for m, n in workloads.small_shapes(24):
        if (m % g == 0 or n % g == 0) and (m * 5 + n) % 3 == 0:
            _subword_roundtrip(m, n, eb, "row" if (m + n) % 2 else "col", seed=m * 31 + n)


@pytest.mark.parametrize("m,n,eb", [(1200, 1800, 2), (1200, 1800, 1), (14414, 6565, 2), (6565, 14414, 2),
                                    (17226, 6052, 1), (3, 20000, 2), (20001, 4, 1), (70001, 2, 2),
                                    (1 << 20, 4, 1), (4, 1 << 20, 1), (1 << 20, 2, 2), (1800, 1200, 2)])
def test_subword_config_shapes(m, n, eb):
    _subword_roundtrip(m, n, eb, seed=m ^ n)


def test_subword_batched_and_unsupported():
    B, m, n, eb = 3, 50, 37, 2
    stride = m * n + 6
    host = workloads.random_words(B * stride, eb, seed=9)
    buf = to_dev(host)
    ipt.c2r_batched(buf, B, stride, m, n, elem_bytes=eb)
    got = buf.cpu().numpy().view(host.dtype)
    for k in range(B):
        o = k * stride
        assert got[o:o + m * n].tobytes() == oracle.transpose(host[o:o + m * n], m, n).tobytes()
        assert got[o + m * n:o + stride].tobytes() == host[o + m * n:o + stride].tobytes()
    ipt.r2c_batched(buf, B, stride, m, n, elem_bytes=eb)
    assert dev_bytes(buf) == host.tobytes()
    with pytest.raises(ipt.IptError):
        ipt.c2r(buf, 7, 9, elem_bytes=2)


# ---------------------------------------------------------------------------------------
# Round 2: every call the bench times, compared in full; scale cases of the separate
# rotation and of the fused pass; robustness of the fused pass's cross-CTA waits.
# ---------------------------------------------------------------------------------------
def _oracle_pool():
    import concurrent.futures as cf
    return cf.ThreadPoolExecutor(max_workers=4)  # ctypes releases the GIL in the oracle


def _fast_words(count, eb, seed):
    return workloads.fast_random_words(count, eb, seed)


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.timeout(1800)
def test_bench_sweep_calls_full(eb):
    """The exact calls bench.py times (workloads.sweep_shapes(48), BASELINE configs[1]):
    ipt_c2r(m, n) and ipt_r2c(m, n) of every shape, each compared IN FULL with the oracle's
    plain transpose (Theorem 1 buffer form; c2r = P_{m,n}, r2c = P_{n,m}, reading C18).
    Covers gcd 1, the fused rotation (gcd 2..32), the separate rotation (gcd > 32) and
    both engines as the planner picks them."""
    shapes = workloads.sweep_shapes(48)
    pool = _oracle_pool()
    maxel = max(m * n for m, n in shapes)
    dbuf = torch.empty(maxel * eb, dtype=torch.uint8, device=DEV)
    pending = []
    for k, (m, n) in enumerate(shapes):
        for op in ("c2r", "r2c"):
            host = _fast_words(m * n, eb, seed=1000 * k + (op == "r2c") + 10 * eb)
            want = pool.submit(getattr(oracle, "ipt_" + op), host, m, n)
            x = dbuf[:m * n * eb]
            x.copy_(torch.from_numpy(host.view(np.uint8)))
            getattr(ipt, op)(x, m, n, elem_bytes=eb)
            got = x.cpu().numpy()
            pending.append(((m, n, op), got, want))
            while len(pending) > 3:
                key, g, w = pending.pop(0)
                assert g.tobytes() == w.result().tobytes(), key
    for key, g, w in pending:
        assert g.tobytes() == w.result().tobytes(), key
    pool.shutdown()


@pytest.mark.parametrize("m,n,eb", [(19800, 13200, 4), (13200, 19800, 4), (14000, 10500, 8), (6000, 9000, 16)])
def test_separate_rotation_at_hbm_scale(m, n, eb):
    """gcd > 32: the column rotation (Eq. 23 before / Eq. 36 after) runs as its own
    column-tile pass (COL_ROT) on matrices far larger than L2 (0.8-1.1 GB), compared in
    full with the oracle in both directions."""
    import math
    assert math.gcd(m, n) > 32
    assert ipt.plan_info(m, n, eb)["launches"] == 3
    host = _fast_words(m * n, eb, seed=m + n + eb)
    x = to_dev(host)
    ipt.c2r(x, m, n, elem_bytes=eb)
    assert dev_bytes(x) == oracle.ipt_c2r(vwords(host, eb), m, n).tobytes()
    ipt.r2c(x, m, n, elem_bytes=eb)
    assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()
    y = to_dev(host)
    ipt.r2c(y, m, n, elem_bytes=eb)
    assert dev_bytes(y) == oracle.ipt_r2c(vwords(host, eb), m, n).tobytes()


def test_fused_c2r_beyond_2gib():
    """Fused rotation + row pass (gcd 2) with the C2R engine on a matrix of > 2 GiB, alone and
    as a batch of two (matrix stride > 2^31 bytes: the wrap rows are copied by a kernel, not
    a pitched memcpy), compared in full."""
    m, n, eb = 30002, 18002, 4
    info = ipt.plan_info(m, n, eb)
    assert info["engine"] == "c2r" and info["c"] == 2 and info["launches"] == 2, info
    assert m * n * eb > (1 << 31)
    host = _fast_words(m * n, eb, seed=2)
    x = to_dev(host)
    ipt.c2r(x, m, n, elem_bytes=eb)
    assert dev_bytes(x) == oracle.transpose(host, m, n).tobytes()
    ipt.r2c(x, m, n, elem_bytes=eb)
    assert dev_bytes(x) == host.tobytes()
    del x
    m2, n2 = 24002, 12002  # gcd 2; 1.15 GB each, stride 1.15 GB * 1 + gap
    assert math.gcd(m2, n2) == 2
    stride = m2 * n2 + 16
    hb = _fast_words(2 * stride, eb, seed=3)
    x = to_dev(hb)
    ipt.c2r_batched(x, 2, stride, m2, n2, elem_bytes=eb)
    got = x.cpu().numpy().view(np.uint32)
    for k in range(2):
        o = k * stride
        assert got[o:o + m2 * n2].tobytes() == oracle.transpose(hb[o:o + m2 * n2], m2, n2).tobytes(), k
        assert got[o + m2 * n2:o + stride].tobytes() == hb[o + m2 * n2:o + stride].tobytes()
    ipt.r2c_batched(x, 2, stride, m2, n2, elem_bytes=eb)
    assert dev_bytes(x) == hb.tobytes()


@pytest.mark.timeout(600)
def test_fused_rotation_concurrent_with_busy_kernels():
    """The fused pass's cross-CTA waits must not assume co-residency: both fused directions
    (C2R staircases and R2C post-rotation, gcd 2..32) run on two streams while a third
    stream keeps the SMs busy with long GEMMs, so the fused kernels start with only part of
    their grid resident.  Work order by ticket guarantees progress (row_shuffle.cu
    row_rot_kernel); results compared in full."""
    shapes = [(6 * 1201, 6 * 1007, 4), (4 * 999, 4 * 1250, 8), (2 * 3001, 2 * 2203, 4), (30 * 137, 30 * 151, 4)]
    hosts = [_fast_words(m * n, eb, seed=i) for i, (m, n, eb) in enumerate(shapes)]
    xs = [to_dev(h) for h in hosts]
    a = torch.randn(8192, 8192, device=DEV, dtype=torch.bfloat16)
    torch.cuda.synchronize()
    busy, s1, s2 = torch.cuda.Stream(), torch.cuda.Stream(), torch.cuda.Stream()
    for rep in range(3):
        with torch.cuda.stream(busy):
            for _ in range(20):
                a = (a @ a).clamp_(-1, 1)
        for k, ((m, n, eb), x) in enumerate(zip(shapes, xs)):
            s = s1 if k % 2 == 0 else s2
            for engine in ("c2r", "r2c"):
                with forced_engine(engine), torch.cuda.stream(s):
                    ipt.c2r(x, m, n, elem_bytes=eb, stream=s)
                    ipt.r2c(x, m, n, elem_bytes=eb, stream=s)
        with torch.cuda.stream(s1):
            ipt.c2r(xs[0], *shapes[0][:2], elem_bytes=shapes[0][2], stream=s1)
            ipt.r2c(xs[0], *shapes[0][:2], elem_bytes=shapes[0][2], stream=s1)
    torch.cuda.synchronize()
    for (m, n, eb), x, h in zip(shapes, xs, hosts):
        assert dev_bytes(x) == h.tobytes(), (m, n, eb)
        with forced_engine("r2c"):
            ipt.c2r(x, m, n, elem_bytes=eb)
        assert dev_bytes(x) == oracle.transpose(vwords(h, eb), m, n).tobytes(), (m, n, eb)


def test_concurrent_calls_from_threads_share_no_counters():
    """ipt.h: thread-safe and reentrant.  Several host threads issue calls on their own
    streams and on cudaStreamPerThread-style shared handles at once; every call owns its
    counters (per-call scratch), so all results are exact."""
    import threading
    shapes = [(1811, 2903, 4), (4099, 1024, 8), (1200, 1800, 4), (3000, 4096, 4)]
    hosts = [_fast_words(m * n, eb, seed=50 + i) for i, (m, n, eb) in enumerate(shapes)]
    xs = [to_dev(h) for h in hosts]
    torch.cuda.synchronize()
    errors = []

    def work(k):
        try:
            m, n, eb = shapes[k]
            s = torch.cuda.Stream()
            with torch.cuda.stream(s):
                for _ in range(5):
                    ipt.c2r(xs[k], m, n, elem_bytes=eb, stream=s)
                    ipt.r2c(xs[k], m, n, elem_bytes=eb, stream=s)
                ipt.c2r(xs[k], m, n, elem_bytes=eb, stream=s)
            s.synchronize()
        except Exception as e:  # pragma: no cover
            errors.append(e)

    ts = [threading.Thread(target=work, args=(k,)) for k in range(len(shapes))]
    for t in ts:
        t.start()
    for t in ts:
        t.join()
    assert not errors, errors
    for (m, n, eb), x, h in zip(shapes, xs, hosts):
        assert dev_bytes(x) == oracle.transpose(vwords(h, eb), m, n).tobytes(), (m, n, eb)


@pytest.mark.parametrize("ck", ["0", "1", "16"])
def test_chunked_fused_pass_forced(ck):
    """Chunked fused rotation + row pass (row_chunk_kernel) forced on every fused shape
    (IPT_ROW_CHUNK=1), chunk length cK = max(R, IPT_ROW_CHUNK_K (c-1)) rows: 0 gives chunks of
    one row group, shorter than c - 1 (staircases and R2C blocks then span several chunks'
    boundary copies), 1 the minimum c - 1, 16 the default.  gcd 2..32, both engines, every
    element size, misaligned rows, lagged and unlagged column layouts, row groups, a gapped
    batch -- all compared in full with the oracle."""
    shapes = [(1200, 1816), (1816, 1200), (96, 40), (40, 96), (640, 32 * 33), (2 * 1009, 2 * 1013), (30 * 37, 30 * 41),
              (4 * 99, 4 * 25), (6 * 31, 6 * 77), (64, 48), (48, 64), (2 * 7, 2 * 5), (12, 18), (62, 64)]
    with env_var("IPT_ROW_CHUNK", "1"), env_var("IPT_ROW_CHUNK_K", ck):
        for lag in ("1", "0"):
            with env_var("IPT_COL_LAG", lag):
                for eb in (4, 8, 16):
                    for engine in ("c2r", "r2c"):
                        run_packed(shapes, eb, ipt.c2r, "row", engine, seed=eb * 11 + len(ck))
        with env_var("IPT_ROW_STAGE", "200000"):
            run_packed(shapes, 4, ipt.c2r, "row", None, seed=5)
        m, n, batch = 2 * 150, 2 * 501, 3
        host = workloads.random_words(1 + batch * (m * n + 7), 8, seed=91)
        hv = vwords(host, 8)
        x = to_dev(host)
        ipt.c2r_batched(x.data_ptr() + 8, batch, m * n + 7, m, n, elem_bytes=8)
        got = vwords(x.cpu().numpy(), 8)
        for k in range(batch):
            o = 1 + k * (m * n + 7)
            assert got[o:o + m * n].tobytes() == oracle.ipt_c2r(hv[o:o + m * n], m, n).tobytes()
        ipt.r2c_batched(x.data_ptr() + 8, batch, m * n + 7, m, n, elem_bytes=8)
        assert dev_bytes(x) == np.ascontiguousarray(host).tobytes()


def test_chunked_fused_pass_each_pass():
    """Per-pass parity of the chunked fused pass against the oracle's gather-form snapshots
    (C2R: [r_j + d'^{-1}] then p_j o q; R2C: q^{-1} o p^{-1} then [d' + r^{-1}])."""
    for (m, n) in [(1200, 1816), (1816, 1200), (6 * 301, 6 * 71)]:
        assert 1 < math.gcd(m, n) <= 32
        host = workloads.random_words(m * n, 4, seed=m ^ n)
        with env_var("IPT_ROW_CHUNK", "1"):
            for engine in ("c2r", "r2c"):
                with forced_engine(engine):
                    if engine == "c2r":
                        _, snaps = oracle.c2r_gather_forms(host, m, n, snapshots=True)
                    else:
                        _, snaps = oracle.r2c_gather_forms(host, n, m, snapshots=True)
                    for k, e in enumerate([snaps[1], snaps[3]], start=1):
                        x = to_dev(host)
                        with debug_passes(k):
                            ipt.c2r(x, m, n, elem_bytes=4)
                        assert dev_bytes(x) == e.tobytes(), (m, n, engine, k)


@pytest.mark.parametrize("pipe", ["0", "1"])
def test_row_pass_kernels_both(pipe):
    """The pipelined row pass (bulk-copy producer warp, default) and the previous kernel
    (IPT_ROW_PIPE=0) on gcd-1 and separate-rotation shapes: rows misaligned to 16 bytes, row
    groups, lagged side rows, single- and double-buffered rows, tiny rows (< 16 bytes)."""
    shapes = [(1031, 97), (97, 1031), (513, 700), (700, 513), (2003, 129), (129, 2003), (333, 4099), (5, 3), (3, 5),
              (7, 2), (2, 7), (3000, 17011)]
    with env_var("IPT_ROW_PIPE", pipe):
        for eb in (4, 8, 16):
            for engine in ("c2r", "r2c"):
                run_packed(shapes, eb, ipt.c2r, "row", engine, seed=eb + 3 * len(pipe))
        with env_var("IPT_FUSE_ROT", "0"):
            run_packed([(1200, 1800), (640, 32 * 33)], 4, ipt.c2r, "row", None, seed=8)


@pytest.mark.parametrize("sup", ["2", "3", "8"])
def test_super_tile_unit_order(sup):
    """Lagged column pass with units in band-major order inside super-tiles of S consecutive
    tiles (the default for tall tiles, e.g. config 5a; forced here on small shapes with many
    bands per tile via a small IPT_COL_SMEM): ragged last super-tiles, both engines, batches."""
    shapes = [(1200, 1800), (2003, 129), (129, 2003), (3001, 700), (700, 3001), (333, 4099)]
    with env_var("IPT_COL_SUPER", sup), env_var("IPT_COL_LAGD", "8"), env_var("IPT_COL_SMEM", "12000"):
        for eb in (4, 8):
            for engine in ("c2r", "r2c"):
                run_packed(shapes, eb, ipt.c2r, "row", engine, seed=eb + int(sup))
        m, n, batch = 300, 1001, 3
        host = workloads.random_words(batch * m * n, 4, seed=17)
        x = to_dev(host)
        ipt.c2r_batched(x, batch, m * n, m, n, elem_bytes=4)
        got = x.cpu().numpy().view(np.uint32)
        for k in range(batch):
            assert got[k * m * n:(k + 1) * m * n].tobytes() == oracle.transpose(host[k * m * n:(k + 1) * m * n], m, n).tobytes()


@pytest.mark.parametrize("mask", ["3", "7", "1", "0"])
def test_column_tma_staging(mask):
    """Column pass with TMA staging (IPT_COL_TMA mask: 1 box loads of the matrix, 2 of the
    lagged side block, 4 tile::gather4 for R2C): pitches that are multiples of 16 bytes (TMA)
    next to ones that are not (cp.async hulls), ragged rightmost tiles (zero-filled box columns),
    last bands (zero-filled box rows), units whose rows wrap past M - 1, batches packed and
    gapped, both engines, every element size; full comparison with the oracle."""
    shapes = [(1200, 1800), (1801, 1200), (1200, 1801), (640, 1024), (1024, 640), (2003, 132), (132, 2003),
              (4096, 3000), (300, 1004), (1004, 300), (96, 40), (37, 64)]
    with env_var("IPT_COL_TMA", mask):
        for eb in (4, 8, 16):
            for engine in ("c2r", "r2c"):
                with forced_engine(engine):
                    for (m, n) in shapes:  # own (256-byte-aligned) allocation per matrix: TMA-eligible
                        host = workloads.random_words(m * n, eb, seed=m * 7 + n + eb)
                        x = to_dev(host)
                        ipt.c2r(x, m, n, elem_bytes=eb)
                        assert dev_bytes(x) == oracle.transpose(vwords(host, eb), m, n).tobytes(), (m, n, eb, engine)
                        ipt.r2c(x, m, n, elem_bytes=eb)
                        assert dev_bytes(x) == np.ascontiguousarray(host).tobytes(), (m, n, eb, engine)
                run_packed(shapes, eb, ipt.c2r, "row", engine, seed=eb + int(mask))  # mostly unaligned bases
        for packed in (True, False):
            m, n, batch = 400, 1204, 3
            stride = m * n + (0 if packed else 4)
            host = workloads.random_words(batch * stride, 4, seed=23)
            x = to_dev(host)
            ipt.c2r_batched(x, batch, stride, m, n, elem_bytes=4)
            got = x.cpu().numpy().view(np.uint32)
            for k in range(batch):
                o = k * stride
                assert got[o:o + m * n].tobytes() == oracle.transpose(host[o:o + m * n], m, n).tobytes(), (packed, k)
            ipt.r2c_batched(x, batch, stride, m, n, elem_bytes=4)
            assert dev_bytes(x) == host.tobytes()


@pytest.mark.parametrize("eb", [4, 8])
@pytest.mark.timeout(1800)
def test_bench_sweep_calls_sampled_all(eb):
    """Every call bench.py times (workloads.sweep_shapes(200) x c2r/r2c, BASELINE configs[1]),
    in the launch configuration the bench uses. Shapes 0..47 are compared in full above; here
    all 200 run on the index pattern (element l holds l) and each output is checked
    (a) on 2^17 sampled destinations plus the first and last 4096, against the oracle's
        Eqs. 7-10 (oracle.source_many), and
    (b) in full by two properties that hold at any size: the result is a permutation of the
        input (sum and sum of squares of the words unchanged, int64 wrap-around) and r2c
        restores the input exactly."""
    shapes = workloads.sweep_shapes(200)
    dt = torch.int32 if eb == 4 else torch.int64
    maxel = max(m * n for m, n in shapes)
    rng = np.random.default_rng(eb)
    base = torch.arange(maxel, dtype=torch.int64, device=DEV)
    for k, (m, n) in enumerate(shapes):
        total = m * n
        x = base[:total].to(dt)
        s1 = x.to(torch.int64).sum().item()
        s2 = (x.to(torch.int64) * x.to(torch.int64)).sum().item()
        for op in ("c2r", "r2c"):
            if op == "r2c":
                x = base[:total].to(dt)
            pos = np.concatenate([np.arange(min(4096, total)), np.arange(max(0, total - 4096), total),
                                  rng.integers(0, total, size=1 << 17)]).astype(np.int64)
            getattr(ipt, op)(x, m, n, elem_bytes=eb)
            got = x[torch.from_numpy(pos).to(DEV)].to(torch.int64).cpu().numpy()
            want = oracle.source_many(op, m, n, pos)
            bad = np.nonzero(got != want)[0]
            assert bad.size == 0, (m, n, op, eb, int(pos[bad[0]]), int(got[bad[0]]), int(want[bad[0]]))
            x64 = x.to(torch.int64)
            assert x64.sum().item() == s1 and (x64 * x64).sum().item() == s2, (m, n, op, eb)
            getattr(ipt, "r2c" if op == "c2r" else "c2r")(x, m, n, elem_bytes=eb)
            assert torch.equal(x, base[:total].to(dt)), (m, n, op, eb, "round trip")


def test_host_buffer_calls_pipelined_on_two_streams():
    """ipt_c2r_host / ipt_r2c_host (include/ipt.h): pinned host matrix -> device -> transpose
    -> host, stream-ordered; consecutive calls alternate two streams and two device buffers
    (the bench's e2e pattern), every result compared in full with the oracle; invalid
    arguments leave the host buffer untouched."""
    shapes = [(1200, 1800, 4), (333, 4099, 8), (2003, 129, 4), (640, 1024, 16), (4096, 3000, 4), (17, 5, 8)]
    streams = [torch.cuda.Stream(), torch.cuda.Stream()]
    devs = [torch.empty(max(m * n * eb for m, n, eb in shapes), dtype=torch.uint8, device=DEV) for _ in range(2)]
    hosts, wants = [], []
    for k, (m, n, eb) in enumerate(shapes):
        host = workloads.random_words(m * n, eb, seed=k + 40)
        h = torch.from_numpy(np.ascontiguousarray(host).view(np.uint8).reshape(-1).copy()).pin_memory()
        hosts.append(h)
        wants.append(oracle.transpose(vwords(host, eb), m, n).tobytes())
        ipt.c2r_host(h, devs[k % 2], m, n, elem_bytes=eb, stream=streams[k % 2])
    torch.cuda.synchronize()
    for k, (m, n, eb) in enumerate(shapes):
        assert hosts[k].numpy().tobytes() == wants[k], (m, n, eb)
        ipt.r2c_host(hosts[k], devs[k % 2], m, n, elem_bytes=eb, stream=streams[k % 2])
    torch.cuda.synchronize()
    for k, (m, n, eb) in enumerate(shapes):
        host = workloads.random_words(m * n, eb, seed=k + 40)
        assert hosts[k].numpy().tobytes() == np.ascontiguousarray(host).tobytes(), (m, n, eb)
    h = hosts[0].clone()
    with pytest.raises(ipt.IptError) as e:
        ipt.c2r_host(h, 0, 1200, 1800, elem_bytes=4)
    assert e.value.status == 1 and torch.equal(h, hosts[0])
