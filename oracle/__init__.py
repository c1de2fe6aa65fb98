"""CPU oracle for the decomposed in-place transpose.  TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` leg may import this package.  The product package
(``paper_conf_ppopp_catanzarokg14_b200``) never imports it, and it imports nothing from
the product: the two share no code, header, table or constant generator.

The arithmetic lives in ``oracle/ipt_oracle.c`` (plain C, 64-bit, literal loops in the
paper's order, every function citing PAPER.md); this module only marshals numpy buffers
to it via ctypes, plus the export-level semantics of the C ABI (which permutation each
``ipt_*`` call must realise; SURVEY.md §8.c.1 / DESIGN.md readings C11, C18), written
from Theorems 1-2 as calls to the plain transpose.

Parity status: every function here is pinned (tests/test_oracle.py): Fig. 1 and Fig. 2
fixtures (tests/golden/), numpy's out-of-place transpose, Theorems 3/6/7, inverse pairs
of the §4 gather forms, brute force over all small shapes.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_SRC = os.path.join(_HERE, "ipt_oracle.c")
_LIB = os.path.join(_HERE, "libipt_oracle.so")

_i64 = ctypes.c_int64
_vp = ctypes.c_void_p


def build(force: bool = False) -> str:
    """Compile the C oracle with gcc (plain -O2, no OpenMP: the oracle as it stands)."""
    if force or not os.path.exists(_LIB) or os.path.getmtime(_LIB) < os.path.getmtime(_SRC):
        tmp = _LIB + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", "-O2", "-std=c11", "-Wall", "-shared", "-fPIC", _SRC, "-o", tmp])
        os.replace(tmp, _LIB)
    return _LIB


_lib = None


def lib() -> ctypes.CDLL:
    global _lib
    if _lib is None:
        L = ctypes.CDLL(build())
        for name in ("oracle_mmi", "oracle_gcd"):
            getattr(L, name).restype = _i64
            getattr(L, name).argtypes = [_i64, _i64]
        for name in ("oracle_eq22_d", "oracle_eq23_r", "oracle_eq24_dp", "oracle_eq26_sp",
                     "oracle_eq31_dpinv", "oracle_eq32_p", "oracle_eq35_pinv", "oracle_eq36_rinv"):
            getattr(L, name).restype = _i64
            getattr(L, name).argtypes = [_i64, _i64, _i64, _i64]
        for name in ("oracle_eq33_q", "oracle_eq34_qinv"):
            getattr(L, name).restype = _i64
            getattr(L, name).argtypes = [_i64, _i64, _i64]
        for name in ("oracle_c2r_source", "oracle_r2c_source"):
            getattr(L, name).restype = None
            getattr(L, name).argtypes = [_i64, _i64, _i64, _i64, ctypes.POINTER(_i64), ctypes.POINTER(_i64)]
        L.oracle_source_many.restype = None
        L.oracle_source_many.argtypes = [_i64, _i64, ctypes.c_int, _vp, _i64, _vp]
        for name in ("oracle_c2r_definition", "oracle_r2c_definition", "oracle_transpose"):
            getattr(L, name).restype = None
            getattr(L, name).argtypes = [_vp, _vp, _i64, _i64, ctypes.c_int]
        for name in ("oracle_c2r_alg1", "oracle_r2c_alg1"):
            getattr(L, name).restype = ctypes.c_int
            getattr(L, name).argtypes = [_vp, _i64, _i64, ctypes.c_int, ctypes.c_int, _vp, _vp, _vp, _vp]
        for name in ("oracle_aos_gather", "oracle_aos_scatter"):
            getattr(L, name).restype = None
            getattr(L, name).argtypes = [_vp, _vp, _vp, _i64, ctypes.c_int]
        for name in ("oracle_c2r_gather_forms", "oracle_r2c_gather_forms"):
            getattr(L, name).restype = ctypes.c_int
            getattr(L, name).argtypes = [_vp, _i64, _i64, ctypes.c_int, _vp, _vp, _vp, _vp]
        _lib = L
    return _lib


def _ptr(a: np.ndarray | None):
    return None if a is None else a.ctypes.data_as(_vp)


def _flat(a: np.ndarray) -> np.ndarray:
    a = np.ascontiguousarray(a).reshape(-1)
    return a


# ----------------------------------------------------------------------------------------
# Scalar index functions (Eqs. 22-36)
# ----------------------------------------------------------------------------------------
def gcd(x: int, y: int) -> int:
    return int(lib().oracle_gcd(x, y))


def mmi(x: int, y: int) -> int:
    """Modular multiplicative inverse; mmi(x, 1) = 0 (reading C4)."""
    return int(lib().oracle_mmi(x, y))


def c2r_source(m, n, i, j):
    """Eqs. 7-8: (s(i,j), c(i,j))."""
    a, b = _i64(), _i64()
    lib().oracle_c2r_source(m, n, i, j, ctypes.byref(a), ctypes.byref(b))
    return int(a.value), int(b.value)


def r2c_source(m, n, i, j):
    """Eqs. 9-10: (t(i,j), d(i,j))."""
    a, b = _i64(), _i64()
    lib().oracle_r2c_source(m, n, i, j, ctypes.byref(a), ctypes.byref(b))
    return int(a.value), int(b.value)


def source_many(op: str, m: int, n: int, pos: np.ndarray) -> np.ndarray:
    """Eqs. 7-10 vectorised: for linear destinations pos (i*n + j of the m x n array) the
    linear source offsets of C2R (op="c2r", Eq. 11) or R2C (op="r2c", Eq. 12)."""
    pos = np.ascontiguousarray(pos, dtype=np.int64)
    out = np.empty_like(pos)
    lib().oracle_source_many(m, n, 1 if op == "r2c" else 0, _ptr(pos), pos.size, _ptr(out))
    return out


def eq22_d(m, n, i, j): return int(lib().oracle_eq22_d(m, n, i, j))
def eq23_r(m, n, i, j): return int(lib().oracle_eq23_r(m, n, i, j))
def eq24_dp(m, n, i, j): return int(lib().oracle_eq24_dp(m, n, i, j))
def eq26_sp(m, n, i, j): return int(lib().oracle_eq26_sp(m, n, i, j))
def eq31_dpinv(m, n, i, j): return int(lib().oracle_eq31_dpinv(m, n, i, j))
def eq32_p(m, n, i, j): return int(lib().oracle_eq32_p(m, n, i, j))
def eq33_q(m, n, i): return int(lib().oracle_eq33_q(m, n, i))
def eq34_qinv(m, n, i): return int(lib().oracle_eq34_qinv(m, n, i))
def eq35_pinv(m, n, i, j): return int(lib().oracle_eq35_pinv(m, n, i, j))
def eq36_rinv(m, n, i, j): return int(lib().oracle_eq36_rinv(m, n, i, j))


# ----------------------------------------------------------------------------------------
# Whole-array operations.  Arrays are flat numpy buffers of any dtype (opaque words of
# itemsize bytes); results are new arrays, inputs are never modified.
# ----------------------------------------------------------------------------------------
def transpose(X: np.ndarray, x: int, y: int) -> np.ndarray:
    """Theorem 1 buffer form: row-major x-by-y X -> row-major y-by-x Y, Y[j x + i] = X[i y + j]."""
    X = _flat(X)
    assert X.size == x * y
    Y = np.empty_like(X)
    lib().oracle_transpose(_ptr(X), _ptr(Y), x, y, X.itemsize)
    return Y


def c2r_definition(A: np.ndarray, m: int, n: int) -> np.ndarray:
    """Eq. 11 (out of place gather) on an m x n row-major buffer."""
    A = _flat(A)
    assert A.size == m * n
    B = np.empty_like(A)
    lib().oracle_c2r_definition(_ptr(A), _ptr(B), m, n, A.itemsize)
    return B


def r2c_definition(A: np.ndarray, m: int, n: int) -> np.ndarray:
    """Eq. 12 (out of place gather) on an m x n row-major buffer."""
    A = _flat(A)
    assert A.size == m * n
    B = np.empty_like(A)
    lib().oracle_r2c_definition(_ptr(A), _ptr(B), m, n, A.itemsize)
    return B


def _run_steps(fn, A, m, n, nsnap, snapshots, extra):
    A = _flat(A).copy()
    assert A.size == m * n
    snaps = [np.full_like(A, 0) for _ in range(nsnap)] if snapshots else [None] * nsnap
    rc = fn(_ptr(A), m, n, A.itemsize, *extra, *[_ptr(s) for s in snaps])
    if rc != 0:
        raise MemoryError("oracle allocation failed")
    return A, snaps


def c2r_alg1(A: np.ndarray, m: int, n: int, snapshots: bool = False, counts: bool = False,
             linearization: str = "row"):
    """Algorithm 1 in place on a copy of A.

    Returns the result; with ``snapshots`` also the array after each of the three outer
    loops (the first is None when gcd(m,n) == 1); with ``counts`` also
    (A reads, A writes, tmp reads, tmp writes)."""
    cnt = np.zeros(4, dtype=np.int64) if counts else None
    lin = {"row": 0, "col": 1}[linearization]
    out, snaps = _run_steps(lambda p, mm, nn, eb, lin_, s0, s1, s2: lib().oracle_c2r_alg1(
        p, mm, nn, eb, lin_, s0, s1, s2, _ptr(cnt)), A, m, n, 3, snapshots, (lin,))
    if snapshots and gcd(m, n) == 1:
        snaps[0] = None
    res = [out]
    if snapshots:
        res.append(snaps)
    if counts:
        res.append(tuple(int(v) for v in cnt))
    return res[0] if len(res) == 1 else tuple(res)


def r2c_alg1(A: np.ndarray, m: int, n: int, snapshots: bool = False, counts: bool = False,
             linearization: str = "row"):
    """Inverse of Algorithm 1 for an m x n C2R, in place on a copy of A."""
    cnt = np.zeros(4, dtype=np.int64) if counts else None
    lin = {"row": 0, "col": 1}[linearization]
    out, snaps = _run_steps(lambda p, mm, nn, eb, lin_, s0, s1, s2: lib().oracle_r2c_alg1(
        p, mm, nn, eb, lin_, s0, s1, s2, _ptr(cnt)), A, m, n, 3, snapshots, (lin,))
    if snapshots and gcd(m, n) == 1:
        snaps[2] = None
    res = [out]
    if snapshots:
        res.append(snaps)
    if counts:
        res.append(tuple(int(v) for v in cnt))
    return res[0] if len(res) == 1 else tuple(res)


def c2r_gather_forms(A: np.ndarray, m: int, n: int, snapshots: bool = False):
    """§4.2 all-gather C2R: [r_j] -> d'^{-1}_i -> p_j -> q (Eqs. 23, 31, 32, 33)."""
    out, snaps = _run_steps(lib().oracle_c2r_gather_forms, A, m, n, 4, snapshots, ())
    if snapshots and gcd(m, n) == 1:
        snaps[0] = None
    return (out, snaps) if snapshots else out


def r2c_gather_forms(A: np.ndarray, m: int, n: int, snapshots: bool = False):
    """§4.3 all-gather R2C: q^{-1} -> p^{-1}_j -> d'_i -> [r^{-1}_j] (Eqs. 34, 35, 24, 36)."""
    out, snaps = _run_steps(lib().oracle_r2c_gather_forms, A, m, n, 4, snapshots, ())
    if snapshots and gcd(m, n) == 1:
        snaps[3] = None
    return (out, snaps) if snapshots else out


# ----------------------------------------------------------------------------------------
# Export-level semantics of the C ABI (include/ipt.h), from Theorems 1-2
# and reading C18: ``layout`` says how the m x n input is stored; c2r produces its n x m
# transpose in the same layout; r2c with the same arguments is the exact inverse.
# ----------------------------------------------------------------------------------------
ROW_MAJOR, COL_MAJOR = 0, 1


def export_permutation(op: str, m: int, n: int, layout: int):
    """(x, y) such that the export equals 'transpose the row-major x-by-y buffer'."""
    if op == "c2r":
        return (m, n) if layout == ROW_MAJOR else (n, m)
    if op == "r2c":
        return (n, m) if layout == ROW_MAJOR else (m, n)
    raise ValueError(op)


def ipt_c2r(X: np.ndarray, m: int, n: int, layout: int = ROW_MAJOR) -> np.ndarray:
    x, y = export_permutation("c2r", m, n, layout)
    return transpose(X, x, y)


def ipt_r2c(X: np.ndarray, m: int, n: int, layout: int = ROW_MAJOR) -> np.ndarray:
    x, y = export_permutation("r2c", m, n, layout)
    return transpose(X, x, y)


def aos_to_soa(X: np.ndarray, count: int, fields: int) -> np.ndarray:
    """§6.1: an AoS of `count` structs of `fields` fields is a row-major
    count x fields array; its transpose is the SoA layout."""
    return transpose(X, count, fields)


def soa_to_aos(X: np.ndarray, count: int, fields: int) -> np.ndarray:
    return transpose(X, fields, count)


def warp_load_aos_registers(words: np.ndarray, S: int, lanes: int = 32) -> np.ndarray:
    """§6.2, reading C16: after a warp-cooperative load of `lanes`
    consecutive S-word structs, lane l's register k holds word l*S + k of the chunk.
    Returned as an array R[k, l] (register index major)."""
    w = _flat(words)
    assert w.size == S * lanes
    R = np.empty((S, lanes), dtype=w.dtype)
    for lane in range(lanes):
        for k in range(S):
            R[k, lane] = w[lane * S + k]
    return R


def aos_gather(src: np.ndarray, idx: np.ndarray, words: int) -> np.ndarray:
    """§6.2 random-access gather (Fig. 9; reading C17): dst[k] =
    src[idx[k]] struct by struct (structs of `words` 4-byte words).  Plain loops in C."""
    src = np.ascontiguousarray(src, dtype=np.uint32).reshape(-1)
    idx = np.ascontiguousarray(idx, dtype=np.uint32).reshape(-1)
    assert src.size % words == 0 and (idx.size == 0 or int(idx.max()) < src.size // words)
    dst = np.empty(idx.size * words, dtype=np.uint32)
    lib().oracle_aos_gather(_ptr(src), _ptr(idx), _ptr(dst), idx.size, words)
    return dst


def aos_scatter(src: np.ndarray, idx: np.ndarray, words: int, ndst: int | None = None) -> np.ndarray:
    """§6.2 random-access scatter: dst[idx[k]] = src[k] (idx a permutation of the
    destination structs; destinations not named by idx stay zero)."""
    src = np.ascontiguousarray(src, dtype=np.uint32).reshape(-1)
    idx = np.ascontiguousarray(idx, dtype=np.uint32).reshape(-1)
    count = idx.size
    assert src.size >= count * words
    ndst = count if ndst is None else ndst
    assert count == 0 or int(idx.max()) < ndst
    dst = np.zeros(ndst * words, dtype=np.uint32)
    lib().oracle_aos_scatter(_ptr(src), _ptr(idx), _ptr(dst), count, words)
    return dst
