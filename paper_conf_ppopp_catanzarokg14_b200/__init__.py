"""B200-native decomposed in-place transpose (Catanzaro, Keller, Garland, PPoPP'14).

Thin Python binding of the C ABI in include/ipt.h: argument marshalling only.  Every
step of the transpose runs in the CUDA kernels of libipt.so (built in-tree for sm_100a
by __graft_entry__.build()).  There is no CPU fallback: importing this package without
the built library raises.

Buffers are torch CUDA tensors (any dtype; elem_bytes defaults to the element size, so
complex128 carries 16-byte elements) or raw device pointers (int).  Calls are
asynchronous on the given stream (default: torch's current stream of the tensor's
device).
"""
from __future__ import annotations

import ctypes
import os

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "libipt.so")

ROW_MAJOR = 0
COL_MAJOR = 1
_LAYOUTS = {"row": ROW_MAJOR, "col": COL_MAJOR, ROW_MAJOR: ROW_MAJOR, COL_MAJOR: COL_MAJOR}

STATUS = {0: "IPT_OK", 1: "IPT_ERR_INVALID_ARGUMENT", 2: "IPT_ERR_UNSUPPORTED",
          3: "IPT_ERR_OUT_OF_MEMORY", 4: "IPT_ERR_CUDA"}

# Every symbol declared in include/ipt.h.
EXPORTS = ("ipt_c2r", "ipt_r2c", "ipt_c2r_batched", "ipt_r2c_batched", "ipt_c2r_host", "ipt_r2c_host", "ipt_aos_to_soa",
           "ipt_soa_to_aos", "ipt_scratch_bytes", "ipt_status_string", "ipt_plan_info",
           "ipt_launch_count", "ipt_profile_enable", "ipt_profile_read", "ipt_debug_tile_copy",
           "ipt_debug_aos_copy", "ipt_debug_aos_fill", "ipt_debug_warp_load_dump", "ipt_debug_warp_store",
           "ipt_debug_aos_gather", "ipt_debug_aos_scatter")
AOS_DIRECT, AOS_VECTOR, AOS_COALESCED = 0, 1, 2
PROFILE_KINDS = 8
KERNEL_KINDS = ("row_shuffle", "col_shuffle", "col_rotate", "skinny")


class IptError(RuntimeError):
    def __init__(self, status: int, where: str):
        super().__init__(f"{where}: {STATUS.get(status, status)}")
        self.status = status


if not os.path.exists(LIB_PATH):
    raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() (nvcc, sm_100a). "
                      "There is no CPU fallback.")

_lib = ctypes.CDLL(LIB_PATH)
_i64, _int, _vp = ctypes.c_int64, ctypes.c_int, ctypes.c_void_p
_lib.ipt_c2r.argtypes = [_vp, _i64, _i64, _int, _int, _vp]
_lib.ipt_r2c.argtypes = [_vp, _i64, _i64, _int, _int, _vp]
_lib.ipt_c2r_batched.argtypes = [_vp, _i64, _i64, _i64, _i64, _int, _int, _vp]
_lib.ipt_r2c_batched.argtypes = [_vp, _i64, _i64, _i64, _i64, _int, _int, _vp]
_lib.ipt_c2r_host.argtypes = [_vp, _vp, _i64, _i64, _int, _int, _vp]
_lib.ipt_r2c_host.argtypes = [_vp, _vp, _i64, _i64, _int, _int, _vp]
_lib.ipt_aos_to_soa.argtypes = [_vp, _i64, _i64, _int, _vp]
_lib.ipt_soa_to_aos.argtypes = [_vp, _i64, _i64, _int, _vp]
_lib.ipt_scratch_bytes.argtypes = [_i64, _i64, _int, ctypes.POINTER(ctypes.c_size_t), ctypes.POINTER(ctypes.c_size_t)]
_lib.ipt_status_string.argtypes = [_int]
_lib.ipt_status_string.restype = ctypes.c_char_p
_lib.ipt_plan_info.argtypes = [_i64, _i64, _int, _int, ctypes.POINTER(_i64)]
_lib.ipt_launch_count.argtypes = []
_lib.ipt_launch_count.restype = ctypes.c_uint64
_lib.ipt_profile_enable.argtypes = [_int]
_lib.ipt_profile_enable.restype = None
_lib.ipt_profile_read.argtypes = [ctypes.POINTER(_i64), ctypes.POINTER(ctypes.c_double),
                                  ctypes.POINTER(ctypes.c_double)]
_lib.ipt_profile_read.restype = _i64
_lib.ipt_debug_tile_copy.argtypes = [_vp, _i64, _i64, _int, _int, _int, _int, _vp]
_lib.ipt_debug_tile_copy.restype = _int
_lib.ipt_debug_aos_copy.argtypes = [_vp, _vp, _i64, _int, _int, _vp]
_lib.ipt_debug_aos_fill.argtypes = [_vp, _i64, _int, _int, _vp]
_lib.ipt_debug_warp_load_dump.argtypes = [_vp, _vp, _i64, _int, _vp]
_lib.ipt_debug_warp_store.argtypes = [_vp, _vp, _i64, _int, _vp]
_lib.ipt_debug_aos_gather.argtypes = [_vp, _vp, _vp, _i64, _int, _int, _vp]
_lib.ipt_debug_aos_scatter.argtypes = [_vp, _vp, _vp, _i64, _int, _int, _vp]
for _f in ("ipt_debug_aos_copy", "ipt_debug_aos_fill", "ipt_debug_warp_load_dump", "ipt_debug_warp_store",
           "ipt_debug_aos_gather", "ipt_debug_aos_scatter"):
    getattr(_lib, _f).restype = _int
for _f in ("ipt_c2r", "ipt_r2c", "ipt_c2r_batched", "ipt_r2c_batched", "ipt_c2r_host", "ipt_r2c_host", "ipt_aos_to_soa",
           "ipt_soa_to_aos", "ipt_scratch_bytes", "ipt_plan_info"):
    getattr(_lib, _f).restype = _int


def library() -> ctypes.CDLL:
    return _lib


def _ptr_eb_stream(buf, elem_bytes, stream):
    """(device pointer, element bytes, stream handle) of a tensor or raw pointer."""
    if isinstance(buf, int):
        if elem_bytes is None:
            raise ValueError("elem_bytes is required with a raw pointer")
        ptr, eb, dev = buf, elem_bytes, None
    else:
        if not buf.is_cuda:
            raise ValueError("buffer must be a CUDA tensor (no CPU fallback)")
        if not buf.is_contiguous():
            raise ValueError("buffer must be contiguous")
        ptr, dev = buf.data_ptr(), buf.device
        eb = elem_bytes if elem_bytes is not None else buf.element_size()
    if stream is None:
        import torch
        stream = torch.cuda.current_stream(dev).cuda_stream
    elif not isinstance(stream, int):
        stream = stream.cuda_stream
    return ptr, eb, stream


def _check(status: int, where: str):
    if status != 0:
        raise IptError(status, where)


def c2r(buf, m: int, n: int, elem_bytes: int | None = None, layout="row", stream=None):
    """In place: the m x n matrix in `layout` becomes its n x m transpose (same layout)."""
    p, eb, st = _ptr_eb_stream(buf, elem_bytes, stream)
    _check(_lib.ipt_c2r(p, m, n, eb, _LAYOUTS[layout], st), "ipt_c2r")
    return buf


def r2c(buf, m: int, n: int, elem_bytes: int | None = None, layout="row", stream=None):
    """Exact inverse of c2r with the same arguments."""
    p, eb, st = _ptr_eb_stream(buf, elem_bytes, stream)
    _check(_lib.ipt_r2c(p, m, n, eb, _LAYOUTS[layout], st), "ipt_r2c")
    return buf


def c2r_batched(buf, batch: int, stride_elems: int, m: int, n: int, elem_bytes: int | None = None,
                layout="row", stream=None):
    p, eb, st = _ptr_eb_stream(buf, elem_bytes, stream)
    _check(_lib.ipt_c2r_batched(p, batch, stride_elems, m, n, eb, _LAYOUTS[layout], st), "ipt_c2r_batched")
    return buf


def r2c_batched(buf, batch: int, stride_elems: int, m: int, n: int, elem_bytes: int | None = None,
                layout="row", stream=None):
    p, eb, st = _ptr_eb_stream(buf, elem_bytes, stream)
    _check(_lib.ipt_r2c_batched(p, batch, stride_elems, m, n, eb, _LAYOUTS[layout], st), "ipt_r2c_batched")
    return buf


def _host_ptr(host):
    if isinstance(host, int):
        return host
    if host.is_cuda or not host.is_contiguous():
        raise ValueError("host buffer must be a contiguous CPU tensor (pinned for asynchronous copies)")
    return host.data_ptr()


def c2r_host(host, dev, m: int, n: int, elem_bytes: int | None = None, layout="row", stream=None):
    """ipt_c2r_host: host -> dev, c2r on dev, dev -> host, stream-ordered (include/ipt.h)."""
    p, eb, st = _ptr_eb_stream(dev, elem_bytes if elem_bytes is not None else
                               (None if isinstance(host, int) else host.element_size()), stream)
    _check(_lib.ipt_c2r_host(_host_ptr(host), p, m, n, eb, _LAYOUTS[layout], st), "ipt_c2r_host")
    return host


def r2c_host(host, dev, m: int, n: int, elem_bytes: int | None = None, layout="row", stream=None):
    """ipt_r2c_host: the inverse of c2r_host with the same arguments."""
    p, eb, st = _ptr_eb_stream(dev, elem_bytes if elem_bytes is not None else
                               (None if isinstance(host, int) else host.element_size()), stream)
    _check(_lib.ipt_r2c_host(_host_ptr(host), p, m, n, eb, _LAYOUTS[layout], st), "ipt_r2c_host")
    return host


def aos_to_soa(buf, count: int, fields: int, field_bytes: int | None = None, stream=None):
    p, eb, st = _ptr_eb_stream(buf, field_bytes, stream)
    _check(_lib.ipt_aos_to_soa(p, count, fields, eb, st), "ipt_aos_to_soa")
    return buf


def soa_to_aos(buf, count: int, fields: int, field_bytes: int | None = None, stream=None):
    p, eb, st = _ptr_eb_stream(buf, field_bytes, stream)
    _check(_lib.ipt_soa_to_aos(p, count, fields, eb, st), "ipt_soa_to_aos")
    return buf


def scratch_bytes(m: int, n: int, elem_bytes: int):
    g, o = ctypes.c_size_t(), ctypes.c_size_t()
    _check(_lib.ipt_scratch_bytes(m, n, elem_bytes, ctypes.byref(g), ctypes.byref(o)), "ipt_scratch_bytes")
    return int(g.value), int(o.value)


def plan_info(m: int, n: int, elem_bytes: int, layout="row"):
    out = (_i64 * 10)()
    _check(_lib.ipt_plan_info(m, n, elem_bytes, _LAYOUTS[layout], out), "ipt_plan_info")
    keys = ("engine", "M", "N", "c", "launches", "cluster", "tile_w", "onchip_bytes", "row_cluster",
            "scratch_bytes")
    d = dict(zip(keys, (int(v) for v in out)))
    d["engine"] = {0: "none", 1: "c2r", 2: "r2c", 3: "skinny"}[d["engine"]]
    return d


def launch_count() -> int:
    return int(_lib.ipt_launch_count())


def profile_enable(on: bool = True) -> None:
    """Bracket every launch with CUDA events on its stream (see ipt_profile_read)."""
    _lib.ipt_profile_enable(1 if on else 0)


def profile_read():
    """{kind: (launches, device ms, algorithmic bytes)} since the last read."""
    n = (_i64 * PROFILE_KINDS)()
    ms = (ctypes.c_double * PROFILE_KINDS)()
    by = (ctypes.c_double * PROFILE_KINDS)()
    if _lib.ipt_profile_read(n, ms, by) < 0:
        raise IptError(4, "ipt_profile_read")
    return {KERNEL_KINDS[k]: (int(n[k]), float(ms[k]), float(by[k]))
            for k in range(len(KERNEL_KINDS)) if n[k]}


def debug_tile_copy(buf, M: int, N: int, elem_bytes: int, tile_bytes: int, cluster: int, barrier: bool,
                    stream=None):
    """Identity pass of the column-tile kernel (include/ipt_debug.h): measurement only."""
    p, eb, st = _ptr_eb_stream(buf, elem_bytes, stream)
    _check(_lib.ipt_debug_tile_copy(p, M, N, eb, tile_bytes, cluster, 1 if barrier else 0, st),
           "ipt_debug_tile_copy")
    return buf


def _dev_stream(t, stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream(t.device).cuda_stream
    return stream if isinstance(stream, int) else stream.cuda_stream


def aos_copy(src, dst, count: int, words: int, variant: int, stream=None):
    """Consumer kernel dst[k] = src[k] over `count` structs of `words` 4-byte words
    (variant AOS_DIRECT / AOS_VECTOR / AOS_COALESCED; include/ipt_debug.h)."""
    _check(_lib.ipt_debug_aos_copy(src.data_ptr(), dst.data_ptr(), count, words, variant,
                                   _dev_stream(dst, stream)), "ipt_debug_aos_copy")


def aos_fill(dst, count: int, words: int, variant: int, stream=None):
    _check(_lib.ipt_debug_aos_fill(dst.data_ptr(), count, words, variant, _dev_stream(dst, stream)),
           "ipt_debug_aos_fill")


def aos_gather(src, idx, dst, count: int, words: int, variant: int, stream=None):
    """Random-access consumer dst[k] = src[idx[k]] (include/ipt_debug.h)."""
    _check(_lib.ipt_debug_aos_gather(src.data_ptr(), idx.data_ptr(), dst.data_ptr(), count, words, variant,
                                     _dev_stream(dst, stream)), "ipt_debug_aos_gather")


def aos_scatter(src, idx, dst, count: int, words: int, variant: int, stream=None):
    """Random-access consumer dst[idx[k]] = src[k] (idx a permutation)."""
    _check(_lib.ipt_debug_aos_scatter(src.data_ptr(), idx.data_ptr(), dst.data_ptr(), count, words, variant,
                                      _dev_stream(dst, stream)), "ipt_debug_aos_scatter")


def warp_load_dump(src, dump, nchunks: int, words: int, stream=None):
    _check(_lib.ipt_debug_warp_load_dump(src.data_ptr(), dump.data_ptr(), nchunks, words,
                                         _dev_stream(dump, stream)), "ipt_debug_warp_load_dump")


def warp_store(regs, dst, nchunks: int, words: int, stream=None):
    _check(_lib.ipt_debug_warp_store(regs.data_ptr(), dst.data_ptr(), nchunks, words, _dev_stream(dst, stream)),
           "ipt_debug_warp_store")


def status_string(s: int) -> str:
    return _lib.ipt_status_string(s).decode()
