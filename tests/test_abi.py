"""C-ABI library checks that need no GPU: it loads, exports every symbol include/*.h
declares, and rejects bad arguments before touching the device."""
import ctypes
import os
import re

import pytest

from conftest import ROOT

INCLUDE = os.path.join(ROOT, "include")


def declared_symbols():
    syms = set()
    for f in os.listdir(INCLUDE):
        if f.endswith(".h"):
            text = re.sub(r"/\*.*?\*/", "", open(os.path.join(INCLUDE, f)).read(), flags=re.S)
            syms |= set(re.findall(r"\b(ipt_[a-z0-9_]+)\s*\(", text))
    return sorted(syms)


@pytest.fixture(scope="module")
def ipt():
    from paper_conf_ppopp_catanzarokg14_b200 import _build
    _build.build()
    import paper_conf_ppopp_catanzarokg14_b200 as mod
    return mod


def test_header_declares_the_north_star_entry_points():
    syms = declared_symbols()
    for s in ("ipt_c2r", "ipt_r2c", "ipt_c2r_batched", "ipt_r2c_batched", "ipt_aos_to_soa",
              "ipt_soa_to_aos", "ipt_scratch_bytes", "ipt_status_string"):
        assert s in syms


def test_library_exports_every_declared_symbol(ipt):
    lib = ipt.library()
    for s in declared_symbols():
        assert hasattr(lib, s), s
    assert set(declared_symbols()) == set(ipt.EXPORTS)


def test_device_code_is_sm100a(ipt):
    import subprocess
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", ipt.LIB_PATH],
                         capture_output=True, text=True).stdout
    assert "sm_100a" in out


def test_status_strings(ipt):
    for code, name in ipt.STATUS.items():
        assert ipt.status_string(code) == name


def test_argument_validation_without_device(ipt):
    lib = ipt.library()
    fake = 1 << 20  # never dereferenced: validation fails (or the call is a no-op) first
    assert lib.ipt_c2r(fake, 4, 6, 3, 0, None) == 1          # elem_bytes not in {4,8,16}
    assert lib.ipt_c2r(fake, 4, 6, 4, 7, None) == 1          # bad layout
    assert lib.ipt_c2r(fake, -1, 6, 4, 0, None) == 1         # negative dimension
    assert lib.ipt_c2r(None, 4, 6, 4, 0, None) == 1          # NULL with m*n > 0
    assert lib.ipt_c2r(fake + 2, 4, 6, 4, 0, None) == 1      # misaligned to elem_bytes
    assert lib.ipt_c2r(fake, 1 << 40, 1 << 40, 8, 0, None) == 1  # size overflow
    assert lib.ipt_c2r_batched(fake, 2, 10, 4, 6, 4, 0, None) == 1  # stride < m*n
    # sub-word elements: 4-byte aligned base, one side a multiple of 4 / elem_bytes
    assert lib.ipt_c2r(fake + 2, 4, 6, 2, 0, None) == 1      # misaligned to 4
    assert lib.ipt_c2r(fake, 3, 5, 2, 0, None) == 2          # both sides odd: unsupported
    assert lib.ipt_c2r(fake, 6, 10, 1, 0, None) == 2         # neither side a multiple of 4
    assert lib.ipt_c2r_batched(fake, 2, 25, 4, 6, 2, 0, None) == 2  # stride not whole words
    # multi-word records: any multiple of 4 up to 4096, 4-byte aligned base
    assert lib.ipt_c2r(fake, 4, 6, 6, 0, None) == 1          # not a multiple of 4
    assert lib.ipt_c2r(fake, 4, 6, 4100, 0, None) == 1       # beyond 4096
    assert lib.ipt_c2r(fake + 2, 4, 6, 12, 0, None) == 1     # misaligned to 4
    assert lib.ipt_c2r(fake + 4, 1, 6, 12, 0, None) == 0     # identity, 4-byte alignment enough
    assert lib.ipt_c2r(fake, 1 << 40, 1 << 40, 24, 0, None) == 1  # size overflow
    assert lib.ipt_c2r_batched(fake, 2, 10, 4, 6, 32, 0, None) == 1  # stride < m*n
    # identities: nothing is enqueued, no device needed
    assert lib.ipt_c2r(fake, 1, 1000, 4, 0, None) == 0
    assert lib.ipt_r2c(fake, 1000, 1, 8, 1, None) == 0
    assert lib.ipt_c2r(None, 0, 5, 4, 0, None) == 0
    assert lib.ipt_aos_to_soa(fake, 1000, 1, 4, None) == 0
    assert lib.ipt_c2r_batched(fake, 0, 24, 4, 6, 4, 0, None) == 0


def test_oracle_and_product_share_nothing():
    """The oracle is test infrastructure: the product package never references it, and the
    oracle never references the product."""
    pkg = os.path.join(ROOT, "paper_conf_ppopp_catanzarokg14_b200")
    banned = ("import oracle", "from oracle", "libipt_oracle", "ipt_oracle", "oracle_", '"oracle"')
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                text = open(os.path.join(dirpath, f)).read()
                assert not any(b in text for b in banned), f
    for f in os.listdir(os.path.join(ROOT, "oracle")):
        if f.endswith((".py", ".c", ".h")):
            text = open(os.path.join(ROOT, "oracle", f)).read()
            assert "import paper_conf" not in text and "csrc" not in text, f

