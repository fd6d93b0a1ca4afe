"""CPU tests of the C-ABI boundary: the library loads, exports every symbol
include/nfc.h declares, the ctypes layouts match the header's sizes, and the
argument-validation paths that run before any CUDA call return the documented
status codes."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def nfc():
    import __graft_entry__
    from paper_conf_hpca_hul18_b200 import build
    build.build()
    from paper_conf_hpca_hul18_b200 import nfc as m
    return m


def _declared(headers=("nfc.h", "nfc_debug.h")):
    src = "".join(open(os.path.join(ROOT, "include", h)).read() for h in headers)
    return sorted(set(re.findall(r"NFC_API\s+[\w\s\*]*?\b(nfc_\w+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = _declared()
    for must in ("nfc_build_chain", "nfc_load_tables", "nfc_process_batch", "nfc_collect_stats"):
        assert must in names


def test_library_exports_every_declared_symbol(nfc):
    lib = ctypes.CDLL(nfc.LIB_PATH)
    for name in _declared():
        assert hasattr(lib, name), name
    assert set(_declared(('nfc.h',))) == set(nfc.EXPORTS)
    assert set(_declared(('nfc_debug.h',))) == set(nfc.DEBUG_EXPORTS)


def test_ctypes_layouts_match_header(nfc):
    import nfcgen
    assert ctypes.sizeof(nfc.Batch) == 40
    assert ctypes.sizeof(nfc.Result) == 40
    assert nfc.RESULT_DTYPE.itemsize == 16
    assert nfcgen.ACL_RULE.itemsize == 48 and nfcgen.SA.itemsize == 48
    assert nfcgen.ROUTE4.itemsize == 8 and nfcgen.ROUTE6.itemsize == 20 and nfcgen.NEXTHOP.itemsize == 8


def test_validation_before_cuda(nfc):
    lib = nfc.lib
    h = ctypes.c_void_p()
    opts = nfc.ChainOpts(0, 0, 0)
    empty = (ctypes.c_uint32 * 1)(1)
    assert lib.nfc_build_chain(empty, 0, ctypes.byref(opts), ctypes.byref(h)) == nfc.NFC_EUNSUP
    seven = (ctypes.c_uint32 * 7)(1, 2, 3, 4, 5, 6, 1)
    assert lib.nfc_build_chain(seven, 7, ctypes.byref(opts), ctypes.byref(h)) == nfc.NFC_EUNSUP
    rep = (ctypes.c_uint32 * 2)(nfc.IPSEC, nfc.IPSEC)   # repeated IPsec / NAT: unsupported (repeated ACL/DPI: NEXT-2)
    assert lib.nfc_build_chain(rep, 2, ctypes.byref(opts), ctypes.byref(h)) == nfc.NFC_EUNSUP
    rep = (ctypes.c_uint32 * 3)(nfc.ACL, nfc.NAT, nfc.NAT)
    assert lib.nfc_build_chain(rep, 3, ctypes.byref(opts), ctypes.byref(h)) == nfc.NFC_EUNSUP
    bad = (ctypes.c_uint32 * 1)(9)
    assert lib.nfc_build_chain(bad, 1, ctypes.byref(opts), ctypes.byref(h)) == nfc.NFC_EINVAL
    assert lib.nfc_build_chain(None, 1, ctypes.byref(opts), ctypes.byref(h)) == nfc.NFC_EINVAL
    assert len(lib.nfc_last_error()) > 0
    assert lib.nfc_load_tables(None, 1, None, 0) == nfc.NFC_EINVAL
    assert lib.nfc_collect_stats(None, None, 0, 0) == nfc.NFC_EINVAL
    assert nfc.version().startswith("nfc-b200")


def test_flags_validation_before_cuda(nfc):
    # NFC_F_UNFUSED (NEXT-1 baseline) does not offer IPsec chains; unknown flag bits are rejected
    lib = nfc.lib
    h = ctypes.c_void_p()
    esp = (ctypes.c_uint32 * 2)(nfc.ACL, nfc.IPSEC)
    assert lib.nfc_build_chain(esp, 2, ctypes.byref(nfc.ChainOpts(0, nfc.F_UNFUSED, 0)), ctypes.byref(h)) == nfc.NFC_EUNSUP
    one = (ctypes.c_uint32 * 1)(nfc.ACL)
    assert lib.nfc_build_chain(one, 1, ctypes.byref(nfc.ChainOpts(0, 0x80, 0)), ctypes.byref(h)) == nfc.NFC_EINVAL


def test_no_oracle_in_product():
    # the product path never imports, includes or links the oracle
    pkg = os.path.join(ROOT, "paper_conf_hpca_hul18_b200")
    bad = re.compile(r"(import\s+oracle|from\s+oracle|#include\s+\S*oracle|liboracle|oracle\.h)")
    for dp, _, fs in os.walk(pkg):
        for f in fs:
            if f.endswith((".py", ".cu", ".cpp", ".h", ".cuh")):
                txt = open(os.path.join(dp, f)).read()
                assert not bad.search(txt), f


def test_stream_dpi_validation_before_cuda(nfc):
    """nfc_dpi_stream_create: NULL / malformed arguments are NFC_EINVAL before any CUDA
    call; the struct layout matches the header (8 pointers + 2 u32 = 56 B)."""
    assert ctypes.sizeof(nfc.StreamResult) == 56
    L = nfc.lib
    h = ctypes.c_void_p()
    good = np.frombuffer(b"abcab", dtype=np.uint8).copy()
    off = np.array([0, 3, 5], dtype=np.uint32)
    act = np.zeros(2, dtype=np.uint8)
    spec = nfc.DpiSpec(2, good.ctypes.data, off.ctypes.data, act.ctypes.data)
    assert L.nfc_dpi_stream_create(0, None, 16, ctypes.byref(h)) == nfc.NFC_EINVAL
    assert L.nfc_dpi_stream_create(0, ctypes.byref(spec), 0, ctypes.byref(h)) == nfc.NFC_EINVAL
    bad_off = np.array([0, 3, 3], dtype=np.uint32)          # empty pattern
    bad = nfc.DpiSpec(2, good.ctypes.data, bad_off.ctypes.data, act.ctypes.data)
    assert L.nfc_dpi_stream_create(0, ctypes.byref(bad), 16, ctypes.byref(h)) == nfc.NFC_EINVAL
    assert b"empty pattern" in L.nfc_last_error()
    assert L.nfc_dpi_stream_process(None, None, None, None) == nfc.NFC_EINVAL
    assert L.nfc_dpi_stream_destroy(None) == nfc.NFC_OK


def test_stream_dpi_fails_loudly_without_gpu(nfc):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    blob = np.frombuffer(b"abc", dtype=np.uint8).copy()
    with pytest.raises(nfc.NfcError):
        nfc.DpiStream(blob, np.array([0, 3], dtype=np.uint32), np.zeros(1, dtype=np.uint8), max_flows=8)


@pytest.mark.parametrize("rx,code", [(b"ab*", "NFC_EOK_CLASS"), (b"a+", "NFC_EOK_CLASS"), (b"a{2,}", "NFC_EOK_CLASS"),
                                     (b"a*", "NFC_EINVAL"), (b"(ab)*", "NFC_EINVAL"), (b"*a", "NFC_EINVAL"),
                                     (b"a?", "NFC_EINVAL"), (b"(a", "NFC_EINVAL"), (b"[ab", "NFC_EINVAL"),
                                     (b"a)", "NFC_EINVAL"), (b"\\q", "NFC_EINVAL"), (b"a{0}", "NFC_EINVAL"),
                                     # anchors are not silently taken as literal bytes
                                     (b"^GET", "NFC_EUNSUP"), (b"a$", "NFC_EUNSUP"), (b"(x|^y)", "NFC_EUNSUP"),
                                     # longest match above 1024 B / nested repeats: rejected up front, fast
                                     (b"((a{64}){64}){64}", "NFC_EUNSUP"), (b"(a{64}){17}", "NFC_EOK_CLASS"),
                                     (b"(((((a{64}){64}){64}){64}){64}){64}", "NFC_EUNSUP"),
                                     (b"[^$]x", "NFC_EOK_CLASS")])
def test_regex_rejected_before_cuda(nfc, rx, code):
    """Syntax errors and empty-matching expressions are NFC_EINVAL, anchors and NFA
    blow-ups NFC_EUNSUP -- decided by the host compiler before any CUDA call, fast
    (R#33, R#35)."""
    blob = np.frombuffer(rx, dtype=np.uint8).copy()
    off = np.array([0, len(rx)], dtype=np.uint32)
    act = np.zeros(1, dtype=np.uint8)
    spec = nfc.DpiSpec(1, blob.ctypes.data, off.ctypes.data, act.ctypes.data)
    h = ctypes.c_void_p()
    rc = nfc.lib.nfc_dpi_stream_create_regex(0, ctypes.byref(spec), 16, 0, ctypes.byref(h))
    if code == "NFC_EOK_CLASS":
        # valid: the compile succeeds ('^' / '$' inside a class are bytes; unbounded and long
        # matches walk flow-serially) and only the CUDA setup can fail
        assert rc in (nfc.NFC_OK, nfc.NFC_ECUDA)
        if rc == nfc.NFC_OK:
            nfc.lib.nfc_dpi_stream_destroy(h)
        return
    assert rc == getattr(nfc, code)
