"""C-ABI library checks that need no GPU (-m "not gpu")."""
import ctypes
import os
import re

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "smiler.h")
PKG = os.path.join(ROOT, "paper_conf_sigmod_zhout15_b200")


def declared_functions():
    src = open(HEADER).read()
    return re.findall(r"SMILER_API\s+[\w\s\*]+?\b(smiler_\w+)\s*\(", src)


@pytest.fixture(scope="module")
def built():
    from paper_conf_sigmod_zhout15_b200 import build
    return build.build()


def test_header_declares_the_boundary():
    fns = set(declared_functions())
    # the three calls of the north star plus merge and the per-step entry points
    for f in ("smiler_index_build", "smiler_knn", "smiler_free", "smiler_merge_topk",
              "smiler_index_build_shard", "smiler_knn_ex", "smiler_lower_bounds", "smiler_dtw",
              "smiler_index_envelope", "smiler_last_error", "smiler_abi_version", "smiler_lower_bounds_ex",
              "smiler_predict", "smiler_stream_create_ex"):
        assert f in fns, f


def test_library_exports_every_declared_symbol(built):
    L = ctypes.CDLL(built)
    for f in declared_functions():
        assert hasattr(L, f), "libsmiler.so does not export %s" % f


def test_abi_version_and_stats_layout(built):
    import paper_conf_sigmod_zhout15_b200 as pkg
    assert pkg.smiler_abi_version() == 4
    # struct sizes match the header (8 x 8-byte counters, 2 int32, 8 doubles,
    # cascade_pruned, ns_cascade)
    assert ctypes.sizeof(pkg.KnnStats) == 8 * 8 + 2 * 4 + 8 * 8 + 8 + 8
    assert ctypes.sizeof(pkg.KnnOpts) == 11 * 4 + 4 + 8   # + padding + shared_tau


def test_no_gpu_means_error_not_fallback(built):
    """Without a CUDA device the library refuses (ECUDA); it never computes on the CPU."""
    import torch
    if torch.cuda.is_available():
        pytest.skip("a GPU is present")
    import paper_conf_sigmod_zhout15_b200 as pkg
    x = np.zeros(100, np.int16)
    with pytest.raises(pkg.SmilerError) as ei:
        pkg.smiler_index_build(x, None, 8, 2.0)
    assert ei.value.code == -4
    assert "no CPU fallback" in str(ei.value)


def test_null_safe_free_and_last_error(built):
    import paper_conf_sigmod_zhout15_b200 as pkg
    pkg.smiler_free(None)
    L = ctypes.CDLL(built)
    L.smiler_last_error.restype = ctypes.c_char_p
    assert isinstance(L.smiler_last_error(), bytes)


def test_bad_arguments_map_to_einval(built):
    import paper_conf_sigmod_zhout15_b200 as pkg
    L = pkg.smiler.lib()
    h = ctypes.c_void_p()
    x = np.zeros(10, np.int16)
    # argument checks happen before any device access
    assert L.smiler_index_build(None, 0, 10, None, 1, 8, 1.0, 0, None, ctypes.byref(h)) == -1
    assert L.smiler_index_build(x.ctypes.data, 0, 0, None, 1, 8, 1.0, 0, None, ctypes.byref(h)) == -1
    assert L.smiler_index_build(x.ctypes.data, 0, 10, None, 1, 0, 1.0, 0, None, ctypes.byref(h)) == -1
    assert L.smiler_index_build(x.ctypes.data, 7, 10, None, 1, 8, 1.0, 0, None, ctypes.byref(h)) == -1
    assert L.smiler_knn(None, None, None, 1, None, 1, 1, None, None, None) == -1


def test_product_never_touches_the_oracle():
    """The product package shares no code with oracle/ and never imports it."""
    for dirpath, _, files in os.walk(PKG):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src, f
                assert "orc_" not in src, f
    osrc = open(os.path.join(ROOT, "oracle", "oracle.c")).read()
    assert "smiler" not in osrc.replace("SMiLer", "")
