"""CPU-side checks of the C-ABI library: it builds/loads, exports every symbol include/specinfer.h
declares, and validates host-checkable arguments before touching a device."""
import ctypes
import os
import re

import pytest

import paper_conf_asplos_miaoozcwzwzyssc24_b200 as spi
from paper_conf_asplos_miaoozcwzwzyssc24_b200 import build_lib

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def lib():
    build_lib.build()
    return spi.load_library()


def test_header_symbols_exported(lib):
    hdr = open(os.path.join(ROOT, "include", "specinfer.h")).read()
    declared = set(re.findall(r"\b(specinfer_[a-z_]+)\s*\(", hdr))
    assert declared == set(spi.EXPORTED_SYMBOLS)
    for name in declared:
        assert getattr(lib, name) is not None


def test_status_strings_and_launch_counts(lib):
    for s in range(6):
        assert lib.specinfer_status_string(s)
    assert spi.specinfer_launches_per_call("tree_attention") == 1
    assert spi.specinfer_launches_per_call("kv_commit") == 2
    assert spi.specinfer_launches_per_call("nope") == -1


def test_host_validation_without_gpu(lib):
    """Shape errors are returned synchronously before any device work."""
    bad_dim = spi.make_shape(2, 8, 4, 4, 64, head_dim=64)
    assert lib.specinfer_tree_prepare(ctypes.byref(bad_dim), None, None, None, None, None, None) in (1, 2)
    assert lib.specinfer_workspace_size(ctypes.byref(bad_dim)) == 0
    too_many_nodes = spi.make_shape(2, 300, 4, 4, 400)
    assert lib.specinfer_workspace_size(ctypes.byref(too_many_nodes)) == 0
    gqa_bad = spi.make_shape(2, 8, 6, 4, 64)
    assert lib.specinfer_workspace_size(ctypes.byref(gqa_bad)) == 0
    ok = spi.make_shape(16, 21, 32, 32, 2069, vocab=32000, max_depth=8)
    assert lib.specinfer_workspace_size(ctypes.byref(ok)) > 0
    # NULL pointers -> INVALID_ARG (checked before the device)
    assert lib.specinfer_tree_attention(ctypes.byref(ok), None, None, None, None, None, None, None, None, None,
                                        None) == 1
    assert lib.specinfer_kv_commit(ctypes.byref(ok), None, None, None, None, None, None) == 1


def test_no_cpu_fallback():
    """The product path refuses CPU tensors instead of computing anything on the host."""
    import torch
    import workloads as W
    tb = W.make_tree_batch([W.chain_tree(3)], [2])
    shape = spi.make_shape(1, 3, 2, 2, 8)
    with pytest.raises(ValueError):
        spi.specinfer_tree_prepare(shape, tb.parent, tb.depth, tb.prefix_len, tb.n_nodes,
                                   torch.empty(1024, dtype=torch.uint8))
