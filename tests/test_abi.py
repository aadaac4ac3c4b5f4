"""C-ABI library: builds, loads and exports every symbol of include/glp.h.
No compute calls without a GPU (those live in test_gpu_*.py)."""
import ctypes
import os
import re

import pytest
import torch

import paper_conf_sigmod_yelhls21_b200 as glp
from paper_conf_sigmod_yelhls21_b200 import _build

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_symbols():
    src = open(os.path.join(ROOT, "include", "glp.h")).read()
    return sorted(set(re.findall(r"^\s*(?:glp_status|const char \*)\s*(glp_\w+)\s*\(", src, re.M)))


def test_header_declares_boundary():
    syms = declared_symbols()
    for s in ["glp_graph_create", "glp_run", "glp_labels_get", "glp_graph_destroy", "glp_last_error"]:
        assert s in syms


def test_library_builds_and_exports_all_symbols():
    lib_path = _build.build()
    lib = ctypes.CDLL(lib_path)
    for s in declared_symbols():
        assert hasattr(lib, s), s
    assert set(declared_symbols()) == set(glp.EXPORTS)


def test_struct_layout_matches_header():
    # the ctypes mirror against the compiled header's sizeof (glp_struct_sizes)
    mine = [ctypes.sizeof(t) for t in (glp.glp_csr, glp.glp_dist, glp.glp_params, glp.glp_run_info,
                                        glp.glp_iter_stat, glp.glp_kernel_stat)]
    assert mine == glp.glp_struct_sizes()  # (glp_params.struct_size is also checked by glp_run)


def test_version_and_partition_host_only():
    assert "sm_100a" in glp.glp_version()
    assert glp.glp_partition(10, 3) == [0, 4, 8, 10]
    off = torch.tensor([0, 10, 10, 12, 20, 40], dtype=torch.int64)
    b = glp.glp_partition(5, 2, off, edge_balanced=True)
    assert b[0] == 0 and b[-1] == 5 and b == sorted(b)


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-GPU failure path")
def test_no_gpu_fails_loudly():
    off = torch.tensor([0, 1, 2], dtype=torch.int64)
    col = torch.tensor([1, 0], dtype=torch.int32)
    with pytest.raises(glp.GlpError) as e:
        glp.glp_graph_create(2, off, col)
    assert e.value.status == 6  # GLP_ERR_UNSUPPORTED, never a CPU fallback


def test_bad_params_rejected_before_device_use():
    lib = glp.load_library()
    assert lib.glp_graph_create(None, None, None, None) == 1
    assert lib.glp_graph_destroy(None) == 0
    assert lib.glp_run(None, 0, 1, None, 0, None, None) == 1
