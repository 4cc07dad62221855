"""C-ABI checks that need no GPU: the library loads, exports every entry
point include/libsat.h declares, and rejects bad arguments before touching a
device."""
import ctypes
import os
import re
import subprocess

import pytest

import paper_conf_cluster_chenwttm18_b200 as sat

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
HEADER = os.path.join(ROOT, "include", "libsat.h")


def declared_functions():
    text = open(HEADER).read()
    text = re.sub(r"/\*.*?\*/", "", text, flags=re.S)
    return sorted(set(re.findall(r"^\s*(?:sat_status|const char\s*\*|int|size_t)\s+(sat_\w+)\s*\(",
                                 text, flags=re.M)))


def test_header_declares_the_boundary():
    names = declared_functions()
    for must in ["sat_plan_create", "sat_plan_destroy", "sat_plan_workspace_bytes", "sat_compute",
                 "sat_compute_batched", "sat_compute_band", "sat_compute_host", "sat_compute_dist",
                 "sat_comm_unique_id", "sat_comm_create", "sat_comm_destroy", "sat_status_string",
                 "sat_last_error", "sat_version"]:
        assert must in names


def test_library_exports_every_declared_symbol():
    L = sat.lib()
    out = subprocess.check_output(["nm", "-D", "--defined-only", sat.LIB_PATH], text=True)
    exported = set(line.split()[-1] for line in out.splitlines() if line.strip())
    for name in declared_functions():
        assert name in exported, name
        assert getattr(L, name) is not None


def test_library_is_sm100a_only():
    out = subprocess.check_output(["cuobjdump", "--list-elf", sat.LIB_PATH], text=True)
    assert "sm_100a" in out
    for bad in ("sm_90", "sm_80", "sm_103"):
        assert bad not in out


def test_status_strings():
    L = sat.lib()
    names = [L.sat_status_string(i).decode() for i in range(6)]
    assert names == ["SAT_OK", "SAT_ERR_INVALID_ARGUMENT", "SAT_ERR_UNSUPPORTED", "SAT_ERR_CUDA",
                     "SAT_ERR_NCCL", "SAT_ERR_OUT_OF_MEMORY"]
    assert L.sat_version() >= 100


def test_null_plan_is_rejected_without_a_device():
    L = sat.lib()
    st = L.sat_compute(None, None, None, 4, 4, 4, 16, 0, None)
    assert st == 1
    assert "NULL" in L.sat_last_error().decode()
    assert L.sat_plan_create(None, 0, 0, 1, 1, 1) == 1
    h = ctypes.c_void_p()
    assert L.sat_plan_create(ctypes.byref(h), 0, 7, 1, 1, 1) == 1  # unknown pair
    assert L.sat_plan_create(ctypes.byref(h), 0, 0, 0, 1, 1) == 1  # non-positive limit
    assert L.sat_plan_destroy(None) == 0
    assert L.sat_comm_destroy(None) == 0
    assert L.sat_dist_acc_bytes(0) == 4 and L.sat_dist_acc_bytes(1) == 8


def test_plan_create_without_gpu_fails_cleanly():
    import torch
    if torch.cuda.is_available():
        pytest.skip("has a GPU")
    L = sat.lib()
    h = ctypes.c_void_p()
    assert L.sat_plan_create(ctypes.byref(h), 0, 0, 16, 16, 1) == 3  # SAT_ERR_CUDA
    assert not h.value


def test_band_partition_covers_rows_in_rank_order():
    for H in (0, 1, 7, 65536, 65537):
        for P in (1, 2, 3, 8):
            spans = [sat.band_partition(H, P, r) for r in range(P)]
            assert spans[0][0] == 0 and spans[-1][1] == H
            for (a0, a1), (b0, b1) in zip(spans, spans[1:]):
                assert a1 == b0
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= 1
            assert sizes == sorted(sizes, reverse=True)
