"""C-ABI checks that need no GPU (-m "not gpu"): the library builds and loads,
exports every function include/rmt.h declares, host-only entry points behave,
and compute calls fail loudly (no CPU fallback) when no device is present."""
import ctypes
import os
import re

import pytest
import torch

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def L():
    from paper_conf_isca_waddenlgss14_b200 import _build, rmt
    _build.build()
    return rmt.lib()


def _declared():
    src = open(os.path.join(ROOT, "include", "rmt.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(rmt_[a-z_0-9]+)\s*\(", src)))


def test_header_symbols_exported(L):
    names = _declared()
    assert len(names) >= 10
    for n in names:
        assert hasattr(L, n), f"librmt.so does not export {n}"


def test_names_and_strerror(L):
    from paper_conf_isca_waddenlgss14_b200 import rmt
    for k, i in rmt.KERNELS.items():
        assert L.rmt_kernel_name(i).decode() == k
    for v, i in rmt.VARIANTS.items():
        assert L.rmt_variant_name(i).decode() == v
    assert L.rmt_strerror(-1).decode() == "invalid argument"


def test_workspace_sizes(L):
    from paper_conf_isca_waddenlgss14_b200 import rmt
    assert rmt.workspace_size("blackscholes", "none", 1 << 16) == 0
    assert rmt.workspace_size("blackscholes", "intra_reg", 1 << 16) == 0
    assert rmt.workspace_size("blackscholes", "inter_cluster", 1 << 16) == 0  # mailbox lives in DSMEM
    inter = rmt.workspace_size("blackscholes", "inter_group", 1 << 16)
    assert inter > 0 and inter % 256 == 0
    assert rmt.workspace_size("reduction", "none", 1 << 20) >= 148 * 8 * 8


def test_fault_api_validation(L):
    from paper_conf_isca_waddenlgss14_b200 import rmt
    with pytest.raises(rmt.RmtError):
        rmt.inject_fault(2, "store_val", 0, 0)
    with pytest.raises(rmt.RmtError):
        rmt.inject_fault(0, "store_val", 32, 0)
    rmt.inject_fault(1, "store_val", 3, 10)
    rmt.clear_faults()
    with pytest.raises(rmt.RmtError):
        rmt.set_ablation(7)
    rmt.set_ablation("full")


@pytest.mark.skipif(torch.cuda.is_available(), reason="checks the no-device path")
def test_launch_fails_loudly_without_device(L):
    from paper_conf_isca_waddenlgss14_b200 import rmt
    b = rmt._Bufs()
    rc = L.rmt_launch(0, 0, ctypes.byref(b), 16, 8, None, 0, None)
    assert rc != 0
