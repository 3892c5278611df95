"""The C-ABI library loads and exports every symbol include/hccmf.h declares (-m "not gpu").

No compute call is made without a GPU; calls that need a device must fail
loudly (HCCMF_ECUDA), never fall back to the CPU."""
import ctypes
import os
import re

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _declared():
    src = open(os.path.join(ROOT, "include", "hccmf.h")).read()
    return sorted(set(re.findall(r"HCCMF_API\s+[\w\s\*]+?\b(hccmf_\w+)\s*\(", src)))


def test_header_declares_the_north_star_calls():
    names = _declared()
    for need in ("hccmf_create", "hccmf_load_ratings", "hccmf_partition", "hccmf_train_epoch", "hccmf_rmse",
                 "hccmf_get_factors"):
        assert need in names
    assert len(names) >= 19


def test_library_exports_every_declared_symbol():
    import __graft_entry__
    __graft_entry__.build()
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    L = ctypes.CDLL(pkg.LIB_PATH)
    for name in _declared():
        assert hasattr(L, name), name
    assert pkg.version().startswith("hccmf")


def test_sm100a_cubin_present():
    import subprocess
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    out = subprocess.run(["/usr/local/cuda/bin/cuobjdump", "--list-elf", pkg.LIB_PATH], capture_output=True,
                         text=True).stdout
    assert "sm_100a" in out


def test_argument_errors_without_device():
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    L = pkg.lib()
    h = ctypes.c_void_p()
    assert L.hccmf_create(10, 10, 6, 0.005, 0.01, ctypes.byref(h)) == pkg.EINVAL  # k % 4 != 0
    assert L.hccmf_create(10, 10, 8, -1.0, 0.01, ctypes.byref(h)) == pkg.EINVAL
    assert L.hccmf_create(0, 10, 8, 0.005, 0.01, ctypes.byref(h)) == pkg.EINVAL
    assert L.hccmf_create(10, 10, 8, 0.005, 0.01, None) == pkg.EINVAL
    assert L.hccmf_train_epoch(None, 0, 0) == pkg.EINVAL


@pytest.mark.skipif(os.path.exists("/dev/nvidia0"), reason="checks the no-GPU behaviour")
def test_no_cpu_fallback_without_device():
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    with pytest.raises(pkg.HccmfError) as ei:
        pkg.Model(10, 10, 8)
    assert ei.value.code == pkg.ECUDA


def test_loopback_hub_lifecycle_without_device():
    # the hub is host-only; a loopback handle needs a device and fails loudly without one
    import paper_conf_icpp_huangylhbl21_b200 as pkg
    L = pkg.lib()
    hub = ctypes.c_void_p()
    assert L.hccmf_hub_create(0, ctypes.byref(hub)) == pkg.EINVAL
    assert L.hccmf_hub_create(3, ctypes.byref(hub)) == pkg.OK and hub.value
    h = ctypes.c_void_p()
    assert L.hccmf_create_loopback(10, 10, 8, 0.005, 0.01, hub, 3, 0, ctypes.byref(h)) == pkg.EINVAL  # rank >= world
    assert L.hccmf_create_loopback(10, 10, 6, 0.005, 0.01, hub, 0, 0, ctypes.byref(h)) == pkg.EINVAL  # k % 4 != 0
    if not os.path.exists("/dev/nvidia0"):
        assert L.hccmf_create_loopback(10, 10, 8, 0.005, 0.01, hub, 1, 0, ctypes.byref(h)) == pkg.ECUDA
    assert L.hccmf_comm_counts(None, None, 0, None) == pkg.EINVAL
    L.hccmf_hub_destroy(hub)
    L.hccmf_hub_destroy(None)
