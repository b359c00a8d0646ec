"""The C ABI library loads on a CPU-only host and exports every function include/acsr.h
declares (no compute calls: there may be no GPU)."""
import ctypes
import os
import re

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def declared_functions():
    src = open(os.path.join(ROOT, "include", "acsr.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(acsr_[a-z_0-9]+)\s*\(", src)))


def test_header_declares_the_four_paper_calls():
    names = declared_functions()
    for f in ("acsr_bin", "acsr_spmv", "acsr_pagerank_step", "acsr_update_edges"):
        assert f in names


def test_library_exports_every_declared_symbol():
    import paper_conf_sc_ashariseps14_b200 as acsr
    lib = ctypes.CDLL(acsr.LIB_PATH)
    for name in declared_functions():
        assert hasattr(lib, name), name
    assert set(acsr.EXPORTED) <= set(declared_functions())


def test_host_side_queries_without_gpu():
    import paper_conf_sc_ashariseps14_b200 as acsr
    assert acsr.version() >= 100
    small = acsr.acsr_bin_workspace_bytes(1000, 1000, 10000)
    big = acsr.acsr_bin_workspace_bytes(1 << 20, 1 << 20, 16 << 20)
    assert 0 < small < big
    assert acsr._lib.acsr_status_string(3) == b"ACSR_ERR_CAPACITY"
    # host-detected argument errors return synchronously without touching a device
    assert acsr._lib.acsr_bin(-1, 0, 0, None, None, None, None, None, None, 0, None) == acsr.ACSR_ERR_INVALID_VALUE
    # acsr_bin_ex: unknown plan flags are rejected before anything is enqueued
    assert acsr._lib.acsr_bin_ex(10, 10, 10, None, None, None, None, None, None, 0, 0x80,
                                 None) == acsr.ACSR_ERR_INVALID_VALUE
    assert acsr._lib.acsr_spmv(7, 0, 0, None, None, None, None, None, None, None, None, None, 0,
                               None) == acsr.ACSR_ERR_INVALID_VALUE
