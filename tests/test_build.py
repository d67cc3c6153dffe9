"""The in-tree native build (what __graft_entry__.build() runs) succeeds and the AOT
library exports a generic sm_100a function for every registered kernel (CPU box)."""
import ctypes
import os


def test_native_build_and_aot_registry():
    from paper_conf_cgo_georgakoudispb25_b200 import _build
    lib, aot = _build.build()
    assert os.path.exists(lib)
    if not os.path.exists(aot):     # no nvcc on this host
        return
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
    assert set(_build.ENTRIES) == set(W.SPECS)
    L = ctypes.CDLL(aot)
    assert hasattr(L, "proteus_aot_function")
