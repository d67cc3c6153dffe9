"""The specializations the GPU path will build, compiled here with the real NVRTC for
sm_100a (backend 2: real compiler, fake load/launch).  -m "not gpu": runs without a
device, so NVRTC errors in any workload kernel surface on the CPU box.

Also checks, from the cubins' resource usage, that specialization reaches the code
generator: register counts differ between generic-shaped (mode none) and folded
(mode all) builds, and no specialized kernel spills.
"""
import ctypes
import os
import re
import shutil
import subprocess

import pytest

from paper_conf_cgo_georgakoudispb25_b200 import proteus as P
from paper_conf_cgo_georgakoudispb25_b200 import workloads as W

CUOBJDUMP = shutil.which("cuobjdump") or "/usr/local/cuda/bin/cuobjdump"

# (entry, grid, block, args) at the BASELINE.json config shapes; pointers are dummies
CASES = {
    "daxpy": ((4096,), (256,), [2.0, 1 << 20, 0, 0]),
    "adam_step": ((977,), (256,), [0, 0, 0, 0, 1000000, 1e-3, 0.9, 0.999, 1e-8, 1024.0, 0.01,
                                   1, 0.1, 0.001]),
    "adam_run": ((977,), (256,), [0, 0, 0, 0, 1000000, 1e-3, 0.9, 0.999, 1e-8, 1024.0, 0.01,
                                  1, 100, 0]),
    "stencil4": ((8, 16, 6), (32, 4), [(ctypes.c_uint64 * 16)(), 0, 256, 256, 256, 2, 258, 0,
                                       256, 0.296875, 0.125, -0.0078125]),
    "stencil4_smem": ((8, 32, 9), (32, 8), [0, 0, 256, 256, 256, 2, 258, 0, 256, 0.296875, 0.125,
                                            -0.0078125]),
    "xs_lookup": ((78125,), (128,), [0] * 7 + [0x50524F54455553, 10 ** 7, 68, 11303, 12, 0, 0,
                                               0, 0]),
    "xs_index": ((273,), (256,), [0, 68, 11303, 0]),
    "xs_bin": ((148,), (1024,), [0x50524F54455553, 10 ** 7, 12, 0, 0]),
    "xs_scan": ((384,), (128,), [148, 12, 0, 0, 0]),
    "xs_scatter": ((148,), (1024,), [0x50524F54455553, 10 ** 7, 12, 0, 0, 0, 0]),
    "micro_column": ((250000,), (128,), [0] * 8 + [1000000, 64, 2, 20.0, 250.0]),
    "stencil4_ws": ((4, 32, 4), (32, 5), [(ctypes.c_uint64 * 16)(), 0, 256, 256, 256, 2, 258, 0,
                                          256, 0.296875, 0.125, -0.0078125]),
    "stencil4_p2p": ((4, 32, 4), (32, 5), [(ctypes.c_uint64 * 16)(), 0, 256, 256, 128, 2, 130,
                                           128, 256, 0.296875, 0.125, -0.0078125, 0, 0]),
    "micro_spec_sweep": ((1184,), (256,), [0, 1 << 32, 2, 0.525, 0]),
    "scale_count": ((4,), (128,), [0, 1000, 0.5]),
}


@pytest.fixture(scope="module")
def nvrtc_backend(tmp_path_factory):
    P.proteus_finalize()
    P.testing_use_fake_backend(2)
    yield str(tmp_path_factory.mktemp("cache"))
    P.proteus_finalize()
    P.testing_use_fake_backend(0)


def res_usage(cubin: bytes, tmpdir) -> dict:
    path = os.path.join(tmpdir, "k.cubin")
    with open(path, "wb") as f:
        f.write(cubin)
    out = subprocess.run([CUOBJDUMP, "-res-usage", path], capture_output=True, text=True,
                         check=True).stdout
    m = re.search(r"REG:(\d+) STACK:(\d+) SHARED:(\d+) LOCAL:(\d+)", out)
    assert m, out
    return dict(reg=int(m.group(1)), stack=int(m.group(2)), local=int(m.group(4)))


# xs_lookup at minBlocks 9 (56 registers) keeps a few slot-level values on the stack: 24 B
# since r02bm (the warp's bin range, eb0/eb1, for the multi-bin shuffle path), 16 B in
# r02bg (the concentration loaded per nuclide, XS_CA_LDG), 32 B before; one or two
# L1-resident reloads per nuclide.  That beats the spill-free 64-register build (0.887 vs
# 0.911 ms, profiles/r02/ab_xs_pipe_r02ag.txt; 0.874 vs 0.909 ms, ab_xs_caldg_r02bg.txt).
SPILL_BYTES_OK = {"xs_lookup": 24}


def compile_case(entry, mode, cache_dir):
    P.proteus_finalize()
    P.testing_use_fake_backend(2)
    P.proteus_init(device=0, cache_dir=cache_dir, mode=mode)
    k = W.register(entry, with_generic=False)
    g, b, args = CASES[entry]
    fn, cubin = P.proteus_get_specialization(k, g, b, args)
    src = P.proteus_specialized_source(k, g, b, args)
    return cubin, src


def test_every_registered_kernel_has_a_case():
    assert set(CASES) == set(W.SPECS)


@pytest.mark.parametrize("entry", list(CASES))
def test_specialization_compiles_for_sm100a(nvrtc_backend, entry, tmp_path):
    cubin, src = compile_case(entry, "all", nvrtc_backend)
    assert cubin[:4] == b"\x7fELF"
    # the specialization is named <entry>__jit (the AOT kernel keeps <entry>): ncu and the
    # launch lists tell the variants apart
    assert (entry + "__jit").encode() + b"\x00" in cubin
    assert "__launch_bounds__" in src and "PROTEUS_A" in src
    ru = res_usage(cubin, str(tmp_path))
    # no spills in the specialized kernel: no local memory, no stack frame (ptxas spills
    # live registers to the stack around calls, e.g. the fp64 division slow path, which
    # r01's xs_lookup did), no LDL/STL in the SASS -- except xs_lookup's bounded one
    stack_ok = SPILL_BYTES_OK.get(entry, 0)
    assert ru["local"] == 0 and ru["stack"] <= stack_ok, ru
    if not stack_ok:
        assert not re.search(r"\b(LDL|STL)\b", sass(cubin, str(tmp_path)))


def test_specialization_changes_codegen(nvrtc_backend, tmp_path):
    """RCF+LB must reach ptxas: the microphysics register budget changes when nz is
    folded (the generic build holds two 64-level chunks per lane)."""
    spec, _ = compile_case("micro_column", "all", nvrtc_backend)
    none, _ = compile_case("micro_column", "none", nvrtc_backend)
    r_spec = res_usage(spec, str(tmp_path))["reg"]
    r_none = res_usage(none, str(tmp_path))["reg"]
    assert r_spec < r_none, (r_spec, r_none)


def sass(cubin: bytes, tmpdir) -> str:
    path = os.path.join(tmpdir, "k.cubin")
    with open(path, "wb") as f:
        f.write(cubin)
    return subprocess.run([CUOBJDUMP, "-sass", path], capture_output=True, text=True,
                          check=True).stdout


def test_stencil_specialization_uses_tma_and_folds_constants(nvrtc_backend, tmp_path):
    """SASS evidence: the specialized stencil streams tiles with TMA (UTMALDG) on mbarriers
    (SYNCS), and the folded coefficient a2 = -1/128 appears as an immediate."""
    cubin, _ = compile_case("stencil4", "all", nvrtc_backend)
    s = sass(cubin, str(tmp_path))
    assert "UTMALDG.3D" in s and "SYNCS" in s
    assert "-0.0078125" in s
    none, _ = compile_case("stencil4", "none", nvrtc_backend)
    assert "-0.0078125" not in sass(none, str(tmp_path))


def test_xs_search_unrolled_when_grid_folded(nvrtc_backend, tmp_path):
    """RCF on n_grid: G = 11303 = 0x2c27 (the per-nuclide row stride of egrid and recs,
    and the bisection bound) is an immediate of the specialization, not of the build with
    nothing folded."""
    cubin, _ = compile_case("xs_lookup", "all", nvrtc_backend)
    assert "0x2c27" in sass(cubin, str(tmp_path)).lower()
    none, _ = compile_case("xs_lookup", "none", nvrtc_backend)
    assert "0x2c27" not in sass(none, str(tmp_path)).lower()


def test_bound_globals_compile_and_use_the_bound_address(nvrtc_backend, tmp_path):
    """A specialization with device globals bound (P@19299-21805) compiles for sm_100a
    and addresses the bound storage: the bound address's high word is an immediate in the
    SASS (the low word is folded into load offsets), absent from an unbound build."""
    P.proteus_finalize()
    P.testing_use_fake_backend(2)
    P.proteus_init(device=0, cache_dir=nvrtc_backend, mode="all")
    k = W.register("scale_count", with_generic=False)
    k.bind_global("proteus_demo_scale", 0x7F1234560000)
    k.bind_global("proteus_demo_count", 0x7F1234561000)
    g, b, args = CASES["scale_count"]
    fn, cubin = P.proteus_get_specialization(k, g, b, args)
    assert "0x7f12" in sass(cubin, str(tmp_path)).lower()
    free = P.proteus_register_kernel("scale_count", W.kernel_source("scale_count"),
                                     *W.SPECS["scale_count"][:2], None, "")
    _, cubin2 = P.proteus_get_specialization(free, g, b, args)
    assert "0x7f12" not in sass(cubin2, str(tmp_path)).lower()


def test_lineinfo_is_opt_in_and_keyed(nvrtc_backend, tmp_path):
    """PROTEUS_F_LINEINFO: without it the cubin carries no line table (smaller, faster to
    compile); with it, -lineinfo reaches NVRTC; the two are distinct keys (distinct disk
    files) and the SASS instructions are the same."""
    P.proteus_finalize()
    P.proteus_init(device=0, cache_dir=str(tmp_path / "c"), mode="all")
    k = W.register("adam_step", with_generic=False)
    g, b, args = CASES["adam_step"]
    _, plain = P.proteus_get_specialization(k, g, b, args)
    P.proteus_finalize()
    P.proteus_init(device=0, cache_dir=str(tmp_path / "c"),
                   flags=P.F_RCF | P.F_LB | P.F_FOLD_DIMS | P.F_DISK | P.F_LINEINFO)
    k = W.register("adam_step", with_generic=False)
    _, lined = P.proteus_get_specialization(k, g, b, args)
    assert len(os.listdir(tmp_path / "c")) == 2          # two keys, two cubin files
    assert b".nv_debug_line_sass" in lined and b".nv_debug_line_sass" not in plain
    strip = lambda s: [ln.split("/*")[1] for ln in s.splitlines() if re.match(r"\s+/\*[0-9a-f]{4}\*/", ln)]
    assert strip(sass(plain, str(tmp_path))) == strip(sass(lined, str(tmp_path)))


# ---------------------------------------------------------------- NEXT-1: IR-level path
@pytest.mark.parametrize("entry", list(CASES))
def test_ir_level_specialization_compiles(nvrtc_backend, entry, tmp_path):
    """PROTEUS_F_IR (mode "ir"): the kernel compiled to LTO-IR with the annotated values and
    grid dims as extern device constants, a constants module per key, nvJitLink -lto: a
    valid sm_100a cubin named <entry>__jit_ir, no spills, about the registers of the source
    path (the link-time optimizer folded what NVRTC folds from literals)."""
    cubin, src = compile_case(entry, "ir", nvrtc_backend)
    assert cubin[:4] == b"\x7fELF"
    assert "//@@proteus-ir-kernel@@" in src and "extern __device__ const" in src
    assert (entry + "__jit_ir").encode() + b"\x00" in cubin
    ru = res_usage(cubin, str(tmp_path))
    assert ru["local"] == 0 and ru["stack"] <= SPILL_BYTES_OK.get(entry, 0), ru
    ref, _ = compile_case(entry, "all", nvrtc_backend)
    assert abs(ru["reg"] - res_usage(ref, str(tmp_path))["reg"]) <= 8   # same code, LTO pipeline


def test_ir_level_folds_constants_and_compiles_kernel_ir_once(nvrtc_backend, tmp_path):
    """The IR path folds the stencil coefficients at link time (a2 = -1/128 is an immediate
    of the SASS, TMA kept) and compiles the kernel's LTO-IR once: a second key differing
    only in an annotated value (a0) and the grid costs a constants module + link only."""
    cubin, _ = compile_case("stencil4_ws", "ir", str(tmp_path / "fresh"))   # no disk hits
    s = sass(cubin, str(tmp_path))
    assert "-0.0078125" in s and "UTMALDG" in s
    k = W.register("stencil4_ws", with_generic=False)
    g, b, args = CASES["stencil4_ws"]
    args2 = list(args)
    args2[9] = 0.25
    P.proteus_get_specialization(k, (4, 32, 8), b, args2)
    st = P.proteus_cache_stats()
    assert st["compiles"] == 2 and st["ir_compiles"] == 1, st


@pytest.mark.parametrize("mode,suffix", [("none", "__jit_none"), ("lb", "__jit_lb"),
                                         ("rcf", "__jit_vd"), ("dims", "__jit_lbd"),
                                         ("values", "__jit_lbv"), ("all", "__jit")])
def test_every_mode_names_its_kernel(nvrtc_backend, mode, suffix):
    """distinct kernel names per variant -- the generic AOT kernel is <entry>,
    the product specialization <entry>__jit, each ablation mode <entry>__jit_<mode>."""
    cubin, _ = compile_case("daxpy", mode, nvrtc_backend)
    assert ("daxpy" + suffix).encode() + b"\x00" in cubin
