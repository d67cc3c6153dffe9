"""libproteus on the CPU box: ABI exports, key parity with the Python key oracle, the
literal emitter, and the cache state machine on the fake backend.
All -m "not gpu"."""
import ctypes
import math
import os
import re
import struct
import threading
import time

import numpy as np
import pytest

from oracle import key as K
from paper_conf_cgo_georgakoudispb25_b200 import proteus as P

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
GENERIC = 0x1234

DAXPY_SRC = r'''
#include "proteus_device.h"
extern "C" __global__ PROTEUS_LAUNCH_BOUNDS
void daxpy(double a_rt, long long n_rt, const double* x, double* y) {
  const double a = PROTEUS_SPEC(1, a_rt);
  const long long n = PROTEUS_SPEC(2, n_rt);
  long long i = (long long)blockIdx.x * PROTEUS_BLOCKDIM_X + threadIdx.x;
  if (i < n) y[i] = a * x[i] + y[i];
}
'''
DAXPY_TYPES = [P.F64, P.I64, P.PTR, P.PTR]


@pytest.fixture
def fake(tmp_path):
    P.proteus_finalize()
    P.testing_use_fake_backend(True)
    P.testing_fake_control(False, 0)
    state = {"dir": str(tmp_path / "cache")}

    def init(**kw):
        kw.setdefault("cache_dir", state["dir"])
        return P.proteus_init(device=0, **kw)

    state["init"] = init
    yield state
    P.proteus_finalize()
    P.testing_use_fake_backend(False)
    P.testing_fake_control(False, 0)


def reg_daxpy(src=DAXPY_SRC, generic=None, options=""):
    return P.proteus_register_kernel("daxpy", src, DAXPY_TYPES, [1, 2], generic, options)


def _declared(h):
    text = open(os.path.join(ROOT, "include", h)).read()
    return set(re.findall(r"^\s*(?:proteus_status|const char\*)\s+(proteus_\w+)\(", text, re.M))


def _exported(lib_path):
    import subprocess
    out = subprocess.run(["nm", "-D", "--defined-only", lib_path], capture_output=True,
                         text=True, check=True).stdout
    return {ln.split()[-1] for ln in out.splitlines() if " T " in ln}


def test_every_declared_symbol_is_exported():
    """proteus.h's C ABI is exported by the product library and the test hooks of
    proteus_testing.h only by libproteus_testing.so (not by the product .so)."""
    api, hooks = _declared("proteus.h"), _declared("proteus_testing.h")
    assert len(api) >= 17 and len(hooks) >= 4
    for n in sorted(api):
        assert hasattr(P.lib, n), n
    prod = _exported(P.LIB_PATH)
    assert api <= prod
    assert not any(n.startswith("proteus_testing") for n in prod), sorted(prod)
    assert not any("fake" in n.lower() for n in prod), sorted(n for n in prod if "fake" in n.lower())
    assert hooks <= _exported(P.TESTING_PATH)


def test_not_initialised_is_an_error():
    P.proteus_finalize()
    with pytest.raises(P.ProteusError) as e:
        P.proteus_cache_stats()
    assert e.value.status == 2


def test_kernel_id_and_key_bytes_match_python_oracle(fake):
    fake["init"]()
    k = reg_daxpy(options="-fmad=false")
    kid, toolkit, arch = k.info()
    assert arch == "sm_100a" and toolkit.startswith("fake|proteus-2|hdr=")
    assert kid == K.kernel_id(DAXPY_SRC, "daxpy", "-fmad=false", toolkit, arch)
    for a, n, g, b in [(2.0, 1 << 20, (1024, 1, 1), (256, 1, 1)),
                       (-0.0, 7, (1, 2, 3), (32, 4, 2)), (1e-310, -5, (9, 1, 1), (1024, 1, 1))]:
        kb, h = P.proteus_key(k, g, b, [a, n, 0, 0])
        want = K.key_bytes(kid, K.F_RCF | K.F_LB | K.F_FOLD_DIMS, 1,
                           [(1, K.F64, a), (2, K.I64, n)], g, b)
        assert kb == want
        assert h == K.key_hash(want)


def test_listing1_adam_key_matches_oracle(fake):
    """Adam as in Listing 1 (P@38745): 13 args, annotate 5..11 and 13 (not 12, mode)."""
    fake["init"]()
    src = '#include "proteus_device.h"\nextern "C" __global__ void adam(){}\n'
    types = [P.PTR] * 4 + [P.F32] * 5 + [P.I32, P.U64, P.I32, P.F32]
    ann = [13, 5, 6, 7, 8, 9, 10, 11]            # any order accepted
    k = P.proteus_register_kernel("adam", src, types, ann)
    kid, _, _ = k.info()
    vals = [0, 0, 0, 0, 0.9, 0.999, 1e-8, 1024.0, 1e-3, 7, 1000000, 1, 0.01]
    kb, _ = P.proteus_key(k, (977,), (256,), vals)
    ann_vals = [(i, types[i - 1], struct.pack({P.F32: "<f", P.I32: "<i", P.U64: "<Q"}[types[i - 1]],
                                              vals[i - 1])) for i in sorted(ann)]
    assert kb == K.key_bytes(kid, 7, 1, ann_vals, (977, 1, 1), (256, 1, 1))
    # a non-annotated argument (mode, arg 12) does not change the key
    vals2 = list(vals)
    vals2[11] = 0
    assert P.proteus_key(k, (977,), (256,), vals2)[0] == kb
    vals3 = list(vals)
    vals3[12] = 0.02
    assert P.proteus_key(k, (977,), (256,), vals3)[0] != kb


@pytest.mark.parametrize("ann,types", [([0], DAXPY_TYPES), ([5], DAXPY_TYPES),
                                       ([1, 1], DAXPY_TYPES), ([3], DAXPY_TYPES)])
def test_registration_validation(fake, ann, types):
    fake["init"]()
    with pytest.raises(P.ProteusError) as e:
        P.proteus_register_kernel("daxpy", DAXPY_SRC, types, ann)
    assert e.value.status == 1


def test_launch_validation(fake):
    fake["init"]()
    k = reg_daxpy()
    with pytest.raises(P.ProteusError):
        P.proteus_launch(k, (1,), (2048,), [1.0, 1, 0, 0])
    with pytest.raises(P.ProteusError):
        P.proteus_launch(k, (0,), (32,), [1.0, 1, 0, 0])


def _parse_literal(lit):
    lit = lit.strip()
    assert lit[0] == "(" and lit[-1] == ")"
    body = lit[1:-1]
    m = re.fullmatch(r"__int_as_float\(0x([0-9a-f]{8})\)", body)
    if m:
        return ("f32bits", int(m.group(1), 16))
    m = re.fullmatch(r"__longlong_as_double\(0x([0-9a-f]{16})ll\)", body)
    if m:
        return ("f64bits", int(m.group(1), 16))
    if body.endswith("f"):
        return ("f32", float.fromhex(body[:-1]))
    if "p" in body:
        return ("f64", float.fromhex(body))
    return ("int", body)


def _bits32(x):
    return struct.unpack("<I", struct.pack("<f", x))[0]


def test_literals_reproduce_bits_exactly(fake):
    """RCF must fold the exact runtime value (P@22119): hex-float round trip."""
    fake["init"]()
    src = '#include "proteus_device.h"\nextern "C" __global__ void k(float a, double b){}\n'
    k = P.proteus_register_kernel("k", src, [P.F32, P.F64], [1, 2])
    rs = np.random.default_rng(5)
    pats32 = [0x00000000, 0x80000000, 0x00000001, 0x007FFFFF, 0x3F800000, 0x7F7FFFFF,
              0x7F800000, 0xFF800000, 0x7FC00001] + list(rs.integers(0, 2 ** 32, 200))
    for bits in pats32:
        a = ctypes.c_float.from_buffer_copy(struct.pack("<I", int(bits)))
        b = ctypes.c_double(float(rs.standard_normal()) * 10 ** float(rs.integers(-300, 300)))
        src_out = P.proteus_specialized_source(k, (1,), (32,), [a, b])
        la = re.search(r"#define PROTEUS_A1_OR\(x\) (.*)", src_out).group(1)
        lb = re.search(r"#define PROTEUS_A2_OR\(x\) (.*)", src_out).group(1)
        kind, v = _parse_literal(la)
        if kind == "f32bits":
            assert v == int(bits)
            assert not math.isfinite(struct.unpack("<f", struct.pack("<I", int(bits)))[0])
        else:
            assert kind == "f32"
            assert _bits32(v) == int(bits)          # exact in fp32 (incl. -0.0, subnormals)
        kind, v = _parse_literal(lb)
        assert kind == "f64" and struct.pack("<d", v) == struct.pack("<d", b.value)


def test_integer_literal_extremes(fake):
    fake["init"]()
    src = '#include "proteus_device.h"\nextern "C" __global__ void k(int a, long long b, unsigned c, unsigned long long d){}\n'
    k = P.proteus_register_kernel("k", src, [P.I32, P.I64, P.U32, P.U64], [1, 2, 3, 4])
    s = P.proteus_specialized_source(k, (1,), (32,), [-2 ** 31, -2 ** 63, 2 ** 32 - 1, 2 ** 64 - 1])
    assert "#define PROTEUS_A1_OR(x) (-2147483647-1)" in s
    assert "#define PROTEUS_A2_OR(x) (-9223372036854775807ll-1ll)" in s
    assert "#define PROTEUS_A3_OR(x) (4294967295u)" in s
    assert "#define PROTEUS_A4_OR(x) (18446744073709551615ull)" in s


@pytest.mark.parametrize("mode,rcf,lb", [("none", False, False), ("lb", False, True),
                                         ("rcf", True, False), ("all", True, True)])
def test_ablation_modes_prelude(fake, mode, rcf, lb):
    """The paper's None / LB / RCF / LB+RCF modes (P@39538-40272)."""
    fake["init"](mode=mode)
    k = reg_daxpy()
    s = P.proteus_specialized_source(k, (4,), (128,), [3.0, 500, 0, 0])
    assert ("PROTEUS_A1_OR" in s) == rcf and ("PROTEUS_A2_OR" in s) == rcf
    assert ("__launch_bounds__(128, 1)" in s) == lb
    assert ("#define PROTEUS_BDX 128u" in s) == rcf   # launch dims fold with RCF
    assert s.endswith(DAXPY_SRC)


def test_min_blocks_enters_prelude_and_key(fake):
    fake["init"](min_blocks_per_sm=3)
    k = reg_daxpy()
    s = P.proteus_specialized_source(k, (4,), (128,), [3.0, 500, 0, 0])
    assert "__launch_bounds__(128, 3)" in s
    kb, _ = P.proteus_key(k, (4,), (128,), [3.0, 500, 0, 0])
    assert struct.unpack_from("<I", kb, 20)[0] == 3


def test_launch_attrs_reach_every_launch_path_not_the_key(fake):
    """proteus_kernel_set_launch_attrs (programmatic dependent launch): applied to the
    specialized, generic (async miss) and proteus_launch_aot launches; unknown bits are
    rejected; the key and the specialization are unchanged."""
    fake["init"]()
    k = reg_daxpy()
    kb0, _ = P.proteus_key(k, (4,), (128,), [3.0, 500, 0, 0])
    with pytest.raises(P.ProteusError):
        k.set_launch_attrs(2)
    k.set_launch_attrs(P.LAUNCH_PDL)
    kb1, _ = P.proteus_key(k, (4,), (128,), [3.0, 500, 0, 0])
    assert kb0 == kb1
    P.proteus_launch(k, (4,), (128,), [3.0, 500, 0, 0])
    assert P.testing_fake_counts()["last_attrs"] == P.LAUNCH_PDL
    k.set_launch_attrs(0)
    P.proteus_launch(k, (4,), (128,), [3.0, 500, 0, 0])
    assert P.testing_fake_counts()["last_attrs"] == 0


def stats():
    return P.proteus_cache_stats(0)


def test_cache_levels_and_staleness(fake):
    """misses/compiles/hits across levels, staleness, corruption."""
    K_ = 12
    fake["init"]()
    k = reg_daxpy()
    c0 = P.testing_fake_counts()["compiles"]
    for i in range(K_):
        P.proteus_launch(k, (8,), (256,), [float(i), 2048, 0, 0])
    s = stats()
    assert s["misses"] == K_ and s["compiles"] == K_ and s["mem_hits"] == 0
    assert s["entries"] == K_ and s["disk_bytes_written"] > 0
    for i in range(K_):
        P.proteus_launch(k, (8,), (256,), [float(i), 2048, 0, 0])
    s = stats()
    assert s["mem_hits"] == K_ and s["compiles"] == K_ and s["launches"] == 2 * K_
    # non-annotated args (pointers) do not create keys
    P.proteus_launch(k, (8,), (256,), [0.0, 2048, 1234, 5678])
    assert stats()["mem_hits"] == K_ + 1
    files = sorted(os.listdir(fake["dir"]))
    assert len(files) == K_ and all(re.fullmatch(r"cache-jit-[0-9a-f]{16}\.cubin", f) for f in files)
    # a new "process": the persistent level feeds the in-memory level (P@25500)
    P.proteus_finalize()
    fake["init"]()
    k = reg_daxpy()
    for i in range(K_):
        P.proteus_launch(k, (8,), (256,), [float(i), 2048, 0, 0])
    s = stats()
    assert s["disk_hits"] == K_ and s["compiles"] == 0 and s["misses"] == K_
    assert P.testing_fake_counts()["compiles"] == c0 + K_
    # corrupt one file: exactly one reject + one recompile, then it is rewritten
    P.proteus_finalize()
    victim = os.path.join(fake["dir"], files[3])
    data = bytearray(open(victim, "rb").read())
    data[-5] ^= 0xFF
    open(victim, "wb").write(bytes(data))
    fake["init"]()
    k = reg_daxpy()
    for i in range(K_):
        P.proteus_launch(k, (8,), (256,), [float(i), 2048, 0, 0])
    s = stats()
    assert s["disk_rejects"] == 1 and s["compiles"] == 1 and s["disk_hits"] == K_ - 1
    # a truncated file is rejected too
    P.proteus_finalize()
    open(victim, "wb").write(open(victim, "rb").read()[:40])
    fake["init"]()
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [3.0, 2048, 0, 0])
    P.proteus_launch(k, (8,), (256,), [4.0, 2048, 0, 0])
    s = stats()
    assert s["disk_rejects"] + s["disk_hits"] == 2 and s["compiles"] == s["disk_rejects"]
    # edited source -> new kernel_id -> K new misses, no stale hits (P@26005)
    P.proteus_finalize()
    fake["init"]()
    k2 = reg_daxpy(src=DAXPY_SRC + "// edited\n")
    for i in range(K_):
        P.proteus_launch(k2, (8,), (256,), [float(i), 2048, 0, 0])
    s = stats()
    assert s["compiles"] == K_ and s["disk_hits"] == 0


def test_grid_and_block_are_keyed(fake):
    fake["init"]()
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    P.proteus_launch(k, (16,), (256,), [1.0, 2048, 0, 0])
    P.proteus_launch(k, (8,), (128,), [1.0, 2048, 0, 0])
    P.proteus_launch(k, (8,), (128, 2), [1.0, 2048, 0, 0])
    assert stats()["compiles"] == 4
    c = P.testing_fake_counts()
    assert c["last_grid"] == (8, 1, 1) and c["last_block"] == (128, 2, 1)


def test_disk_disabled(fake):
    fake["init"](flags=P.F_RCF | P.F_LB | P.F_FOLD_DIMS)
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    assert not os.path.exists(fake["dir"]) or not os.listdir(fake["dir"])
    assert stats()["disk_bytes_written"] == 0


def test_compile_failure_falls_back_to_generic(fake):
    fake["init"]()
    P.testing_fake_control(True, 0)
    k = reg_daxpy(generic=GENERIC)
    g0 = P.testing_fake_counts()["generic_launches"]
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    s = stats()
    assert s["compile_failures"] == 1 and s["generic_launches"] == 2
    assert P.testing_fake_counts()["generic_launches"] == g0 + 2
    assert P.testing_fake_counts()["last_fn"] == GENERIC
    k2 = P.proteus_register_kernel("daxpy", DAXPY_SRC + "\n", DAXPY_TYPES, [1, 2])
    with pytest.raises(P.ProteusError) as e:
        P.proteus_launch(k2, (8,), (256,), [1.0, 2048, 0, 0])
    assert e.value.status == 4 and "injected" in str(e.value)


def test_async_launches_generic_while_compiling_and_dedupes(fake):
    fake["init"](async_workers=2)
    P.testing_fake_control(False, 300)
    k = reg_daxpy(generic=GENERIC)
    c0 = P.testing_fake_counts()
    for _ in range(5):
        P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])   # same key, in flight
    s = stats()
    assert s["generic_launches"] == 5 and s["misses"] == 1
    assert s["inflight"] == 1
    P.proteus_wait_idle()
    s = stats()
    assert s["inflight"] == 0 and s["compiles"] == 1
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    c1 = P.testing_fake_counts()
    assert c1["compiles"] - c0["compiles"] == 1
    assert c1["spec_launches"] - c0["spec_launches"] == 1
    assert c1["last_fn"] != GENERIC
    assert stats()["mem_hits"] == 1


def test_async_without_generic_compiles_synchronously(fake):
    fake["init"](async_workers=2)
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    s = stats()
    assert s["compiles"] == 1 and s["generic_launches"] == 0 and s["inflight"] == 0


def test_concurrent_launches_are_consistent(fake):
    fake["init"](async_workers=3)
    P.testing_fake_control(False, 5)
    k = reg_daxpy(generic=GENERIC)
    nkeys, nthreads, reps = 20, 8, 60
    errs = []

    def run(t):
        try:
            for r in range(reps):
                P.proteus_launch(k, (8,), (256,), [float((r + t) % nkeys), 2048, 0, 0])
        except Exception as e:   # pragma: no cover
            errs.append(e)

    th = [threading.Thread(target=run, args=(t,)) for t in range(nthreads)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    P.proteus_wait_idle()
    assert not errs
    s = stats()
    assert s["misses"] == nkeys and s["compiles"] == nkeys
    assert s["launches"] == nthreads * reps
    assert s["mem_hits"] + s["generic_launches"] == nthreads * reps


def test_cache_clear(fake):
    fake["init"]()
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    P.proteus_cache_clear(0, memory=True, disk=True)
    assert stats()["entries"] == 0 and not os.listdir(fake["dir"])
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    assert stats()["compiles"] == 1


def test_env_config(monkeypatch, tmp_path):
    monkeypatch.setenv("PROTEUS_SPECIALIZE", "lb")
    monkeypatch.setenv("PROTEUS_ASYNC", "3")
    monkeypatch.setenv("PROTEUS_CACHE_DIR", str(tmp_path))
    monkeypatch.setenv("PROTEUS_DISK_CACHE", "0")
    c = P.proteus_config_default()
    assert c.flags & (P.F_RCF | P.F_LB | P.F_DISK) == P.F_LB
    assert c.async_workers == 3 and c.cache_dir.decode() == str(tmp_path)
    monkeypatch.setenv("PROTEUS_SPECIALIZE", "bogus")
    with pytest.raises(P.ProteusError):
        P.proteus_config_default()


def test_lru_eviction_in_memory(fake):
    """max_entries (NEXT-4, the paper's planned LRU, P@26536-27373): the least recently
    launched specializations leave the in-memory level; a re-launch is served by disk."""
    fake["init"](max_entries=3)
    k = reg_daxpy()
    for a in (1.0, 2.0, 3.0):
        P.proteus_launch(k, (8,), (256,), [a, 2048, 0, 0])
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])        # 1.0 is now most recent
    P.proteus_launch(k, (8,), (256,), [4.0, 2048, 0, 0])        # evicts 2.0 (LRU)
    s = stats()
    assert s["entries"] == 3 and s["evictions"] == 1 and s["compiles"] == 4
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])        # still resident
    assert stats()["mem_hits"] == 2
    P.proteus_launch(k, (8,), (256,), [2.0, 2048, 0, 0])        # evicted -> disk hit
    s = stats()
    assert s["disk_hits"] == 1 and s["compiles"] == 4 and s["entries"] == 3
    assert s["evictions"] == 2


def test_disk_size_cap_deletes_least_recently_used(fake):
    fake["init"]()
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    one = os.path.getsize(os.path.join(fake["dir"], os.listdir(fake["dir"])[0]))
    P.proteus_finalize()
    fake["init"](max_disk_bytes=3 * one + one // 2)              # room for 3 files
    k = reg_daxpy()
    for a in (2.0, 3.0, 4.0, 5.0):
        P.proteus_launch(k, (8,), (256,), [a, 2048, 0, 0])
        time.sleep(0.01)
    s = stats()
    assert len(os.listdir(fake["dir"])) == 3 and s["disk_evictions"] == 2
    P.proteus_finalize()
    fake["init"]()
    k = reg_daxpy()
    for a in (3.0, 4.0, 5.0):                                      # the newest three survive
        P.proteus_launch(k, (8,), (256,), [a, 2048, 0, 0])
    assert stats()["disk_hits"] == 3


def test_lru_eviction_under_concurrency(fake):
    fake["init"](max_entries=4, async_workers=2)
    P.testing_fake_control(False, 2)
    k = reg_daxpy(generic=GENERIC)
    errs = []

    def run(t):
        try:
            for r in range(80):
                P.proteus_launch(k, (8,), (256,), [float((r * 7 + t) % 13), 2048, 0, 0])
        except Exception as e:   # pragma: no cover
            errs.append(e)

    th = [threading.Thread(target=run, args=(t,)) for t in range(6)]
    for t in th:
        t.start()
    for t in th:
        t.join()
    P.proteus_wait_idle()
    assert not errs
    s = stats()
    assert s["entries"] <= 4 and s["launches"] == 6 * 80 and s["evictions"] > 0


def test_bound_globals_enter_key_and_prelude(fake):
    """Device-global linking (P@19299-21805): bindings are keyed (matching the Python key
    oracle's G section) and every bound global is redirected in the prelude; an unbound
    kernel's key has no G section."""
    fake["init"]()
    k = reg_daxpy()
    kid, _, _ = k.info()
    args = [2.0, 64, 0, 0]
    kb0, _ = P.proteus_key(k, (1,), (64,), args)
    assert kb0 == K.key_bytes(kid, 7, 1, [(1, K.F64, 2.0), (2, K.I64, 64)], (1, 1, 1), (64, 1, 1))
    k.bind_global("zeta", 0x7F0000001000)
    k.bind_global("alpha", 0x7F0000002000)
    kb, h = P.proteus_key(k, (1,), (64,), args)
    want = K.key_bytes(kid, 7, 1, [(1, K.F64, 2.0), (2, K.I64, 64)], (1, 1, 1), (64, 1, 1),
                       {"zeta": 0x7F0000001000, "alpha": 0x7F0000002000})
    assert kb == want and h == K.key_hash(want) and kb[:len(kb0)] == kb0
    src = P.proteus_specialized_source(k, (1,), (64,), args)
    assert ("#define PROTEUS_GLOBAL_alpha (*reinterpret_cast<decltype(&alpha)>"
            "(0x00007f0000002000ull))") in src
    assert src.index("PROTEUS_GLOBAL_alpha") < src.index("PROTEUS_GLOBAL_zeta")
    k.bind_global("zeta", 0x7F0000003000)          # rebinding replaces the address
    assert P.proteus_key(k, (1,), (64,), args)[0] == K.key_bytes(
        kid, 7, 1, [(1, K.F64, 2.0), (2, K.I64, 64)], (1, 1, 1), (64, 1, 1),
        {"zeta": 0x7F0000003000, "alpha": 0x7F0000002000})
    for bad in ("", "9lives", "a-b", "x y", "é"):
        with pytest.raises(P.ProteusError) as e:
            k.bind_global(bad, 0x1000)
        assert e.value.status == 1
    with pytest.raises(P.ProteusError):
        k.bind_global("ok", 0)


def test_memoised_hits_follow_the_cache(fake):
    """The per-thread hit memo (launch with the same annotated values and dims as the last
    hit of the kernel skips key build + hash + lookup) never outlives what it points at:
    other values, an LRU eviction, a cache_clear, a new minBlocks or a re-init all go
    back through the cache."""
    fake["init"](max_entries=1, cache_dir="")
    k = reg_daxpy()
    launch = lambda a, n=2048: P.proteus_launch(k, (8,), (256,), [a, n, 0, 0])
    launch(1.0)
    launch(1.0)                      # hit: fills the memo
    fn1 = P.testing_fake_counts()["last_fn"]
    launch(1.0)                      # memoised hit
    s = stats()
    assert (s["compiles"], s["mem_hits"]) == (1, 2)
    assert P.testing_fake_counts()["last_fn"] == fn1
    launch(2.0)                      # other value: miss, compile, evicts a = 1 (cap 1)
    assert stats()["compiles"] == 2 and stats()["evictions"] == 1
    assert P.testing_fake_counts()["last_fn"] != fn1
    launch(1.0)                      # memo points at the evicted entry: must recompile
    assert stats()["compiles"] == 3
    launch(1.0)
    launch(1.0)
    assert stats()["compiles"] == 3
    P.proteus_cache_clear(0, memory=True, disk=False)
    launch(1.0)                      # cleared: recompile
    assert stats()["compiles"] == 1  # counters were reset by the clear
    k.set_min_blocks(2)              # the key changes: a new specialization
    launch(1.0)
    assert stats()["compiles"] == 2
    launch(1.0, n=4096)              # other annotated N
    assert stats()["compiles"] == 3
    P.proteus_finalize()             # a new init may reuse the kernel / device addresses
    fake["init"](cache_dir="")
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [1.0, 2048, 0, 0])
    assert stats()["compiles"] == 1


def test_processes_share_one_cache_dir(tmp_path):
    """R-cache-1: 6 processes (as the 8 ranks of one box) fill ONE cache dir with the same
    K keys concurrently (temp file + rename; a per-key claim file makes the other ranks
    wait for the file instead of compiling the key again): every key is compiled exactly
    once over all processes, the dir then holds exactly K valid entries and no temp or
    claim files, and a fresh process serves all K from disk, 0 compiles."""
    import json
    import subprocess
    import sys
    d = str(tmp_path / "shared")
    K_ = 40
    procs = [subprocess.Popen([sys.executable, os.path.join(ROOT, "tests", "disk_worker.py"), d,
                               str(K_), str(r)], stdout=subprocess.PIPE, text=True)
             for r in range(6)]
    outs = [json.loads(p.communicate(timeout=300)[0].strip().splitlines()[-1]) for p in procs]
    assert all(p.returncode == 0 for p in procs)
    assert all(o["disk_rejects"] == 0 and o["misses"] == K_ for o in outs)
    assert all(o["compiles"] + o["disk_hits"] == K_ for o in outs)
    assert sum(o["compiles"] for o in outs) == K_, outs
    files = sorted(os.listdir(d))
    assert len(files) == K_, files[:5]
    assert all(re.fullmatch(r"cache-jit-[0-9a-f]{16}\.cubin", f) for f in files)
    last = subprocess.run([sys.executable, os.path.join(ROOT, "tests", "disk_worker.py"), d,
                           str(K_), "0"], capture_output=True, text=True, timeout=300)
    o = json.loads(last.stdout.strip().splitlines()[-1])
    assert o["compiles"] == 0 and o["disk_hits"] == K_ and o["disk_rejects"] == 0


def test_prefetch_all_compiles_concurrently(fake):
    """workloads.prefetch_all: the specializations of several launches are compiled by
    concurrent proteus_get_specialization calls (4 keys x 60 ms fake compile finish in well
    under 4 x 60 ms), and the launches that follow are in-memory hits."""
    from paper_conf_cgo_georgakoudispb25_b200 import workloads as W
    fake["init"]()
    P.testing_fake_control(False, 60)
    k = reg_daxpy()
    Ls = [W.Launch(k, (8,), (256,), [float(i), 2048, 0, 0]) for i in range(4)]
    t0 = time.perf_counter()
    W.prefetch_all(Ls)
    el = time.perf_counter() - t0
    assert stats()["compiles"] == 4 and el < 0.2, el
    for L in Ls:
        L.jit()
    s = stats()
    assert s["compiles"] == 4 and s["mem_hits"] == 4 and s["launches"] == 4


def test_cross_process_claim_wait_and_stale_takeover(fake, tmp_path):
    """A fresh claim file of another process makes a miss wait for that process's cubin
    (then a disk hit, no compile); a claim older than the stale limit is taken over."""
    import shutil
    import threading
    src_dir = str(tmp_path / "src")
    fake["init"](cache_dir=src_dir)
    reg_daxpy()
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [3.0, 2048, 0, 0])
    name = os.listdir(src_dir)[0]
    lock = name.replace(".cubin", ".lock")
    P.proteus_finalize()
    # (a) live claim: the "other rank" publishes the file after 0.3 s and drops the claim
    d = str(tmp_path / "shared")
    os.makedirs(d)
    open(os.path.join(d, lock), "w").close()

    def other_rank():
        time.sleep(0.3)
        shutil.copy(os.path.join(src_dir, name), os.path.join(d, name + ".tmp.x"))
        os.rename(os.path.join(d, name + ".tmp.x"), os.path.join(d, name))
        os.remove(os.path.join(d, lock))

    th = threading.Thread(target=other_rank)
    th.start()
    fake["init"](cache_dir=d)
    k = reg_daxpy()
    t0 = time.perf_counter()
    P.proteus_launch(k, (8,), (256,), [3.0, 2048, 0, 0])
    waited = time.perf_counter() - t0
    th.join()
    s = stats()
    assert s["compiles"] == 0 and s["disk_hits"] == 1 and waited >= 0.25, (s, waited)
    P.proteus_finalize()
    # (b) stale claim (a rank that died compiling): taken over at once, compiled here
    d2 = str(tmp_path / "stale")
    os.makedirs(d2)
    lp = os.path.join(d2, lock)
    open(lp, "w").close()
    old = time.time() - 600
    os.utime(lp, (old, old))
    fake["init"](cache_dir=d2)
    k = reg_daxpy()
    t0 = time.perf_counter()
    P.proteus_launch(k, (8,), (256,), [3.0, 2048, 0, 0])
    assert time.perf_counter() - t0 < 5.0
    s = stats()
    assert s["compiles"] == 1 and not os.path.exists(lp)
    assert os.path.exists(os.path.join(d2, name))
    P.proteus_finalize()
    # (c) a FRESH claim whose owner process is dead on this host (a rank killed while
    # compiling, job relaunched at once): taken over without waiting for the age limit,
    # and no temp or aside files are left behind
    import socket
    import subprocess
    import sys
    dead = subprocess.Popen([sys.executable, "-c", "pass"])
    dead.wait()
    d3 = str(tmp_path / "dead")
    os.makedirs(d3)
    lp3 = os.path.join(d3, lock)
    with open(lp3, "w") as f:
        f.write(f"{dead.pid} {socket.gethostname()} .x\n")
    fake["init"](cache_dir=d3)
    k = reg_daxpy()
    t0 = time.perf_counter()
    P.proteus_launch(k, (8,), (256,), [3.0, 2048, 0, 0])
    assert time.perf_counter() - t0 < 2.0
    s = stats()
    assert s["compiles"] == 1 and sorted(os.listdir(d3)) == [name], os.listdir(d3)
    P.proteus_finalize()
    # (d) a fresh claim of a LIVE process on this host (this test process) is respected
    d4 = str(tmp_path / "live")
    os.makedirs(d4)
    with open(os.path.join(d4, lock), "w") as f:
        f.write(f"{os.getpid()} {socket.gethostname()} .y\n")

    def publish_later():
        time.sleep(0.3)
        shutil.copy(os.path.join(src_dir, name), os.path.join(d4, name))
        os.remove(os.path.join(d4, lock))

    th = threading.Thread(target=publish_later)
    th.start()
    fake["init"](cache_dir=d4)
    k = reg_daxpy()
    P.proteus_launch(k, (8,), (256,), [3.0, 2048, 0, 0])
    th.join()
    s = stats()
    assert s["compiles"] == 0 and s["disk_hits"] == 1, s


def test_cache_clear_during_a_miss_never_double_unloads(fake):
    """a cache_clear while another thread's synchronous miss has loaded its
    module but not yet accounted it must leave that module to its owner: every loaded
    module is unloaded exactly once (no unload of a module that is not loaded), none leaks,
    and the launcher still runs its kernel."""
    import threading
    import time
    fake["init"]()
    k = reg_daxpy()
    P.testing_fake_control(False, 0, load_delay_ms=300)
    c0 = P.testing_fake_counts()
    errs = []

    def launcher(a):
        try:
            P.proteus_launch(k, (4,), (64,), [a, 1 << 20, 0, 0])
        except Exception as e:   # pragma: no cover
            errs.append(e)

    ts = [threading.Thread(target=launcher, args=(float(a),)) for a in (1.5, 2.5, 3.5)]
    for t in ts:
        t.start()
    time.sleep(0.1)                       # all three are inside the delayed load
    P.proteus_cache_clear(memory=True)
    for t in ts:
        t.join()
    P.testing_fake_control(False, 0, load_delay_ms=0)
    P.proteus_launch(k, (4,), (64,), [9.5, 1 << 20, 0, 0])   # a normal miss afterwards
    P.proteus_cache_clear(memory=True)
    c1 = P.testing_fake_counts()
    assert not errs, errs
    assert c1["bad_unloads"] == c0["bad_unloads"]
    assert c1["loads"] - c0["loads"] >= 4
    assert c1["live_modules"] == c0["live_modules"], c1     # nothing leaked
    assert c1["spec_launches"] - c0["spec_launches"] >= 4


def test_ir_mode_sources_cache_and_nan_fallback(fake):
    """PROTEUS_F_IR on the fake backend: the specialized source is the constants TU and the
    kernel TU (annotated values and grid dims as extern constants, block dims and launch
    bounds as literals); keys that differ in values or grid share ONE kernel IR compile
    (one per block shape), each key links once; a NaN value (no constant initializer
    keeps its payload) takes the source path; IR keys differ from source-path keys."""
    fake["init"](flags=P.MODES["ir"] | P.F_DISK)
    k = reg_daxpy()
    src = P.proteus_specialized_source(k, (8,), (256,), [2.0, 4096, 0, 0])
    consts, kernel = src.split("\n//@@proteus-ir-kernel@@\n")
    assert "extern __device__ const double proteus_a1 = (0x1p+1);" in consts
    assert "extern __device__ const long long proteus_a2 = (4096ll);" in consts
    assert "extern __device__ const unsigned proteus_gdx = 8u;" in consts
    assert "#define PROTEUS_A1_OR(x) (proteus_a1)" in kernel
    assert "#define PROTEUS_BDX 256u" in kernel and "__launch_bounds__(256, 1)" in kernel
    assert "#define daxpy daxpy__jit_ir" in kernel
    c0 = P.testing_fake_counts()
    for a, grid in ((2.0, 8), (3.0, 8), (3.0, 16), (float("inf"), 8)):
        P.proteus_launch(k, (grid,), (256,), [a, 4096, 0, 0])
    P.proteus_launch(k, (8,), (128,), [2.0, 4096, 0, 0])          # another block shape
    c1 = P.testing_fake_counts()
    assert c1["ir_compiles"] - c0["ir_compiles"] == 2 + 5       # 2 kernel IRs + 5 constants
    assert c1["links"] - c0["links"] == 5
    inf_src = P.proteus_specialized_source(k, (8,), (256,), [float("inf"), 4096, 0, 0])
    assert "proteus_a1 = __builtin_huge_val();" in inf_src
    nan_src = P.proteus_specialized_source(k, (8,), (256,), [float("nan"), 4096, 0, 0])
    assert "//@@proteus-ir-kernel@@" not in nan_src and "PROTEUS_A1_OR(x)" in nan_src
    P.proteus_launch(k, (8,), (256,), [float("nan"), 4096, 0, 0])
    assert P.testing_fake_counts()["links"] == c1["links"]        # source path: no link
    st = P.proteus_cache_stats()
    assert st["ir_compiles"] == 2 and st["compiles"] == 6
    key_ir = P.proteus_key(k, (8,), (256,), [2.0, 4096, 0, 0])
    P.proteus_finalize()
    fake["init"](flags=P.MODES["all"] | P.F_DISK)
    k = reg_daxpy()
    assert P.proteus_key(k, (8,), (256,), [2.0, 4096, 0, 0]) != key_ir


def test_prefetch_compiles_in_the_background(fake):
    """proteus_prefetch: returns at once while the compile runs on the worker pool (started
    on demand when async_workers == 0); a synchronous launch of that key then waits for it
    and launches the specialization (one miss, one compile); a second prefetch of the key is
    a no-op; in async mode a launch during the compile runs the generic kernel."""
    fake["init"]()
    P.testing_fake_control(False, 200)
    k = reg_daxpy(generic=GENERIC)
    args = [2.0, 4096, 0, 0]
    t0 = time.perf_counter()
    P.proteus_prefetch(k, (8,), (256,), args)
    P.proteus_prefetch(k, (8,), (256,), args)           # already compiling: no-op
    assert time.perf_counter() - t0 < 0.1
    c0 = P.testing_fake_counts()
    P.proteus_launch(k, (8,), (256,), args)             # waits for the background compile
    assert time.perf_counter() - t0 >= 0.19
    c1 = P.testing_fake_counts()
    assert c1["spec_launches"] == c0["spec_launches"] + 1 and c1["generic_launches"] == c0["generic_launches"]
    s = stats()
    assert s["misses"] == 1 and s["compiles"] == 1 and s["launches"] == 1
    P.proteus_finalize()
    fake["init"](async_workers=2)
    k = reg_daxpy(generic=GENERIC)
    P.proteus_prefetch(k, (8,), (256,), [3.0, 4096, 0, 0])
    P.proteus_launch(k, (8,), (256,), [3.0, 4096, 0, 0])   # compile still running
    assert P.testing_fake_counts()["last_fn"] == GENERIC
    P.proteus_wait_idle()
    P.proteus_launch(k, (8,), (256,), [3.0, 4096, 0, 0])
    assert P.testing_fake_counts()["last_fn"] != GENERIC
    assert stats()["compiles"] == 1
