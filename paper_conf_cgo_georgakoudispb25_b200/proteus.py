"""Thin ctypes binding of libproteus (include/proteus.h).  Argument marshalling only.

Names mirror the C ABI: proteus_init, proteus_register_kernel, proteus_launch,
proteus_cache_stats, ...  Every failure raises ProteusError with the library's
message.  If libproteus.so is missing this module raises at import: there is no
fallback of any kind (run `python -c "import __graft_entry__ as g; g.build()"`).
"""
from __future__ import annotations

import ctypes
import os
import struct

_PKG = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_PKG, "libproteus.so")
AOT_PATH = os.path.join(_PKG, "libproteus_aot.so")
# CPU-test hooks (fake backend): a separate library on top of libproteus.so, loaded only
# when a testing_* function is called
TESTING_PATH = os.path.join(_PKG, "libproteus_testing.so")

# proteus_type
I32, U32, I64, U64, F32, F64, PTR, OPAQUE = 1, 2, 3, 4, 5, 6, 7, 8
# flags
F_RCF, F_LB, F_FOLD_DIMS, F_DISK, F_TRACE, F_LINEINFO, F_IR = 1, 2, 4, 8, 16, 32, 64
LAUNCH_PDL = 1   # proteus_kernel_set_launch_attrs: programmatic dependent launch
# the paper's None / LB / RCF / LB+RCF ablation (P@39538-40272); launch dims are folded
# with the argument values (RCF), so "none" is plain JIT with nothing folded
MODES = {"none": 0, "lb": F_LB, "rcf": F_RCF | F_FOLD_DIMS, "all": F_RCF | F_LB | F_FOLD_DIMS,
         # attribution of "all" (r02): launch bounds + folded launch dims only, or launch
         # bounds + folded argument values only
         "dims": F_LB | F_FOLD_DIMS, "values": F_LB | F_RCF,
         # NEXT-1: the same folding as "all", done at the IR level (kernel LTO-IR once per
         # kernel / block / minBlocks, per key a constants module + nvJitLink -lto)
         "ir": F_RCF | F_LB | F_FOLD_DIMS | F_IR}

STATUS = {0: "OK", 1: "E_INVALID", 2: "E_NOT_INIT", 3: "E_CUDA", 4: "E_COMPILE", 5: "E_IO",
          6: "E_NOMEM"}


class ProteusError(RuntimeError):
    def __init__(self, status, msg):
        super().__init__(f"proteus {STATUS.get(status, status)}: {msg}")
        self.status = status


class proteus_config(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("cache_dir", ctypes.c_char_p),
                ("flags", ctypes.c_uint), ("async_workers", ctypes.c_int),
                ("min_blocks_per_sm", ctypes.c_int), ("max_entries", ctypes.c_uint64),
                ("max_disk_bytes", ctypes.c_uint64)]


class proteus_cache_stats_t(ctypes.Structure):
    _fields_ = [(n, ctypes.c_uint64) for n in (
        "launches", "mem_hits", "disk_hits", "misses", "compiles", "compile_failures",
        "generic_launches", "inflight", "entries", "cubin_bytes", "disk_bytes_written",
        "disk_rejects")] + [(n, ctypes.c_double) for n in (
            "compile_ms_total", "compile_ms_max", "load_ms_total", "disk_write_ms_total")] + [
                (n, ctypes.c_uint64) for n in ("evictions", "disk_evictions", "ir_compiles")] + [
                    ("ir_ms_total", ctypes.c_double)]

    def as_dict(self):
        return {n: getattr(self, n) for n, _ in self._fields_}


class proteus_fake_counts_t(ctypes.Structure):
    _fields_ = [("compiles", ctypes.c_uint64), ("loads", ctypes.c_uint64),
                ("spec_launches", ctypes.c_uint64), ("generic_launches", ctypes.c_uint64),
                ("last_fn", ctypes.c_void_p), ("last_grid", ctypes.c_uint * 3),
                ("last_block", ctypes.c_uint * 3), ("last_shmem", ctypes.c_uint),
                ("last_attrs", ctypes.c_uint), ("unloads", ctypes.c_uint64),
                ("bad_unloads", ctypes.c_uint64), ("live_modules", ctypes.c_uint64),
                ("ir_compiles", ctypes.c_uint64), ("links", ctypes.c_uint64)]


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} is missing: build the native library first "
                          "(__graft_entry__.build()); there is no non-native fallback")
    L = ctypes.CDLL(LIB_PATH)
    u, i, vp, sz = ctypes.c_uint, ctypes.c_int, ctypes.c_void_p, ctypes.c_size_t
    S = ctypes.c_int
    dims = [u] * 6
    sig = {
        "proteus_config_default": ([ctypes.POINTER(proteus_config)], S),
        "proteus_init": ([ctypes.POINTER(proteus_config)], S),
        "proteus_register_kernel": ([ctypes.c_char_p, ctypes.c_char_p, ctypes.c_char_p,
                                     ctypes.POINTER(ctypes.c_int), i, ctypes.POINTER(ctypes.c_int),
                                     i, vp, ctypes.POINTER(vp)], S),
        "proteus_launch": ([vp, *dims, u, vp, ctypes.POINTER(vp)], S),
        "proteus_kernel_set_min_blocks": ([vp, i], S),
        "proteus_kernel_set_launch_attrs": ([vp, u], S),
        "proteus_kernel_bind_global": ([vp, ctypes.c_char_p, vp], S),
        "proteus_launch_aot": ([vp, *dims, u, vp, ctypes.POINTER(vp)], S),
        "proteus_cache_stats": ([i, ctypes.POINTER(proteus_cache_stats_t)], S),
        "proteus_cache_clear": ([i, i, i], S),
        "proteus_wait_idle": ([], S),
        "proteus_finalize": ([], S),
        "proteus_last_error": ([], ctypes.c_char_p),
        "proteus_kernel_info": ([vp, ctypes.POINTER(ctypes.c_uint64), ctypes.c_char_p, sz,
                                 ctypes.c_char_p, sz], S),
        "proteus_key": ([vp, *dims, ctypes.POINTER(vp), ctypes.c_char_p, sz,
                         ctypes.POINTER(sz), ctypes.POINTER(ctypes.c_uint64)], S),
        "proteus_specialized_source": ([vp, *dims, ctypes.POINTER(vp), ctypes.c_char_p, sz,
                                        ctypes.POINTER(sz)], S),
        "proteus_prefetch": ([vp, *dims, ctypes.POINTER(vp)], S),
        "proteus_get_specialization": ([vp, *dims, ctypes.POINTER(vp), ctypes.POINTER(vp),
                                        ctypes.POINTER(ctypes.c_int), ctypes.c_char_p, sz,
                                        ctypes.POINTER(sz)], S),
        "proteus_encode_tensor_map": ([vp, i, u, vp, ctypes.POINTER(ctypes.c_uint64),
                                       ctypes.POINTER(ctypes.c_uint64),
                                       ctypes.POINTER(ctypes.c_uint32)], S),
        "proteus_ipc_get_handle": ([vp, ctypes.c_char_p, ctypes.POINTER(ctypes.c_uint64)], S),
        "proteus_ipc_open_handle": ([ctypes.c_char_p, ctypes.POINTER(vp)], S),
        "proteus_ipc_close_handle": ([vp], S),
        "proteus_stream_write_u32": ([vp, vp, ctypes.c_uint32], S),
        "proteus_stream_wait_u32": ([vp, vp, ctypes.c_uint32], S),
    }
    for name, (argt, rest) in sig.items():
        f = getattr(L, name)
        f.argtypes = argt
        f.restype = rest
    return L


lib = _load()


def _check(status):
    if status != 0:
        raise ProteusError(status, lib.proteus_last_error().decode(errors="replace"))


# ------------------------------------------------------------------------------- API
def proteus_config_default() -> proteus_config:
    c = proteus_config()
    _check(lib.proteus_config_default(ctypes.byref(c)))
    return c


def proteus_init(device: int = -1, cache_dir: str | None = None, flags: int | None = None,
                 async_workers: int | None = None, min_blocks_per_sm: int | None = None,
                 mode: str | None = None, max_entries: int | None = None,
                 max_disk_bytes: int | None = None):
    """Initialise from proteus_config_default() (env) with explicit overrides."""
    c = proteus_config_default()
    c.device = device
    if cache_dir is not None:
        c.cache_dir = cache_dir.encode()
    if flags is not None:
        c.flags = flags
    if mode is not None:
        c.flags = (c.flags & ~(F_RCF | F_LB | F_FOLD_DIMS | F_IR)) | MODES[mode]
    if async_workers is not None:
        c.async_workers = async_workers
    if min_blocks_per_sm is not None:
        c.min_blocks_per_sm = min_blocks_per_sm
    if max_entries is not None:
        c.max_entries = max_entries
    if max_disk_bytes is not None:
        c.max_disk_bytes = max_disk_bytes
    _check(lib.proteus_init(ctypes.byref(c)))
    return c


def proteus_finalize():
    _check(lib.proteus_finalize())


def proteus_wait_idle():
    _check(lib.proteus_wait_idle())


def proteus_cache_stats(device: int = -1) -> dict:
    s = proteus_cache_stats_t()
    _check(lib.proteus_cache_stats(device, ctypes.byref(s)))
    return s.as_dict()


def proteus_cache_clear(device: int = -1, memory: bool = True, disk: bool = False):
    _check(lib.proteus_cache_clear(device, int(memory), int(disk)))


_CT = {I32: ctypes.c_int32, U32: ctypes.c_uint32, I64: ctypes.c_int64, U64: ctypes.c_uint64,
       F32: ctypes.c_float, F64: ctypes.c_double, PTR: ctypes.c_void_p}


class Kernel:
    """A registered kernel: owns the marshalling of Python values into void** args."""

    def __init__(self, handle, entry, types, annotated):
        self.handle = handle
        self.entry = entry
        self.types = list(types)
        self.annotated = list(annotated)

    def pack(self, args):
        """Python values (ints, floats, data_ptr ints, or ctypes objects) -> void**."""
        if len(args) != len(self.types):
            raise ValueError(f"{self.entry}: expected {len(self.types)} args, got {len(args)}")
        holders = []
        for t, a in zip(self.types, args):
            if isinstance(a, (ctypes._SimpleCData, ctypes.Structure, ctypes.Array)):
                holders.append(a)
            elif t == OPAQUE:
                raise TypeError(f"{self.entry}: OPAQUE args must be ctypes objects")
            else:
                holders.append(_CT[t](a))
        arr = (ctypes.c_void_p * len(holders))(*[ctypes.cast(ctypes.byref(h), ctypes.c_void_p)
                                                  for h in holders])
        return arr, holders

    def set_min_blocks(self, n: int):
        _check(lib.proteus_kernel_set_min_blocks(self.handle, n))

    def set_launch_attrs(self, attrs: int):
        """PROTEUS_LAUNCH_* bits for every later launch of this kernel (LAUNCH_PDL)."""
        _check(lib.proteus_kernel_set_launch_attrs(self.handle, attrs))

    def bind_global(self, name: str, dptr: int):
        """Link the source's device global `name` to the storage at dptr (keyed)."""
        _check(lib.proteus_kernel_bind_global(self.handle, name.encode(), ctypes.c_void_p(dptr)))

    def info(self):
        kid = ctypes.c_uint64()
        tk = ctypes.create_string_buffer(256)
        ar = ctypes.create_string_buffer(64)
        _check(lib.proteus_kernel_info(self.handle, ctypes.byref(kid), tk, 256, ar, 64))
        return kid.value, tk.value.decode(), ar.value.decode()


def proteus_register_kernel(entry: str, source: str, arg_types, annotated_idx,
                            generic_fn: int | None = None, options: str = "") -> Kernel:
    n = len(arg_types)
    types = (ctypes.c_int * max(n, 1))(*arg_types)
    ann = (ctypes.c_int * max(len(annotated_idx), 1))(*annotated_idx)
    h = ctypes.c_void_p()
    _check(lib.proteus_register_kernel(entry.encode(), source.encode(), options.encode(),
                                       types, n, ann, len(annotated_idx),
                                       ctypes.c_void_p(generic_fn or 0), ctypes.byref(h)))
    return Kernel(h, entry, arg_types, annotated_idx)


def _dims(grid, block):
    g = tuple(grid) + (1,) * (3 - len(grid))
    b = tuple(block) + (1,) * (3 - len(block))
    return (*g, *b)


def proteus_launch(k: Kernel, grid, block, args, shmem: int = 0, stream: int = 0):
    arr, _hold = k.pack(args)
    _check(lib.proteus_launch(k.handle, *_dims(grid, block), shmem, ctypes.c_void_p(stream), arr))


def proteus_launch_aot(k: Kernel, grid, block, args, shmem: int = 0, stream: int = 0):
    arr, _hold = k.pack(args)
    _check(lib.proteus_launch_aot(k.handle, *_dims(grid, block), shmem, ctypes.c_void_p(stream),
                                  arr))


def proteus_key(k: Kernel, grid, block, args):
    arr, _hold = k.pack(args)
    buf = ctypes.create_string_buffer(1024)
    n = ctypes.c_size_t()
    h = ctypes.c_uint64()
    _check(lib.proteus_key(k.handle, *_dims(grid, block), arr, buf, 1024, ctypes.byref(n),
                           ctypes.byref(h)))
    return buf.raw[:n.value], h.value


def proteus_specialized_source(k: Kernel, grid, block, args) -> str:
    arr, _hold = k.pack(args)
    n = ctypes.c_size_t()
    _check(lib.proteus_specialized_source(k.handle, *_dims(grid, block), arr, None, 0,
                                          ctypes.byref(n)))
    buf = ctypes.create_string_buffer(n.value + 1)
    _check(lib.proteus_specialized_source(k.handle, *_dims(grid, block), arr, buf, n.value + 1,
                                          ctypes.byref(n)))
    return buf.value.decode()


def proteus_prefetch(k: Kernel, grid, block, args):
    """Start compiling the specialization of this launch in the background (returns at
    once; proteus_wait_idle() waits for it)."""
    arr, _hold = k.pack(args)
    _check(lib.proteus_prefetch(k.handle, *_dims(grid, block), arr))


def proteus_get_specialization(k: Kernel, grid, block, args):
    """Compile/fetch without launching -> (CUfunction int, cubin bytes)."""
    arr, _hold = k.pack(args)
    fn = ctypes.c_void_p()
    st = ctypes.c_int()
    n = ctypes.c_size_t()
    status = lib.proteus_get_specialization(k.handle, *_dims(grid, block), arr, ctypes.byref(fn),
                                            ctypes.byref(st), None, 0, ctypes.byref(n))
    _check(status)
    buf = ctypes.create_string_buffer(n.value)
    _check(lib.proteus_get_specialization(k.handle, *_dims(grid, block), arr, ctypes.byref(fn),
                                          ctypes.byref(st), buf, n.value, ctypes.byref(n)))
    return fn.value, buf.raw[:n.value]


TMA_F64 = 8   # CUtensorMapDataType FLOAT64


def proteus_encode_tensor_map(elem_type: int, base: int, dims, strides, box):
    """-> a 64-B aligned ctypes (c_uint64 * 16) TMA descriptor, passable as an OPAQUE arg."""
    raw = (ctypes.c_uint8 * (128 + 64))()
    off = (-ctypes.addressof(raw)) % 64
    desc = (ctypes.c_uint64 * 16).from_buffer(raw, off)
    desc._keepalive = raw
    rank = len(dims)
    d = (ctypes.c_uint64 * rank)(*dims)
    st = (ctypes.c_uint64 * max(1, rank - 1))(*strides)
    bx = (ctypes.c_uint32 * rank)(*box)
    _check(lib.proteus_encode_tensor_map(ctypes.addressof(desc), elem_type, rank,
                                         ctypes.c_void_p(base), d, st, bx))
    return desc


# ------------------------------------------------- peer memory (fused stencil + halo)
def proteus_ipc_get_handle(dptr: int):
    """-> (64-byte IPC handle of the allocation holding dptr, offset of dptr in it)."""
    h = ctypes.create_string_buffer(64)
    off = ctypes.c_uint64()
    _check(lib.proteus_ipc_get_handle(ctypes.c_void_p(dptr), h, ctypes.byref(off)))
    return h.raw, off.value


def proteus_ipc_open_handle(handle: bytes) -> int:
    """Map another process's allocation; -> its base address in this process."""
    assert len(handle) == 64
    base = ctypes.c_void_p()
    _check(lib.proteus_ipc_open_handle(handle, ctypes.byref(base)))
    return base.value


def proteus_ipc_close_handle(base: int):
    _check(lib.proteus_ipc_close_handle(ctypes.c_void_p(base)))


def proteus_stream_write_u32(stream: int, dptr: int, value: int):
    _check(lib.proteus_stream_write_u32(ctypes.c_void_p(stream), ctypes.c_void_p(dptr),
                                        value & 0xFFFFFFFF))


def proteus_stream_wait_u32(stream: int, dptr: int, value: int):
    _check(lib.proteus_stream_wait_u32(ctypes.c_void_p(stream), ctypes.c_void_p(dptr),
                                       value & 0xFFFFFFFF))


# ------------------------------------------------------------------- testing hooks
_tlib = None


def _testing_lib():
    """libproteus_testing.so (include/proteus_testing.h), loaded on first use; it links the
    libproteus.so already loaded above, so both act on the same runtime."""
    global _tlib
    if _tlib is None:
        if not os.path.exists(TESTING_PATH):
            raise ImportError(f"{TESTING_PATH} is missing (built by __graft_entry__.build())")
        T = ctypes.CDLL(TESTING_PATH)
        i, S = ctypes.c_int, ctypes.c_int
        for name, argt in (("proteus_testing_use_fake_backend", [i]),
                           ("proteus_testing_fake_control", [i, i]),
                           ("proteus_testing_fake_load_delay", [i]),
                           ("proteus_testing_fake_counts", [ctypes.POINTER(proteus_fake_counts_t)])):
            f = getattr(T, name)
            f.argtypes = argt
            f.restype = S
        _tlib = T
    return _tlib


def testing_use_fake_backend(enable: int = 1):
    """Backend of the next proteus_init: 0 CUDA, 1 fake, 2 fake load/launch + real NVRTC.
    Selecting the CUDA backend needs no test library (it is the product default)."""
    if not enable and _tlib is None:
        return
    st = _testing_lib().proteus_testing_use_fake_backend(int(enable))
    if st != 0:
        raise ProteusError(st, "backend selection must precede proteus_init")


def testing_fake_control(fail_compile: bool = False, compile_delay_ms: int = 0,
                         load_delay_ms: int = 0):
    T = _testing_lib()
    _check(T.proteus_testing_fake_control(int(fail_compile), int(compile_delay_ms)))
    _check(T.proteus_testing_fake_load_delay(int(load_delay_ms)))


def testing_fake_counts() -> dict:
    c = proteus_fake_counts_t()
    _check(_testing_lib().proteus_testing_fake_counts(ctypes.byref(c)))
    return dict(compiles=c.compiles, loads=c.loads, spec_launches=c.spec_launches,
                generic_launches=c.generic_launches, last_fn=c.last_fn,
                last_grid=tuple(c.last_grid), last_block=tuple(c.last_block),
                last_shmem=c.last_shmem, last_attrs=c.last_attrs, unloads=c.unloads,
                bad_unloads=c.bad_unloads, live_modules=c.live_modules,
                ir_compiles=c.ir_compiles, links=c.links)


def f32_bits(x: float) -> int:
    return struct.unpack("<I", struct.pack("<f", x))[0]
