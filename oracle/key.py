"""Python key oracle (TEST INFRASTRUCTURE ONLY): specialization key bytes and hash.

Independent of the C++ runtime (paper_conf_cgo_georgakoudispb25_b200/csrc/proteus/);
written from the layout in DESIGN.md §"Specialization key".

What is hashed follows PAPER.md:1 §3.3 "Code caching" (P@24205-24805): "(1) a unique
module identifier bound to source code, (2) the kernel's symbol, and (3) the runtime
values of specialized kernel arguments and launch bound values".  Readings:
  * module id -> kernel_id = FNV-1a-64(source 0 entry 0 options 0 toolkit 0 arch)
    (changes whenever the source changes: P@26005-26536)
  * values are keyed by their raw little-endian bits (so -0.0 != +0.0)
  * grid and block are both keyed (north_star), plus minBlocks and the mode flags
  * hash = FNV-1a-64 over the key bytes (the paper does not name its hash)

key = "PRTK" | u32 version=1 | u64 kernel_id | u32 flags | u32 minB | u8 n_annot |
      n_annot x (u8 idx(1-based) | u8 type | u8 size | raw[size]) |
      u32 gx gy gz bx by bz                              (all little-endian)
      [ "G" | u8 n_glob | n_glob x (u8 len | name | u64 address) ]   only if globals bound
  (device globals linked to the AOT storage, P@19299-21805: their addresses are folded
   into the code, so they are keyed; sorted by name)
"""
from __future__ import annotations

import struct

FNV_OFFSET = 0xCBF29CE484222325
FNV_PRIME = 0x100000001B3

# proteus_type codes (include/proteus.h)
I32, U32, I64, U64, F32, F64, PTR = 1, 2, 3, 4, 5, 6, 7
_FMT = {I32: "<i", U32: "<I", I64: "<q", U64: "<Q", F32: "<f", F64: "<d", PTR: "<Q"}
_SIZE = {I32: 4, U32: 4, I64: 8, U64: 8, F32: 4, F64: 8, PTR: 8}

# flags that enter the key (include/proteus.h)
F_RCF, F_LB, F_FOLD_DIMS, F_DISK = 1, 2, 4, 8
KEY_FLAG_MASK = F_RCF | F_LB | F_FOLD_DIMS


def fnv1a64(data: bytes) -> int:
    h = FNV_OFFSET
    for b in data:
        h ^= b
        h = (h * FNV_PRIME) & 0xFFFFFFFFFFFFFFFF
    return h


def kernel_id(source: str, entry: str, options: str, toolkit: str, arch: str) -> int:
    blob = b"\0".join(s.encode() for s in (source, entry, options, toolkit, arch))
    return fnv1a64(blob)


def raw_bits(typ: int, value) -> bytes:
    """Raw little-endian bytes of a value of proteus_type `typ`.

    `value` may already be bytes of the right size (e.g. a float bit pattern)."""
    if isinstance(value, (bytes, bytearray)):
        assert len(value) == _SIZE[typ]
        return bytes(value)
    return struct.pack(_FMT[typ], value)


def key_bytes(kid: int, flags: int, min_blocks: int, annotated, grid, block,
              globals_=None) -> bytes:
    """annotated: iterable of (idx_1based, type, value); sorted by idx here.
    globals_: {name: device address} of bound device globals (optional)."""
    ann = sorted(annotated, key=lambda a: a[0])
    out = bytearray(b"PRTK")
    out += struct.pack("<IQIIB", 1, kid, flags & KEY_FLAG_MASK, min_blocks, len(ann))
    for idx, typ, val in ann:
        raw = raw_bits(typ, val)
        out += struct.pack("<BBB", idx, typ, len(raw)) + raw
    out += struct.pack("<6I", *grid, *block)
    if globals_:
        out += b"G" + struct.pack("<B", len(globals_))
        for name in sorted(globals_):
            nb = name.encode()
            out += struct.pack("<B", len(nb)) + nb + struct.pack("<Q", globals_[name])
    return bytes(out)


def key_hash(key: bytes) -> int:
    return fnv1a64(key)


def cache_file_name(h: int) -> str:
    """Persistent cache entry name (P@25651 'cache-jit-<hash>.o'; ours holds a cubin)."""
    return "cache-jit-%016x.cubin" % h
