"""Pins for the RNG, the hash and the Python key oracle (-m "not gpu")."""
import os
import struct

import numpy as np

import synthetic
from oracle import key as K

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def read_hex_fixture(name):
    out = bytearray()
    with open(os.path.join(GOLDEN, name)) as f:
        for line in f:
            line = line.split("#", 1)[0].strip()
            if line:
                out += bytes(int(t, 16) for t in line.split())
    return bytes(out)


def test_splitmix64_published_vectors(orc):
    # Vigna's splitmix64.c reference: seed 0 -> first output 0xe220a8397b1dcdaf;
    # seed 1234567 -> 6457827717110365317, 3203168211198807973, 9817491932198370423,
    # 4593380528125082431, 16408922859458223821.
    assert orc.splitmix64(0) == 0xE220A8397B1DCDAF
    g = 0x9E3779B97F4A7C15
    want = [6457827717110365317, 3203168211198807973, 9817491932198370423,
            4593380528125082431, 16408922859458223821]
    got = [orc.splitmix64((1234567 + k * g) % (1 << 64)) for k in range(5)]
    assert got == want
    # the numpy input generator is the same function
    xs = np.array([(1234567 + k * g) % (1 << 64) for k in range(5)], dtype=np.uint64)
    assert [int(v) for v in synthetic.splitmix64_next(xs)] == want


def test_rng_streams_agree_between_oracle_and_inputs(orc):
    idx = np.array([0, 1, 2, 12345, (1 << 40) - 1, 10 ** 7 - 1], dtype=np.uint64)
    for stream in (10, 20, 34, 35):
        a = synthetic.rng(stream, idx)
        b = [orc.rng(synthetic.S0, stream, int(i)) for i in idx]
        assert [int(x) for x in a] == b


def test_fnv1a64_published_vectors(orc):
    # Fowler/Noll/Vo FNV-1a 64-bit test vectors.
    for data, h in [(b"", 0xCBF29CE484222325), (b"a", 0xAF63DC4C8601EC8C),
                    (b"foobar", 0x85944171F73967E8)]:
        assert K.fnv1a64(data) == h
        assert orc.fnv1a64(data) == h


def test_key_layout_matches_hand_assembled_daxpy_fixture():
    want = read_hex_fixture("daxpy_key.txt")
    got = K.key_bytes(0x0123456789ABCDEF, K.F_RCF | K.F_LB | K.F_FOLD_DIMS, 1,
                      [(2, K.I64, 1 << 20), (1, K.F64, 2.0)], (1024, 1, 1), (256, 1, 1))
    assert got == want
    assert len(got) == 49 + (3 + 8) * 2


def test_key_float_identity_is_bitwise():
    a = K.key_bytes(1, 7, 1, [(1, K.F32, 0.0)], (1, 1, 1), (32, 1, 1))
    b = K.key_bytes(1, 7, 1, [(1, K.F32, -0.0)], (1, 1, 1), (32, 1, 1))
    assert a != b and K.key_hash(a) != K.key_hash(b)
    nan1 = struct.pack("<I", 0x7FC00000)
    nan2 = struct.pack("<I", 0x7FC00001)
    assert K.key_bytes(1, 7, 1, [(1, K.F32, nan1)], (1, 1, 1), (32, 1, 1)) != \
        K.key_bytes(1, 7, 1, [(1, K.F32, nan2)], (1, 1, 1), (32, 1, 1))


def test_key_changes_with_launch_shape_and_flags():
    base = K.key_bytes(9, 7, 1, [(1, K.I32, 5)], (10, 1, 1), (256, 1, 1))
    assert base != K.key_bytes(9, 7, 1, [(1, K.I32, 5)], (11, 1, 1), (256, 1, 1))
    assert base != K.key_bytes(9, 7, 1, [(1, K.I32, 5)], (10, 1, 1), (128, 1, 1))
    assert base != K.key_bytes(9, 3, 1, [(1, K.I32, 5)], (10, 1, 1), (256, 1, 1))
    assert base != K.key_bytes(9, 7, 2, [(1, K.I32, 5)], (10, 1, 1), (256, 1, 1))
    # the DISK flag does not enter the key
    assert base == K.key_bytes(9, 7 | K.F_DISK, 1, [(1, K.I32, 5)], (10, 1, 1), (256, 1, 1))


def test_kernel_id_is_bound_to_source():
    # P@26005-26536: a source change must change the module id (no stale hits)
    a = K.kernel_id("__global__ void k(){}", "k", "", "tk", "sm_100a")
    b = K.kernel_id("__global__ void k(){ }", "k", "", "tk", "sm_100a")
    c = K.kernel_id("__global__ void k(){}", "k", "-fmad=false", "tk", "sm_100a")
    assert len({a, b, c}) == 3


def test_listing1_annotation_indices_are_one_based():
    # Listing 1 (P@38745-39163) annotates 5,6,7,8,9,10,11,13 and footnote 5 (P@42483)
    # names them b1, b2, eps, grad_scale, step_size, time_step, vector_size, decay.
    proto = ["p", "m", "v", "g", "b1", "b2", "eps", "grad_scale", "step_size",
             "time_step", "vector_size", "mode", "decay"]
    picked = [proto[i - 1] for i in (5, 6, 7, 8, 9, 10, 11, 13)]
    assert picked == ["b1", "b2", "eps", "grad_scale", "step_size", "time_step",
                      "vector_size", "decay"]
    assert "mode" not in picked
