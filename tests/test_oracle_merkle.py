"""Pins for the Merkle-tree oracle (readings R17-R19 in DESIGN.md), -m "not gpu".

The oracle (oracle/oracle.c orc_merkle) is checked against things other than itself:
* the SHA-256 compression it uses, against hashlib through FIPS 180-4 padding (a single-block
  message's digest IS one compression of its padded block from the IV), and against a Python
  compression whose constants are derived from their definition (cube / square roots of primes);
* the FIPS-mode tree, node by node, against hashlib.sha256 of the concatenated children;
* the root, against the recursive definition root = H(root(left) || root(right));
* the relation between the modes: SHA-256(m) for a 64-byte m = compress(compress(IV, m), pad64);
* the hash count 2N - 1 and the level sizes N, N/2, ..., 1;
* P:97 "any change in the input data will alter the corresponding hash value and propagate up":
  one flipped bit changes exactly the n + 1 digests on the block's path;
* every authentication path verifies, and no path verifies for a wrong block or index;
* a golden file written by tests/golden/make_golden_merkle.py from oracle/ only.
"""
import hashlib
import os
import random
import struct

import numpy as np
import pytest

import oracle
from oracle.py import merkle as pym
from paper_conf_asplos_lucw0cz25_b200 import inputs

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")
FIPS_IV = [0x6A09E667, 0xBB67AE85, 0x3C6EF372, 0xA54FF53A, 0x510E527F, 0x9B05688C, 0x1F83D9AB, 0x5BE0CD19]


def test_derived_constants_match_fips_table():
    # FIPS 180-4 Sec. 4.2.2 first/last constants and Sec. 5.3.3 initial value, as printed there
    assert pym.K[0] == 0x428A2F98 and pym.K[1] == 0x71374491 and pym.K[63] == 0xC67178F2
    assert pym.IV == FIPS_IV


def test_python_compression_is_sha256_via_padding():
    rng = random.Random(1)
    for L in list(range(0, 130)) + [1000]:
        m = bytes(rng.randrange(256) for _ in range(L))
        assert pym.sha256_from_compress(m) == hashlib.sha256(m).digest()


def test_c_compression_single_block_messages_vs_hashlib():
    """digest(m) for |m| <= 55 is one compression of pad(m) from the IV (FIPS 180-4 Sec. 5.1, 6.2)."""
    rng = random.Random(2)
    for L in range(0, 56):
        m = bytes(rng.randrange(256) for _ in range(L))
        h = oracle.sha256_compress(FIPS_IV, pym.sha256_pad(m))
        assert struct.pack(">8I", *h) == hashlib.sha256(m).digest()


def test_c_compression_vs_python_arbitrary_states():
    rng = random.Random(3)
    for _ in range(200):
        st = [rng.getrandbits(32) for _ in range(8)]
        blk = bytes(rng.randrange(256) for _ in range(64))
        assert oracle.sha256_compress(st, blk) == pym.sha256_compress(st, blk)


def test_modes_relation_fips_is_compress_then_constant_pad_block():
    pad64 = pym.sha256_pad(b"\x00" * 64)[64:]          # the constant second block of a 64-byte message
    assert len(pad64) == 64 and pad64[0] == 0x80 and pad64[-2:] == b"\x02\x00"
    rng = random.Random(4)
    for _ in range(50):
        blk = bytes(rng.randrange(256) for _ in range(64))
        c1 = pym.H(blk, 0)
        full = struct.pack(">8I", *pym.sha256_compress(list(struct.unpack(">8I", c1)), pad64))
        assert full == pym.H(blk, 1) == hashlib.sha256(blk).digest()


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("n", [0, 1, 2, 3, 5, 7])
def test_root_and_levels_vs_recursive_definition(mode, n):
    blocks = inputs.gen_blocks(1, n, first_index=n)[0]
    root, nodes = oracle.merkle(blocks, n, mode)
    blist = [bytes(b) for b in blocks]
    assert root == pym.merkle_root_recursive(blist, mode)
    lv = pym.merkle_levels(blist, mode)
    # level-major layout, sizes N, N/2, ..., 1 and 2N - 1 digests in total
    assert [len(x) for x in lv] == [1 << (n - l) for l in range(n + 1)]
    assert nodes.shape == ((2 << n) - 1, 32)
    flat = [bytes(r) for r in nodes]
    assert flat == [d for level in lv for d in level]
    assert flat[-1] == root


def test_fips_mode_nodes_are_hashlib_of_children():
    n = 6
    blocks = inputs.gen_blocks(1, n, first_index=9)[0]
    _, nodes = oracle.merkle(blocks, n, 1)
    N = 1 << n
    for x in range(N):
        assert bytes(nodes[x]) == hashlib.sha256(bytes(blocks[x])).digest()
    off, cnt = 0, N
    while cnt > 1:
        for j in range(cnt // 2):
            kids = bytes(nodes[off + 2 * j]) + bytes(nodes[off + 2 * j + 1])
            assert bytes(nodes[off + cnt + j]) == hashlib.sha256(kids).digest()
        off += cnt
        cnt //= 2


@pytest.mark.parametrize("mode", [0, 1])
def test_single_bit_change_alters_exactly_the_path(mode):
    n = 6
    blocks = inputs.gen_blocks(1, n, first_index=3)[0].copy()
    root, nodes = oracle.merkle(blocks, n, mode)
    rng = random.Random(5)
    for _ in range(8):
        x, byte, bit = rng.randrange(1 << n), rng.randrange(64), rng.randrange(8)
        b2 = blocks.copy()
        b2[x, byte] ^= 1 << bit
        root2, nodes2 = oracle.merkle(b2, n, mode)
        assert root2 != root
        changed = {i for i in range(nodes.shape[0]) if bytes(nodes[i]) != bytes(nodes2[i])}
        path, off, cnt, y = set(), 0, 1 << n, x
        for _l in range(n + 1):
            path.add(off + y)
            off += cnt
            cnt //= 2
            y //= 2
        assert changed == path


@pytest.mark.parametrize("mode", [0, 1])
def test_authentication_paths(mode):
    n = 5
    blocks = inputs.gen_blocks(1, n, first_index=11)[0]
    root, nodes = oracle.merkle(blocks, n, mode)
    for x in range(1 << n):
        path = oracle.merkle_path(nodes, n, x)
        assert oracle.merkle_verify_path(n, mode, bytes(blocks[x]), x, path, root)
        assert not oracle.merkle_verify_path(n, mode, bytes(blocks[x ^ 1]), x, path, root)
        assert not oracle.merkle_verify_path(n, mode, bytes(blocks[x]), x ^ 2, path, root)


def test_batch_equals_single_trees():
    n, B = 4, 5
    blocks = inputs.gen_blocks(B, n, first_index=100)
    for mode in (0, 1):
        roots, nodes = oracle.merkle_batch(blocks, n, mode, nodes=True, nthreads=3)
        for b in range(B):
            r, nd = oracle.merkle(blocks[b], n, mode)
            assert bytes(roots[b]) == r and np.array_equal(nodes[b], nd)


def test_block_generator_is_deterministic_and_index_bound():
    a = inputs.gen_blocks(3, 3, first_index=7)
    b = inputs.gen_blocks(1, 3, first_index=8)
    assert a.shape == (3, 8, 64) and np.array_equal(a[1], b[0])
    assert not np.array_equal(a[0], a[1])
    # word 0 of block 0 of tree 7, LE64: splitmix64(7 << 36)
    w = int(inputs.splitmix64(np.array([7 << 36], dtype=np.uint64), inputs.MERKLE_DATA_SEED)[0])
    assert bytes(a[0, 0, :8]) == w.to_bytes(8, "little")


def test_golden_merkle_roots():
    rows = []
    with open(os.path.join(GOLDEN, "merkle_small.txt")) as f:
        rows = [ln.split() for ln in f if ln.strip() and not ln.startswith("#")]
    assert len(rows) >= 6
    for n_s, mode_s, idx_s, root_hex in rows:
        n, mode, idx = int(n_s), int(mode_s), int(idx_s)
        blocks = inputs.gen_blocks(1, n, first_index=idx)[0]
        root, _ = oracle.merkle(blocks, n, mode, nodes=False)
        assert root.hex() == root_hex
