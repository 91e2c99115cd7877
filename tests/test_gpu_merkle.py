"""GPU parity of the batched Merkle-tree module against the CPU oracle.

Every digest is compared byte for byte (bit-exact): roots, and the full level-major node array
when it is requested.  Shapes cover every stage structure the planner produces: n = 0 (one block),
trees smaller than one thread's subtree, one CTA, several CTAs (two stages), and the shape where the
second stage is a single thread; both hash modes; device and host (pinned) inputs/outputs with
several loader waves; roots-only (scratch between stages) vs node arrays.
"""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")

from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs  # noqa: E402


@pytest.fixture(scope="module")
def mb():
    b = bzk.MerkleBuilder(0)
    yield b
    b.close()


def dev_blocks(B, n, first=0):
    t = torch.empty((B, 1 << n, 64), dtype=torch.uint8, device="cuda")
    bzk.bzk_generate_blocks(t, B, n, first)
    return t


def test_block_generator_matches_host_twin():
    for B, n, first in [(3, 0, 0), (2, 5, 7), (1, 12, 1000)]:
        t = dev_blocks(B, n, first)
        torch.cuda.synchronize()
        assert np.array_equal(t.cpu().numpy(), inputs.gen_blocks(B, n, first))


def check(orc, blocks_np, n, mode, roots, nodes):
    exp_roots, exp_nodes = orc.merkle_batch(blocks_np, n, mode, nodes=nodes is not None)
    got_roots = roots.cpu().numpy()
    assert np.array_equal(got_roots, exp_roots), "roots differ"
    if nodes is not None:
        got = nodes.cpu().numpy()
        bad = np.argwhere(np.any(got != exp_nodes, axis=-1))
        assert bad.size == 0, f"node mismatches at (tree, node) {bad[:8].tolist()}"


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("n", [0, 1, 2, 3, 4, 7, 9, 10, 11, 12, 13])
def test_merkle_sweep_device(mb, orc, mode, n):
    B = 3
    blocks = dev_blocks(B, n, first=n)
    roots, nodes = mb.build(blocks, n, mode)
    torch.cuda.synchronize()
    check(orc, blocks.cpu().numpy(), n, mode, roots, nodes)


@pytest.mark.parametrize("mode", [0, 1])
@pytest.mark.parametrize("n", [10, 11, 16])
def test_merkle_roots_only_uses_scratch(mb, orc, mode, n):
    B = 2
    blocks = dev_blocks(B, n, first=5)
    roots, _ = mb.build(blocks, n, mode, with_nodes=False)
    torch.cuda.synchronize()
    check(orc, blocks.cpu().numpy(), n, mode, roots, None)


def test_merkle_three_stages_and_sampled_paths(mb, orc):
    """n = 21: stages of 2^10, 2^10 and a single block; every root checked, leaves and paths sampled."""
    n, B = 21, 2
    blocks = dev_blocks(B, n, first=40)
    roots, nodes = mb.build(blocks, n, 0)
    torch.cuda.synchronize()
    bl = blocks.cpu().numpy()
    exp_roots, _ = orc.merkle_batch(bl, n, 0, nodes=False)
    assert np.array_equal(roots.cpu().numpy(), exp_roots)
    nd = nodes.cpu().numpy()
    rng = np.random.default_rng(1)
    for b in range(B):
        assert bytes(nd[b, -1]) == bytes(exp_roots[b])
        for x in list(rng.integers(0, 1 << n, 6)) + [0, (1 << n) - 1]:
            x = int(x)
            path = orc.merkle_path(nd[b], n, x)
            assert orc.merkle_verify_path(n, 0, bytes(bl[b, x]), x, path, bytes(exp_roots[b]))


@pytest.mark.parametrize("mode", [0, 1])
def test_merkle_host_memory_waves(orc, mode):
    """Pinned host blocks and outputs, small workspace -> several loader waves with D2H overlap."""
    n, B = 12, 11
    bl = inputs.gen_blocks(B, n, first_index=3)
    host = torch.from_numpy(bl).pin_memory()
    b = bzk.MerkleBuilder(0, workspace_limit=3 * (64 << n) * 2 + (1 << 20))
    try:
        roots, nodes = b.build(host, n, mode)
        check(orc, bl, n, mode, roots, nodes)
        # host in, device out
        r2 = torch.empty((B, 32), dtype=torch.uint8, device="cuda")
        n2 = torch.empty((B, (2 << n) - 1, 32), dtype=torch.uint8, device="cuda")
        b.build(host, n, mode, roots=r2, nodes=n2)
        torch.cuda.synchronize()
        check(orc, bl, n, mode, r2, n2)
    finally:
        b.close()


def test_merkle_batch_composition_invariance(mb):
    n = 11
    blocks = dev_blocks(9, n, first=0)
    r_all, n_all = mb.build(blocks, n, 1)
    r_sub, n_sub = mb.build(blocks[4:7].contiguous(), n, 1)
    torch.cuda.synchronize()
    assert torch.equal(r_all[4:7], r_sub) and torch.equal(n_all[4:7], n_sub)


def test_merkle_root_seeds_sumcheck(orc):
    """the final Merkle root seeds the sum-check challenges (the transcript seed)."""
    n = 8
    blocks = dev_blocks(1, n, first=77)
    mbl = bzk.MerkleBuilder(0)
    roots, _ = mbl.build(blocks, n, 1, with_nodes=False)
    torch.cuda.synchronize()
    seed = bytes(roots[0].cpu().numpy())
    k, d = 6, 2
    t_np = inputs.gen_tables(1, d, k, first_index=0)
    pr = bzk.Prover(0)
    out = pr.prove(torch.from_numpy(t_np.view(np.int64)).cuda(), k, d, seed=seed)
    torch.cuda.synchronize()
    exp = orc.prove(t_np[0], k, d, 0, seed, 0)
    assert np.array_equal(out["challenges"][0].cpu().numpy().view(np.uint64), exp["challenges"])
    pr.close()
    mbl.close()


def test_merkle_argument_errors(mb):
    blocks = dev_blocks(1, 4)
    roots = torch.empty((1, 32), dtype=torch.uint8, device="cuda")
    with pytest.raises(bzk.BzkError):
        bzk.bzk_merkle(mb.ctx, bzk.bzk_merkle_batch(31, 0, 0, 0, 1, blocks.data_ptr(), 0, 0, roots.data_ptr(), None))
    with pytest.raises(bzk.BzkError):
        bzk.bzk_merkle(mb.ctx, bzk.bzk_merkle_batch(4, 2, 0, 0, 1, blocks.data_ptr(), 0, 0, roots.data_ptr(), None))
    with pytest.raises(bzk.BzkError):
        bzk.bzk_merkle(mb.ctx, bzk.bzk_merkle_batch(4, 0, 0, 0, 0, blocks.data_ptr(), 0, 0, roots.data_ptr(), None))
    with pytest.raises(bzk.BzkError):   # misaligned device blocks
        bzk.bzk_merkle(mb.ctx, bzk.bzk_merkle_batch(3, 0, 0, 0, 1, blocks.data_ptr() + 16, 0, 0, roots.data_ptr(),
                                                    None))
