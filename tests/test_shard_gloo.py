"""Multi-process (world_size 2, gloo, CPU) tests of the proof-sharding host logic.

Each rank proves its shard with the CPU oracle (the CUDA path needs a GPU); the gathered result
must be byte-identical to the single-process batch -- the property bench.py relies on at N > 1.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from paper_conf_asplos_lucw0cz25_b200 import inputs, shard

K, D, B = 5, 2, 6
KEYS = ("round_evals", "challenges", "final_evals", "claims")


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    import oracle
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        first, count = shard.shard_range(B, world, rank)
        tabs = inputs.gen_tables(count, D, K, first_index=first)
        out = oracle.prove_batch(tabs, K, D, 0, inputs.DEFAULT_SEED, first, nthreads=1)
        outs = {k: torch.from_numpy(out[k].view(np.int64)) for k in KEYS}
        g = shard.gather_outputs(outs, dist, dst=0)
        t = shard.max_over_ranks(1.0 + rank, dist)
        digests = shard.gather_bytes(bytes.fromhex(shard.output_digest([outs[k] for k in KEYS])), dist)
        if rank == 0:
            q.put({"outs": {k: v.numpy() for k, v in g.items()}, "tmax": t, "ndig": len(digests)})
    finally:
        dist.destroy_process_group()


def test_shard_ranges_cover_batch():
    for Bt in (1, 7, 1024, 8192):
        for W in (1, 2, 3, 8):
            ranges = [shard.shard_range(Bt, W, r) for r in range(W)]
            assert sum(c for _, c in ranges) == Bt
            nxt = 0
            for f, c in ranges:
                assert f == nxt
                nxt = f + c
    assert shard.weak_range(1024, 3) == (3072, 1024)


@pytest.mark.timeout(300)
def test_two_rank_gloo_equals_single_process(orc):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    single = orc.prove_batch(inputs.gen_tables(B, D, K), K, D, 0, inputs.DEFAULT_SEED, 0, nthreads=2)
    for k in KEYS:
        assert np.array_equal(res["outs"][k].view(np.uint64), single[k]), k
    assert res["tmax"] == 2.0 and res["ndig"] == 2


def _gather_worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        first, count = shard.shard_range(7, world, rank)           # uneven shards: 3 / 2 / 2
        t = {"a": torch.arange(first * 4, (first + count) * 4, dtype=torch.int64).reshape(count, 4),
             "b": torch.full((count, 2), rank, dtype=torch.int64)}
        g = shard.gather_outputs(t, dist, dst=0)
        if rank == 0:
            q.put({k: v.numpy() for k, v in g.items()})
        else:
            assert g is None
    finally:
        dist.destroy_process_group()


@pytest.mark.timeout(300)
def test_gather_to_rank0_uneven_shards():
    """shard.gather_outputs: torch.distributed.gather to rank 0 only, shards of unequal size padded
    and trimmed, concatenated in rank order (the c5 strong-scaling gather)."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gather_worker, args=(r, 3, port, q)) for r in range(3)]
    for p in procs:
        p.start()
    res = q.get(timeout=240)
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert np.array_equal(res["a"], np.arange(28).reshape(7, 4))
    assert res["b"][:, 0].tolist() == [0, 0, 0, 1, 1, 2, 2]
