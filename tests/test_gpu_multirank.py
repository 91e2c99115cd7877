"""The multi-rank bench path on the CUDA library: two ranks launched by torchrun, both
pinned to GPU 0 with the gloo backend (this image has one GPU; NCCL needs distinct devices).  Each rank
proves its shard with the CUDA kernels, rank 0 gathers every proof and checks each one against the
CPU oracle's golden digests (tests/golden/c5_proof_digests.txt): weak scaling (c2 shape, 64 proofs per
rank) and strong scaling (c5 shape, 256 proofs split 128 / 128 in waves of 64)."""
import json
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

torch = pytest.importorskip("torch")
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


@pytest.mark.parametrize("cfg,extra,total", [("c2", ["--batch", "64"], 128),
                                             ("c5", ["--batch", "256", "--wave", "64"], 256)])
def test_two_ranks_gather_and_golden(cfg, extra, total):
    env = dict(os.environ, BZK_BENCH_DEVICE="0", BZK_DIST_BACKEND="gloo")
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node", "2", "--master-addr",
           "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"), "--gpus", "2", "--config", cfg,
           "--steps", "1", "--warmup", "3", "--no-e2e", "--no-cpu", *extra]
    r = subprocess.run(cmd, env=env, capture_output=True, text=True, timeout=900, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([ln for ln in r.stdout.splitlines() if ln.startswith("{")][-1])
    assert line["n_gpus"] == 2 and line["dist"]["world_size"] == 2
    assert line["proofs_gathered"]["proofs"] == total
    gold = line["golden_check"]
    assert gold["proofs_checked"] == total and gold["mismatches"] == 0, gold
    assert line["scaling"] == ("strong" if cfg == "c5" else "weak")
