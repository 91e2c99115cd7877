#!/usr/bin/env python
"""bench.py -- batched sum-check proofs/s on B200 (BASELINE.json metric), one JSON line.

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config c2|c1|c3|m0] [--impl ours|reference]
    torchrun --nproc-per-node N bench.py --gpus N ...      (N > 1: one rank per GPU)

A "step" is one bzk_prove call over the whole batch (every round of every proof: round-1 eval,
fused fold+eval rounds, transcript hashing, on-chip tail, final fold).  Default workload =
BASELINE.json configs[1]: 1024 proofs of a degree-2 product of two multilinear tables with 2^20
BN254-Fr entries each (64 GiB of input, resident in HBM; PRESERVE mode so every step proves the
same tables).  Multi-GPU: rank r proves global proofs [r*B, (r+1)*B) (weak scaling, no data-path
collective; NCCL only gathers timings and output digests afterwards).

Timing: W untimed warm-up steps, then K steps bracketed by barrier + cuda synchronize, CUDA events
on the launch stream, max over ranks.  Inputs (64 GiB) are far larger than the 126 MB L2, so no
flush is needed between steps.
"""
from __future__ import annotations

import argparse
import json
import os
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from paper_conf_asplos_lucw0cz25_b200 import shard  # noqa: E402

METRIC = "sum-check proofs/s @2^20-entry tables, 1/2/4/8 B200; % of HBM/int roofline"

CONFIGS = {
    # name: (B per GPU, d, k, order, dist, description)
    "c2": (1024, 2, 20, 0, "uniform", "configs[1]: 1024 proofs x product of 2 multilinears, k=20, BN254 Fr, "
                                      "LSB order, tables resident in HBM"),
    "c1": (16, 2, 12, 0, "uniform", "configs[0]: 16 proofs x d=2, k=12 (oracle-size case)"),
    "c3": (256, 3, 22, 0, "uniform", "configs[2]: 256 GKR-layer-style proofs, degree-3 product f*g*h, k=22, "
                                     "consume mode"),
    "m0": (1024, 1, 20, 1, "uniform", "paper shape (Table 4 analogue): 1024 proofs x single multilinear (d=1), "
                                      "k=20, MSB order = Alg. 1 pairing"),
    "m0lit": (1024, 1, 20, 1, "uniform", "paper-literal Table 4 analogue: 1024 proofs x single multilinear (d=1), "
                                         "k=20, MSB = Alg. 1 pairing, challenges given (no Fiat-Shamir, P:111)"),
    "g2": (1024, 2, 20, 0, "gl", "NEXT-2 second field instance: 1024 proofs x product of 2 multilinears, k=20, "
                                 "Goldilocks p = 2^64 - 2^32 + 1 (8-byte elements: the HBM-bound regime)"),
    "mk20": (256, 0, 20, 0, "blocks", "NEXT-3 batched Merkle trees: 256 trees x 2^20 512-bit blocks (64 MiB per tree, "
                                     "P:295 Table 3 shape), H = one SHA-256 compression per block (P:97), every "
                                     "node level written to HBM"),
    "mk20f": (256, 1, 20, 0, "blocks", "NEXT-3 batched Merkle trees: 256 trees x 2^20 512-bit blocks, H = FIPS "
                                       "SHA-256 of the 64-byte block (two compressions), every node level written"),
    "enc20": (256, 0, 20, 0, "code", "NEXT-4 linear-time encoder: 256 messages x 2^20 BN254 Fr elements (P:320 Table 5 "
                                     "shape), Spielman-style rate-1/2 code, left degrees 10/20, base 64 (readings R21-R24)"),
    "c5": (8192, 2, 20, 0, "uniform", "configs[4]: 8192 proofs x product of 2 multilinears, k=20, BN254 Fr, sharded "
                                      "by proof across the GPUs (strong scaling), waves of <= 1024 proofs per GPU "
                                      "regenerated on the device between waves (untimed)"),
    "zk20": (64, 2, 20, 0, "chain", "NEXT-4 section-4 chain per proof (P:207-213): a 2^20-element input in S=4 segments "
                                    "of 2^18, each encoded (rate 1/2) and committed with a Merkle tree, root of roots, "
                                    "then a d=2, k=20 sum-check seeded with the final root (P:211)"),
    "c4": (64, 2, 16, 0, "vml", "configs[3]: verifiable-ML workload, VGG-16/CIFAR-10-shaped layer sum-checks (2 degree-2 "
                                "sum-checks per layer, k_l = ceil(log2 max(in_l, out_l))), streamed host->device"),
}

# VGG-16 on 32x32x3 CIFAR-10 images: 13 conv 3x3 layers + FC 512-512-10 (our reading of the shapes,
# DESIGN.md sec. 4): k_l = ceil(log2 max(in_l, out_l)); two degree-2 sum-checks per layer.
VGG16_K = [16, 16, 15, 15, 14, 14, 14, 13, 13, 13, 11, 11, 11, 9, 9, 9]

# integer roof: 148 SMs x 64 IMAD/clk/SM (fma-heavy pipe, B300_MICROARCH.md
# rt_SMSP = 2) x 1.965 GHz max SM clock; 272 IMAD per 256-bit Montgomery product (8-limb CIOS:
# 2 n^2 + n = 136 32x32 products, lo + hi each)
IMAD_PER_CLK_SM = 64
SMS = 148
IMAD_PER_MULMOD = 272


def init_pg_quiet(dist, backend, **kw):
    """init_process_group with the process's stdout pointed at stderr: NCCL prints its version banner
    (NCCL_DEBUG=VERSION) to fd 1 at communicator creation, and stdout carries only the JSON line"""
    sys.stdout.flush()
    saved = os.dup(1)
    try:
        os.dup2(2, 1)
        dist.init_process_group(backend, **kw)
    finally:
        sys.stdout.flush()
        os.dup2(saved, 1)
        os.close(saved)


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            m = json.load(f)
        return m.get("hbm_gbs", 6551.0), m.get("sm_max_mhz", 1965.0), "measured"
    except OSError:
        return 6650.0, 1965.0, "fallback"


def alg_mulmods(d: int, k: int, kind: str) -> int:
    """Algorithmic modular products per proof.

    round 1 (eval only): (d+1)(d-1) per pair (all points t = 0..d; the claim is unknown);
    fused round i >= 2: d * 2h fold products + d(d-1) per pair (g_i(1) = claim - g_i(0) derived);
    the tail kernel covers the remaining rounds plus the final fold."""
    tail_log = 8
    i0 = 1 if k - 1 <= tail_log else k - tail_log
    if kind == "round1":
        return (d + 1) * (d - 1) * (1 << (k - 1)) if i0 > 1 else 0
    if kind == "fused":
        return sum(2 * d * (1 << (k - i)) + d * (d - 1) * (1 << (k - i)) for i in range(2, i0))
    if kind == "total":
        return d * d * ((1 << k) - 1)
    raise ValueError(kind)


def alg_bytes_kind(d: int, k: int, kind: str, esz: int = 32) -> int:
    """Algorithmic HBM bytes per proof of a kernel kind: round 1 reads d 2^k x 32 B; a fused round
    i reads 4 d h_i x 32 B and writes 2 d h_i x 32 B (ping-pong)."""
    tail_log = 8
    i0 = 1 if k - 1 <= tail_log else k - tail_log
    if kind == "round1":
        return d * (1 << k) * esz
    return sum(6 * d * (1 << (k - i)) * esz for i in range(2, i0))


class ClockSampler:
    """nvidia-smi clocks + throttle reasons during the timed region (B200_PROFILING.md recipe)."""

    FIELDS = ("clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
              "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
              "clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.proc = None
        self.lines = []

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                                          "--format=csv,noheader,nounits", "-lms", "20"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
            # nvidia-smi needs a few hundred ms to print its first sample: wait for it (up to 3 s) so a
            # short timed region is still covered by samples
            t0 = time.time()
            while not self.lines and time.time() - t0 < 3.0 and self.proc.poll() is None:
                time.sleep(0.02)
            self.lines.clear()
        except OSError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            self.lines.append(line.strip())

    def __exit__(self, *a):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self):
        sm, mx, reasons = [], 0.0, set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for ln in self.lines:
            parts = [p.strip() for p in ln.split(",")]
            if len(parts) < 7:
                continue
            try:
                sm.append(float(parts[0]))
                mx = max(mx, float(parts[1]))
            except ValueError:
                continue
            for n, v in zip(names, parts[3:7]):
                if v.lower().startswith("active"):
                    reasons.add(n)
        sm.sort()
        return {"sm_mhz": sm[len(sm) // 2] if sm else None, "sm_max_mhz": mx or None,
                "reasons": sorted(reasons), "samples": len(sm)}


MERKLE_METRIC = "Merkle trees/s @2^20 512-bit blocks (NEXT-3, P:295 Table 3 shape)"
# ALU-pipe roof of one SHA-256 compression: the rotations/shifts (SHF) and the
# 3-input logic (LOP3) can only issue to the ALU pipe (B300_MICROARCH.md: IADD3/LOP3/SHF/PRMT on the
# alu pipe, rt_SMSP = 2 -> 64 lanes/clk/SM); the additions may go to the FMA pipe.  Per compression:
# 64 rounds x (6 SHF + 4 LOP3) + 48 schedule steps x (6 SHF + 2 LOP3) = 1024 ALU-only instructions.
ALU_PER_CLK_SM = 64
ALU_OPS_PER_COMPRESSION = 64 * 10 + 48 * 8


ENC_METRIC = "linear-time encodings/s @2^20 BN254 Fr elements (NEXT-4, P:320 Table 5 shape)"
# IMAD roof of an edge product: a 256 x 256-bit product accumulated unreduced = 64 IMAD.WIDE = 128 IMAD
# slots (the Montgomery reduction is amortised over a whole row: one per output element)
IMAD_PER_EDGE_PRODUCT = 128


def enc_traffic(cfg, B):
    """average DRAM bytes per k_spmv launch from profiles/traffic.json (ncu capture of one step)"""
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if not os.path.exists(tpath):
        return None
    with open(tpath) as f:
        tj = json.load(f)
    for e in (tj if isinstance(tj, list) else [tj]):
        if e.get("config") == cfg and e.get("kernel_kind") == "encoder_spmv" and e.get("batch") == B:
            return e["dram_bytes_per_launch"]
    return None


def enc_edges(code) -> int:
    return sum(int(a["row_ptr"][-1]) for a in code["A"]) + sum(int(b["row_ptr"][-1]) for b in code["B"]) + \
        int(code["G0"]["row_ptr"][-1])


def cpu_model() -> str:
    try:
        for ln in open("/proc/cpuinfo"):
            if ln.startswith("model name"):
                return ln.split(":", 1)[1].strip()
    except OSError:
        pass
    return "unknown"


def cpu_baseline(cfg, max_proofs=None):
    """The oracle as it stands on this box's host cores: a bounded sample of the same workload
    (default min(B, 4 x cores) proofs -- SURVEY.md 8(d) -- one per thread, all cores busy)."""
    import numpy as np  # noqa: F401

    import oracle
    from paper_conf_asplos_lucw0cz25_b200 import inputs
    B, d, k, order, dist, _ = CONFIGS[cfg]
    cores = len(os.sched_getaffinity(0))
    n = max(1, min(max_proofs or 4 * cores, B))
    threads = min(n, cores)
    oracle.build()
    if dist == "code":
        code = inputs.gen_code(k, 6)
        ms = inputs.gen_tables(n, 1, k, 0)[:, 0]
        t0 = time.perf_counter()
        oracle.encode_batch(code, ms, nthreads=threads)
        dt = time.perf_counter() - t0
        return {"value": n / dt, "unit": "codes/s", "cores": threads, "proofs": n, "kind": "oracle", "cpu_model": cpu_model(),
                "sample": f"{n} codewords of {cfg} (2^{k} elements) on {threads} threads, {dt:.1f} s wall"}
    if dist == "blocks":
        blocks = inputs.gen_blocks(n, k, 0)
        t0 = time.perf_counter()
        oracle.merkle_batch(blocks, k, d, nodes=True, nthreads=threads)
        dt = time.perf_counter() - t0
        return {"value": n / dt, "unit": "trees/s", "cores": threads, "proofs": n, "kind": "oracle", "cpu_model": cpu_model(),
                "sample": f"{n} trees of {cfg} (2^{k} blocks, hash mode {d}) on {threads} threads, {dt:.1f} s wall"}
    if dist == "gl":
        import concurrent.futures as cf
        tabs = inputs.gen_tables_gl(n, d, k, 0)
        t0 = time.perf_counter()
        with cf.ThreadPoolExecutor(threads) as ex:     # ctypes releases the GIL: one proof per thread
            list(ex.map(lambda b: oracle.gl_prove(tabs[b], k, d, order, inputs.DEFAULT_SEED, b), range(n)))
        dt = time.perf_counter() - t0
    elif cfg == "m0lit":
        import concurrent.futures as cf
        tabs = inputs.gen_tables(n, d, k, 0, dist)
        rs = [np.ascontiguousarray(inputs.gen_tables(1, 1, max(1, (k - 1).bit_length()), b, "uniform",
                                                     data_seed=0x5052470000000000)[0, 0, :k]) for b in range(n)]
        t0 = time.perf_counter()
        with cf.ThreadPoolExecutor(threads) as ex:     # the oracle's given-challenge prover (Alg. 1)
            list(ex.map(lambda b: oracle.prove_given(tabs[b], k, d, order, rs[b]), range(n)))
        dt = time.perf_counter() - t0
    else:
        tabs = inputs.gen_tables(n, d, k, 0, dist)
        t0 = time.perf_counter()
        oracle.prove_batch(tabs, k, d, order, inputs.DEFAULT_SEED, 0, nthreads=threads)
        dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "proofs/s", "cores": threads, "proofs": n, "kind": "oracle", "cpu_model": cpu_model(),
            "sample": f"{n} proofs of {cfg} (d={d}, k={k}) on {threads} threads, {dt:.1f} s wall"}


def run_reference(args, rank, world):
    """--impl reference: the CPU oracle (this tier's reference arm), rank 0 only."""
    if rank != 0:
        return
    B, d, k, order, dist, desc = CONFIGS[args.config]
    for _ in range(args.warmup):
        pass  # the oracle has no warm-up state; warm-up steps are not timed and not run
    times = []
    cb = None
    for _ in range(args.steps):
        cb = cpu_baseline(args.config, max_proofs=args.ref_proofs)
        times.append(cb["proofs"] / cb["value"])
    nproofs = cb["proofs"]
    value = nproofs * len(times) / sum(times)
    unit = cb["unit"]
    metric = {"blocks": MERKLE_METRIC, "code": ENC_METRIC}.get(dist, METRIC)
    line = {"impl": "reference", "metric": metric, "value": value,
            "unit": unit, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * sum(times) / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic", "config": {"workload": desc, "batch_sampled": nproofs, "d": d, "k": k},
            "cpu_baseline": {"value": value, "unit": unit, "cores": cb["cores"], "kind": "oracle",
                             "cpu_model": cb.get("cpu_model"), "sample": cb["sample"]},
            "e2e": {"value": value, "unit": unit, "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def run_vml(args, rank, world):
    """configs[3]: per image, 32 VGG-16-shaped sum-checks; tables in pinned host memory streamed
    through the library's loader (bzk_prove_ragged with host tables + host outputs)."""
    import collections

    import torch

    from paper_conf_asplos_lucw0cz25_b200 import bzk
    local = int(os.environ.get("LOCAL_RANK", 0))
    torch.cuda.set_device(local)
    images = args.batch or 64
    chunk = args.vml_chunk or images   # images per job group (default: one job per layer shape k)
    d = 2
    layers = collections.Counter(VGG16_K)
    ks = sorted(layers, reverse=True)
    per_img = {k: 2 * layers[k] for k in ks}                       # proofs per image with this k
    img0 = rank * images
    stream = torch.cuda.Stream()
    host, dev, outs_h, outs_d, base = {}, {}, {}, {}, {}
    off = 0
    for k in ks:
        n = images * per_img[k]
        base[k] = (1 << 20) * ks.index(k) + img0 * per_img[k]      # unique global proof indices per k
        t = torch.empty((n, d, 1 << k, 4), dtype=torch.int64, device="cuda")
        bzk.bzk_generate(t, n, d, k, base[k], "vml", stream=stream)
        stream.synchronize()
        host[k] = t.cpu().pin_memory()
        dev[k] = t
        outs_h[k] = bzk.Prover.alloc_outputs(n, k, d, device="cpu", pin=True)
        outs_d[k] = bzk.Prover.alloc_outputs(n, k, d)
        off += n
    prover = bzk.Prover(local)

    def jobs(tabs, outs, preserve):
        js = []
        for c in range(0, images, chunk):
            for k in ks:
                n0, n = c * per_img[k], min(chunk, images - c) * per_img[k]
                o = {key: v[n0:n0 + n] for key, v in outs[k].items()}
                js.append(prover.batch(tabs[k][n0:n0 + n], k, d, 0, None, base[k] + n0,
                                       bzk.BZK_F_PRESERVE_INPUT if preserve else 0, o, batch=n))
        return js

    hj = jobs(host, outs_h, False)
    dj = jobs(dev, outs_d, True)
    keep = prover._seed_bufs  # noqa: F841 (seed buffer referenced by the job structs)

    def timed(fn, reps):
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record(stream)
        for _ in range(reps):
            fn()
        e1.record(stream)
        stream.synchronize()
        return e0.elapsed_time(e1) / reps

    for _ in range(args.warmup):
        bzk.bzk_prove_ragged(prover.ctx, hj, stream)
    bzk.bzk_prove_ragged(prover.ctx, dj, stream)
    stream.synchronize()
    with ClockSampler(local) as clk:
        t_all = timed(lambda: bzk.bzk_prove_ragged(prover.ctx, hj, stream), args.steps)
    t_comp = timed(lambda: bzk.bzk_prove_ragged(prover.ctx, dj, stream), args.steps)
    scratch = {k: torch.empty_like(dev[k]) for k in ks}

    def copy_all():
        with torch.cuda.stream(stream):
            for k in ks:
                scratch[k].copy_(host[k], non_blocking=True)
    t_copy = timed(copy_all, args.steps)
    t_all = shard.max_over_ranks(t_all, None)
    same = all(torch.equal(outs_h[k][key], outs_d[k][key].cpu()) for k in ks for key in outs_h[k])
    h2d = sum(host[k].numel() * 8 for k in ks)
    d2h = sum(v.numel() * 8 for k in ks for v in outs_h[k].values())
    line = {"metric": "VML-shaped sum-check images/s (32 sum-checks per VGG-16/CIFAR-10 image)",
            "value": round(images * world / (t_all / 1000.0), 2), "unit": "images/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(t_all, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": CONFIGS["c4"][5], "images_per_gpu": images, "chunk_images": chunk,
                       "sumchecks_per_image": sum(per_img.values()), "k_per_layer": VGG16_K, "d": d,
                       "bytes_per_image": h2d // images},
            "sumchecks_per_s": round(images * sum(per_img.values()) / (t_all / 1000.0), 1),
            "overlap": {"T_copy_ms": round(t_copy, 3), "T_comp_ms": round(t_comp, 3), "T_overall_ms": round(t_all, 3),
                        "efficiency": round(max(t_copy, t_comp) / t_all, 4),
                        "h2d_GBps": round(h2d / (t_copy / 1000.0) / 1e9, 2)},
            "e2e": {"value": round(images * world / (t_all / 1000.0), 2), "unit": "images/s",
                    "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h},
            "host_vs_device_outputs_identical": bool(same), "clocks": clk.summary(),
            "context": "paper: 9.52 full VML proofs/s on GH200 (P:19, Table 11) -- whole proofs, not comparable"}
    if rank == 0:
        print(json.dumps(line), flush=True)
    prover.close()


def run_merkle(args, rank, world):
    """NEXT-3: batched Merkle trees (bzk_merkle).  A step builds every tree of the batch: all 2N - 1
    hashes per tree, every node level written to HBM (the tree is what a prover opens later)."""
    import torch

    from paper_conf_asplos_lucw0cz25_b200 import bzk
    local = int(os.environ.get("LOCAL_RANK", 0))
    if os.environ.get("BZK_BENCH_DEVICE") is not None:
        local = int(os.environ["BZK_BENCH_DEVICE"])
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        backend = os.environ.get("BZK_DIST_BACKEND", "nccl")
        if backend == "nccl":
            init_pg_quiet(dist, "nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    B, mode, n, _, _, desc = CONFIGS[args.config]
    if args.batch:
        B = args.batch
    if args.log_blocks is not None:
        n = args.log_blocks
        desc = desc.replace("2^20", "2^%d" % n)
    first, _ = shard.weak_range(B, rank)
    N = 1 << n
    stream = torch.cuda.Stream()
    blocks = torch.empty((B, N, 64), dtype=torch.uint8, device="cuda")
    bzk.bzk_generate_blocks(blocks, B, n, first, stream=stream)
    roots = torch.empty((B, 32), dtype=torch.uint8, device="cuda")
    nodes = torch.empty((B, 2 * N - 1, 32), dtype=torch.uint8, device="cuda")
    mb = bzk.MerkleBuilder(local)
    batch = mb.batch(blocks, n, mode, roots, nodes)

    def barrier():
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        bzk.bzk_merkle(mb.ctx, batch, stream)
    stream.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    bzk.bzk_launch_count(mb.ctx, reset=True)
    barrier()
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            ev[i][0].record(stream)
            bzk.bzk_merkle(mb.ctx, batch, stream)
            ev[i][1].record(stream)
        stream.synchronize()
        barrier()
    launches = bzk.bzk_launch_count(mb.ctx, reset=True)
    my_ms = float(sum(a.elapsed_time(b) for a, b in ev))
    # per-stage device time (roofline of the dominant stage kernel), outside the headline region
    bzk.bzk_profile_enable(mb.ctx, True)
    bzk.bzk_profile_read(mb.ctx, reset=True)
    for _ in range(args.steps):
        bzk.bzk_merkle(mb.ctx, batch, stream)
    prof = bzk.bzk_profile_read(mb.ctx, reset=True)
    bzk.bzk_profile_enable(mb.ctx, False)
    digest = shard.output_digest([roots.cpu()])
    max_ms = shard.max_over_ranks(my_ms, dist, device="cuda")
    digests = [x.hex() for x in shard.gather_bytes(bytes.fromhex(digest), dist, device="cuda")]
    ms_per_step = max_ms / args.steps
    value = B * world * args.steps / (max_ms / 1000.0)
    hbm_peak, sm_max_mhz, peak_src = peaks()
    hashes_per_tree = 2 * N - 1
    # FIPS mode: the second compression of every hash is the constant padding block, whose message
    # schedule is folded into constants (64 x (6 SHF + 4 LOP3) = 640 ALU-only instructions)
    alu_per_hash = ALU_OPS_PER_COMPRESSION + (64 * 10 if mode == 1 else 0)
    stage_ms, stage_cnt = prof["merkle_stage"]
    launches_per_step = max(1, stage_cnt // args.steps)
    # the dominant launch is stage 0 (all but 2^-10 of the hashes); its share of the step's compressions
    # is (2N - 1 - top) / (2N - 1); report the step as the conservative whole-step roof fraction
    achieved = B * hashes_per_tree / (stage_ms / args.steps / 1000.0) / 1e9
    peak = SMS * ALU_PER_CLK_SM * sm_max_mhz * 1e6 / alu_per_hash / 1e9
    bytes_step = B * (N * 64 + (2 * N - 1) * 32 + 32)
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic_merkle.json")
    if os.path.exists(tpath) and n == 20:
        # DRAM bytes of the dominant launch (stage 0) from one `ncu --set full` capture, scaled to B trees
        with open(tpath) as f:
            tj = json.load(f)
        if tj.get("config") == args.config:
            traffic = {"stage0_dram_bytes": int(tj["dram_bytes_per_launch"] * B / tj["batch"]),
                       "stage0_alg_bytes": int(tj["algorithmic_bytes_per_launch"] * B / tj["batch"]),
                       "source": tj["source"]}
    line = {"metric": MERKLE_METRIC, "value": round(value, 2), "unit": "trees/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": desc, "trees_per_gpu": B, "global_trees": B * world, "log_blocks": n,
                       "hash": "sha256-compress" if mode == 0 else "sha256-fips",
                       "l2": "inputs larger than L2 (%.0f GiB vs 126 MB); no flush" % (B * N * 64 / 2**30)},
            "gpu_launches": launches, "gpu_launches_per_step": launches / args.steps,
            "kernel_ms_per_step": {"merkle_stages": round(stage_ms / args.steps, 3),
                                   "launches_per_step": launches_per_step},
            "roofline": {"bound": "alu", "kernel": "k_merkle_stage (all stages of a step)",
                         "achieved": round(achieved, 3), "peak": round(peak, 3), "unit": "Ghash/s",
                         "frac": round(achieved / peak, 4), "traffic": traffic,
                         "alg_hashes_per_step": B * hashes_per_tree, "alu_ops_per_hash": alu_per_hash,
                         "peak_source": f"guide unit counts: {SMS} SMs x {ALU_PER_CLK_SM} ALU lanes/clk x "
                                        f"{sm_max_mhz:.0f} MHz ({peak_src} max clock) / "
                                        f"{alu_per_hash} ALU-only instructions per hash (SHF + LOP3 of the "
                                        "SHA-256 compression(s); additions may issue to the FMA pipe)",
                         "hbm_alg_frac": round(bytes_step / (ms_per_step / 1000.0) / 1e9 / hbm_peak, 4),
                         "hbm_peak_gbs": hbm_peak},
            "clocks": clk.summary(), "digest_rank0": digests[0], "digests_per_rank": len(digests),
            "context": "paper Table 3 (P:251-261): 6.536 trees/ms at 2^20 on GH200 as printed (unit garbled; "
                       "DESIGN.md R20)"}
    if not args.no_e2e:
        # e2e: pinned host blocks in, host roots + node arrays out, through bzk_merkle's loader
        Be = max(1, min(B, 32))
        host_b = blocks[:Be].cpu().pin_memory()
        hr = torch.empty((Be, 32), dtype=torch.uint8, pin_memory=True)
        hn = torch.empty((Be, 2 * N - 1, 32), dtype=torch.uint8, pin_memory=True)
        hb = mb.batch(host_b, n, mode, hr, hn)
        bzk.bzk_merkle(mb.ctx, hb, stream)
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            bzk.bzk_merkle(mb.ctx, hb, stream)
        e1.record(stream)
        stream.synchronize()
        e2e_ms = shard.max_over_ranks(e0.elapsed_time(e1), dist, device="cuda")
        same = torch.equal(hr, roots[:Be].cpu()) and torch.equal(hn[-1], nodes[Be - 1].cpu())
        line["e2e"] = {"value": round(Be * world * args.e2e_steps / (e2e_ms / 1000.0), 2), "unit": "trees/s",
                       "trees_per_gpu": Be, "h2d_bytes_per_step": int(host_b.numel()),
                       "d2h_bytes_per_step": int(hr.numel() + hn.numel()), "steps": args.e2e_steps,
                       "matches_device_run": bool(same),
                       "path": "bzk_merkle(blocks_mem=HOST pinned, outputs_mem=HOST): H2D waves and D2H of node "
                               "levels on two side streams overlapping compute (P:145-147)"}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(args.config)
    if rank == 0:
        print(json.dumps(line), flush=True)
    mb.close()
    if dist:
        dist.destroy_process_group()


def run_encoder(args, rank, world):
    """NEXT-4: batched linear-time encoding (bzk_encode), in place on [B][2n] codeword buffers."""
    import torch

    from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
    local = int(os.environ.get("LOCAL_RANK", 0))
    if os.environ.get("BZK_BENCH_DEVICE") is not None:
        local = int(os.environ["BZK_BENCH_DEVICE"])
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        backend = os.environ.get("BZK_DIST_BACKEND", "nccl")
        if backend == "nccl":
            init_pg_quiet(dist, "nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    B, _, log_n, _, _, desc = CONFIGS[args.config]
    if args.batch:
        B = args.batch
    if args.log_blocks is not None:
        log_n = args.log_blocks
        desc = desc.replace("2^20", "2^%d" % log_n)
    first, _ = shard.weak_range(B, rank)
    n = 1 << log_n
    t_setup = time.perf_counter()
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code, local)
    t_setup = time.perf_counter() - t_setup
    stream = torch.cuda.Stream()
    msgs = torch.empty((B, 1, n, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(msgs, B, 1, log_n, first, "uniform", stream=stream)
    stream.synchronize()
    codes = torch.empty((B, 2 * n, 4), dtype=torch.int64, device="cuda")

    def reset():
        codes[:, :n].copy_(msgs[:, 0])   # untimed: every step encodes the same messages

    def barrier():
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        reset()
        enc.encode(codes, stream=stream)
    stream.synchronize()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    bzk.bzk_launch_count(enc.ctx, reset=True)
    barrier()
    with ClockSampler(local) as clk:
        for i in range(args.steps):
            with torch.cuda.stream(stream):
                reset()
            ev[i][0].record(stream)
            enc.encode(codes, stream=stream)
            ev[i][1].record(stream)
        stream.synchronize()
        barrier()
    launches = bzk.bzk_launch_count(enc.ctx, reset=True)
    my_ms = float(sum(a.elapsed_time(b) for a, b in ev))
    bzk.bzk_profile_enable(enc.ctx, True)
    bzk.bzk_profile_read(enc.ctx, reset=True)
    for _ in range(args.steps):
        enc.encode(codes, stream=stream)
    prof = bzk.bzk_profile_read(enc.ctx, reset=True)
    bzk.bzk_profile_enable(enc.ctx, False)
    with torch.cuda.stream(stream):
        reset()
    enc.encode(codes, stream=stream)
    stream.synchronize()
    digest = shard.output_digest([codes[:, :, :].cpu()]) if B * n <= (1 << 24) else \
        shard.output_digest([codes[:, n:n + 1024].cpu()])
    max_ms = shard.max_over_ranks(my_ms, dist, device="cuda")
    digests = [x.hex() for x in shard.gather_bytes(bytes.fromhex(digest), dist, device="cuda")]
    ms_per_step = max_ms / args.steps
    value = B * world * args.steps / (max_ms / 1000.0)
    hbm_peak, sm_max_mhz, peak_src = peaks()
    edges = enc_edges(code)
    spmv_ms, spmv_cnt = prof["encoder_spmv"]
    achieved = B * edges / (spmv_ms / args.steps / 1000.0) / 1e9
    peak = SMS * IMAD_PER_CLK_SM * sm_max_mhz * 1e6 / IMAD_PER_EDGE_PRODUCT / 1e9
    wbytes = edges * 36
    line = {"metric": ENC_METRIC, "value": round(value, 2), "unit": "codes/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": desc, "codes_per_gpu": B, "global_codes": B * world, "log_n": log_n,
                       "levels": code["levels"], "edges_per_code": edges, "left_degrees": [inputs.ENC_C, inputs.ENC_D],
                       "l2": "codewords larger than L2 (%.0f GiB vs 126 MB); no flush" % (B * 2 * n * 32 / 2**30),
                       "setup_s": round(t_setup, 2)},
            "gpu_launches": launches, "gpu_launches_per_step": launches / args.steps,
            "kernel_ms_per_step": {"encoder_spmv": round(spmv_ms / args.steps, 3),
                                   "launches_per_step": spmv_cnt // max(1, args.steps)},
            "roofline": {"bound": "alu", "kernel": "k_spmv (all products of a step)", "achieved": round(achieved, 2),
                         "peak": round(peak, 2), "unit": "Gproduct/s", "frac": round(achieved / peak, 4),
                         "traffic": enc_traffic(args.config, B), "alg_products_per_step": B * edges,
                         "peak_source": f"guide unit counts: {SMS} SMs x {IMAD_PER_CLK_SM} IMAD/clk x {sm_max_mhz:.0f} "
                                        f"MHz ({peak_src} max clock) / {IMAD_PER_EDGE_PRODUCT} IMAD slots per "
                                        "256x256-bit edge product (reduction amortised per output element)",
                         "weights_bytes": wbytes, "hbm_peak_gbs": hbm_peak},
            "clocks": clk.summary(), "digest_rank0": digests[0], "digests_per_rank": len(digests),
            "context": "paper Table 5 (P:281-291): 0.726 codes/ms at 2^20 on GH200 as printed (parameters of "
                       "the paper's code unknown, R22)"}
    if not args.no_e2e:
        Be = max(1, min(B, 16))
        host = torch.empty((Be, 2 * n, 4), dtype=torch.int64, pin_memory=True)
        host[:, :n].copy_(msgs[:Be, 0])
        enc.encode(host)
        same = torch.equal(host, codes[:Be].cpu())
        barrier()
        t0 = time.perf_counter()
        for _ in range(args.e2e_steps):
            enc.encode(host)       # host buffer: H2D of the messages, D2H of the codewords inside
        torch.cuda.synchronize()
        wall = time.perf_counter() - t0
        e2e_s = shard.max_over_ranks(wall * 1000.0, dist, device="cuda") / 1000.0
        line["e2e"] = {"value": round(Be * world * args.e2e_steps / e2e_s, 2), "unit": "codes/s",
                       "codes_per_gpu": Be, "h2d_bytes_per_step": int(Be * n * 32),
                       "d2h_bytes_per_step": int(Be * 2 * n * 32), "steps": args.e2e_steps,
                       "matches_device_run": bool(same), "timing": "host wall clock around the synchronous call",
                       "path": "bzk_encode(codes_mem=HOST pinned): message H2D and codeword D2H waves on side "
                               "streams overlapping the encoding"}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(args.config, max_proofs=args.ref_proofs)
    if rank == 0:
        print(json.dumps(line), flush=True)
    enc.close()
    if dist:
        dist.destroy_process_group()

# ---------------------------------------------------------------- sum-check (configs c1, c2, c3, c5, m0, m0lit, g2)

GOLDEN_DIGESTS = os.path.join(ROOT, "tests", "golden", "c5_proof_digests.txt")
# IMAD-pipe slots of the kernels' products: a 32 x 32 -> 64-bit limb product is one
# IMAD.WIDE = 2 fma-heavy slots.  Fixed-multiplier fold (fixmul_lz): 64 + 18 products; unreduced
# 256 x 256-bit product into a 544-bit accumulator (mul_acc): 64; full Montgomery product: 136.
SLOT_FIXMUL, SLOT_MULACC, SLOT_MONT = 164, 128, 272
SLOT_TC_ROW = 185   # IMAD instructions in k_multi_tc's epilogue per output row (cuobjdump -sass)


def multi_passes(k: int, m_max: int = 3):
    """api.cu multi_passes: (K, m) of the known-challenge k_multi passes (d = 1, NEXT-1)."""
    tail_log = 8
    i0 = 1 if k - 1 <= tail_log else k - tail_log
    kt, out, K = k - i0 + 1, [], k
    while K > kt:
        m = min(m_max, K - kt)
        out.append((K, m))
        K -= m
    return out


def multi_tc_pass(K: int, m: int) -> bool:
    """api.cu multi_use_tc: three-round passes over >= 2^10 entries run k_multi_tc (tensor cores)"""
    return m == 3 and K >= 10 and os.environ.get("BZK_MULTI_TC", "1") != "0"


def tc_rounds(d: int, gl: bool = False) -> tuple[bool, bool]:
    """api.cu r1_use_tc / ftc_use: (round 1, fused rounds) sum the last product of every point on the
    u8 tensor cores (BN254 d = 2: k_round1_tc, k_fused_tc<2>; d = 3: k_fused_tc<3, ., FIRST>)"""
    if gl:
        return False, False
    on = lambda v: os.environ.get(v, "1") != "0"
    if d == 2:
        return on("BZK_R1_TC"), on("BZK_FUSED_TC")
    if d == 3:
        return on("BZK_D3_TC"), on("BZK_D3_TC")
    return False, False


def imad_slots(d: int, k: int, kind: str, gl: bool = False) -> int:
    """fma-heavy slots of the products one proof's launches of `kind` execute on the integer pipe (the
    kernels' arithmetic): round 1 sums d+1 points per pair, each (d-2) Montgomery
    products + 1 unreduced product; a fused round folds 2d entries per pair and sums d points (g(1)
    derived); a k_multi pass does one unreduced product per entry.  Where a kernel sums the last
    product of every point on the tensor cores (tc_rounds) that unreduced product leaves the count."""
    tail_log = 8
    i0 = 1 if k - 1 <= tail_log else k - tail_log
    tc1, tcf = tc_rounds(d, gl)
    point = 0 if d == 1 else (d - 2) * SLOT_MONT + SLOT_MULACC
    if kind == "round1":
        # k_fused_tc<3, ., 1>: x0(t) x1(t) is a quadratic in t, so its t = 2 value is derived from t = 0, 1, inf
        # and its x0(t) x1(t) are unreduced 512-bit products (64 limb products, SLOT_MULACC) summed on the
        # tensor cores
        if tc1 and d == 3:
            return d * SLOT_MULACC * (1 << (k - 1)) if i0 > 1 else 0
        return (d + 1) * (point - (SLOT_MULACC if tc1 else 0)) * (1 << (k - 1)) if i0 > 1 else 0
    if kind == "fused":
        # k_fused_tc<3, ., 0>: the x0(t) x1(t) products are unreduced 512-bit (64 limb products) too
        pf = (d - 2) * SLOT_MULACC if (tcf and d == 3) else point - (SLOT_MULACC if tcf else 0)
        return sum((2 * d * SLOT_FIXMUL + d * pf) * (1 << (k - i)) for i in range(2, i0))
    passes = multi_passes(k, int(os.environ.get("BZK_MULTI_M", "3")))
    if kind == "multi":
        return sum(SLOT_MULACC * (1 << K) for K, m in passes if not multi_tc_pass(K, m))
    if kind == "multi_tc":
        # k_multi_tc: the products run on the tensor cores; the integer pipe carries the epilogue
        # (column values -> 16 words, one 9-word REDC) once per output row
        return sum(SLOT_TC_ROW * (1 << (K - m)) for K, m in passes if multi_tc_pass(K, m))
    if kind == "small":
        # k_small: every round sums all d+1 points with (d-1) canonical Montgomery products each and
        # folds d entries per pair with one Montgomery product
        return sum(((d + 1) * (d - 1) + d) * SLOT_MONT * (1 << (k - i)) for i in range(1, k + 1))
    raise ValueError(kind)


def multi_bytes(k: int, tc: bool | None = None) -> int:
    """algorithmic HBM bytes per proof of the known-challenge passes (tc: only the k_multi_tc ones /
    only the k_multi ones / None: all): each reads its table once, writes 2^-m"""
    return sum(32 * ((1 << K) + (1 << (K - m))) for K, m in multi_passes(k, int(os.environ.get("BZK_MULTI_M", "3")))
               if tc is None or multi_tc_pass(K, m) == tc)


def proof_digests(out: dict) -> list:
    """per-proof digest (tests/golden/make_golden_c5.py): sha256(round_evals || challenges ||
    final_evals || claim)[:8], LE u64 limbs as the C ABI lays them out"""
    import hashlib
    arrs = [out[k_].cpu().numpy() for k_ in ("round_evals", "challenges", "final_evals", "claims")]
    res = []
    for b in range(arrs[0].shape[0]):
        h = hashlib.sha256()
        for a in arrs:
            h.update(a[b].tobytes())
        res.append(h.hexdigest()[:16])
    return res


def golden_check(digests: list, first: int, cfg: str) -> dict | None:
    """compare per-proof digests with the oracle-written golden file (d = 2, k = 20, LSB, uniform)"""
    if cfg not in ("c2", "c5") or not os.path.exists(GOLDEN_DIGESTS):
        return None
    gold = {}
    for ln in open(GOLDEN_DIGESTS):
        if ln.strip() and not ln.startswith("#"):
            i, dg = ln.split()
            gold[int(i)] = dg
    checked = [(first + n, dg) for n, dg in enumerate(digests) if first + n in gold]
    bad = [i for i, dg in checked if gold[i] != dg]
    return {"proofs_checked": len(checked), "proofs_total": len(digests), "mismatches": len(bad),
            "first_mismatch": bad[0] if bad else None,
            "source": "tests/golden/c5_proof_digests.txt (per-proof SHA-256 of the CPU oracle's outputs, "
                      "written by tests/golden/make_golden_c5.py from oracle/ only)"}


def run_sumcheck(args, rank, world, local):
    import torch

    from paper_conf_asplos_lucw0cz25_b200 import bzk
    torch.cuda.set_device(local)
    dist = None
    # BZK_DIST_FORCE=1 (under torchrun): the process group, the max-over-ranks timing and the gather of
    # the proofs to rank 0 run even at world size 1 (the NCCL path on a one-GPU box)
    if world > 1 or (os.environ.get("BZK_DIST_FORCE") == "1" and "RANK" in os.environ):
        import torch.distributed as dist
        backend = os.environ.get("BZK_DIST_BACKEND", "nccl")
        if backend == "nccl":
            init_pg_quiet(dist, "nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    B, d, k, order, gen_dist, desc = CONFIGS[args.config]
    if args.k is not None:                        # size sweeps (Table 4 analogue): override k
        desc = desc.replace("k=%d" % k, "k=%d" % args.k)
        k = args.k
    strong = args.config == "c5"
    if strong:
        # configs[4]: the GLOBAL batch is fixed; rank r proves the contiguous indices shard_range(B, W, r)
        # in waves of <= --wave proofs, each wave's tables regenerated on the device (untimed)
        global_B = args.batch or B
        first, count = shard.shard_range(global_B, world, rank)
        wave = max(1, min(count, args.wave))
        waves = [(first + w0, min(wave, count - w0)) for w0 in range(0, count, wave)]
    else:
        if args.batch:
            B = args.batch
        first, count = shard.weak_range(B, rank)
        global_B = B * world
        wave = count
        waves = [(first, count)]
    consume = args.config == "c3" or strong
    gl = gen_dist == "gl"
    esz = 8 if gl else 32
    flags = 0 if consume else bzk.BZK_F_PRESERVE_INPUT
    if gl:
        flags |= bzk.BZK_F_FIELD_GOLDILOCKS

    def tshape(n):
        return (n, d, 1 << k) if gl else (n, d, 1 << k, 4)
    given = args.config == "m0lit"
    if given:
        flags |= bzk.BZK_F_GIVEN_CHALLENGES
    stream = torch.cuda.Stream()
    tables = torch.empty(tshape(wave), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(tables, waves[0][1], d, k, waves[0][0], gen_dist, stream=stream)
    prover = bzk.Prover(local)
    out = (bzk.Prover.alloc_outputs_gl if gl else bzk.Prover.alloc_outputs)(count, k, d)
    if given:
        # pre-seeded challenges (the paper's PRG output): canonical values from the generator
        kk = max(1, (k - 1).bit_length())          # generator tables have 2^kk >= k entries
        g = torch.empty((count, 1, 1 << kk, 4), dtype=torch.int64, device="cuda")
        bzk.bzk_generate(g, count, 1, kk, first, "uniform", data_seed=0x5052470000000000, stream=stream)
        with torch.cuda.stream(stream):          # ordered after the generator on the same stream
            out["challenges"].copy_(g[:, 0, :k, :])
        stream.synchronize()

    def wave_out(w0, n):
        return {key: v[w0 - first:w0 - first + n] for key, v in out.items()}
    batches = [prover.batch(tables, k, d, order, None, w0, flags, wave_out(w0, n), batch=n) for w0, n in waves]
    seed_keep = list(prover._seed_bufs)  # noqa: F841 (the job structs point at this seed buffer)
    # weak scaling (one wave per rank): the whole step is captured once and replayed as a CUDA graph
    batch_g = None if strong else prover.batch(tables, k, d, order, None, first, flags | bzk.BZK_F_GRAPH, out)

    def regen(w0, n):
        bzk.bzk_generate(tables, n, d, k, w0, gen_dist, stream=stream)

    def barrier():
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        if batch_g is not None:
            if consume:
                regen(first, count)
            bzk.bzk_prove(prover.ctx, batch_g, stream)   # the first call captures the CUDA graph
        else:
            for (w0, n), b in zip(waves, batches):
                regen(w0, n)
                bzk.bzk_prove(prover.ctx, b, stream)
    stream.synchronize()

    def timed_region(use_graph, profile):
        calls = [(w0, n, batch_g if use_graph else b) for (w0, n), b in zip(waves, batches)]
        ev = [[(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in calls]
              for _ in range(args.steps)]
        bzk.bzk_profile_enable(prover.ctx, profile)
        bzk.bzk_profile_read(prover.ctx, reset=True)
        bzk.bzk_launch_count(prover.ctx, reset=True)
        barrier()
        with ClockSampler(local) as clk:
            for i in range(args.steps):
                for c, (w0, n, b) in enumerate(calls):
                    if consume:
                        regen(w0, n)                     # untimed: outside the events
                    ev[i][c][0].record(stream)
                    bzk.bzk_prove(prover.ctx, b, stream)
                    ev[i][c][1].record(stream)
            stream.synchronize()
            barrier()
        launches = bzk.bzk_launch_count(prover.ctx, reset=True)
        prof = bzk.bzk_profile_read(prover.ctx, reset=True)
        bzk.bzk_profile_enable(prover.ctx, False)
        return [sum(a.elapsed_time(b_) for a, b_ in row) for row in ev], launches, prof, clk.summary()

    # timed region 1 (the headline value): weak scaling replays the whole step as one CUDA graph; the
    # strong-scaling waves are launched call by call
    step_ms, launches, _, clocks = timed_region(batch_g is not None, False)
    # timed region 2 (roofline): the same steps launched kernel by kernel with CUDA events around
    # every launch on the launch stream (per-kernel device time)
    step_ms_prof, _, prof, _ = timed_region(False, True)
    my_ms = float(sum(step_ms))

    # ---------------- outputs: digests, gather to rank 0, golden check (outside the timed regions)
    keys = ("round_evals", "challenges", "final_evals", "claims")
    digest = shard.output_digest([out[key].cpu() for key in keys])
    max_ms = shard.max_over_ranks(my_ms, dist, device="cuda")
    digests = [x.hex() for x in shard.gather_bytes(bytes.fromhex(digest), dist, device="cuda")]
    gathered, gold = None, None
    if dist:
        # the proofs themselves are gathered to rank 0 over NCCL (NVLink) after the timed region
        # (north star: "NCCL is used only to gather proofs and timing"); rank 0 digests the global batch
        torch.cuda.synchronize()
        g0 = time.perf_counter()
        allp = shard.gather_outputs({k_: out[k_] for k_ in keys}, dist, dst=0)
        torch.cuda.synchronize()
        g_ms = (time.perf_counter() - g0) * 1000.0
        if rank == 0:
            gbytes = sum(v.numel() * v.element_size() for v in allp.values())
            gathered = {"proofs": int(allp["claims"].shape[0]), "bytes": int(gbytes), "ms": round(g_ms, 3),
                        "backend": dist.get_backend(), "collective": "gather to rank 0",
                        "global_digest": shard.output_digest([allp[k_].cpu() for k_ in keys])}
            if not gl and d == 2 and k == 20 and order == 0 and gen_dist == "uniform":
                gold = golden_check(proof_digests(allp), 0, args.config if strong else "c2")
    elif not gl and d == 2 and k == 20 and order == 0 and gen_dist == "uniform" and not given:
        gold = golden_check(proof_digests(out), first, args.config if strong else "c2")

    total_proofs = global_B * args.steps
    value = total_proofs / (max_ms / 1000.0)
    ms_per_step = max_ms / args.steps

    # ---------------- roofline of the dominant kernel
    hbm_peak, sm_max_mhz, peak_src = peaks()
    kinds = {"round1_eval": "round1", "fused_fold_eval": "fused", "multi_round": "multi", "small_cluster": "small",
             "multi_round_tc": "multi_tc"}
    dom = max(kinds, key=lambda n: prof[n][0])
    dom_ms, dom_cnt = prof[dom]
    launches_per_step = max(1, dom_cnt / args.steps)
    avg_launch_s = dom_ms / max(1, dom_cnt) / 1000.0
    slot_peak = SMS * IMAD_PER_CLK_SM * sm_max_mhz * 1e6          # fma-heavy slots / s
    slots_per_launch = imad_slots(d, k, kinds[dom], gl) * count / launches_per_step
    if kinds[dom] in ("multi", "multi_tc"):
        tc = kinds[dom] == "multi_tc"
        bytes_per_launch = multi_bytes(k, tc) * count / launches_per_step
        mulmods_per_launch = sum((1 << K) for K, m in multi_passes(k) if multi_tc_pass(K, m) == tc) * count / launches_per_step
    elif kinds[dom] == "small":
        bytes_per_launch = d * (1 << k) * esz * count / launches_per_step
        mulmods_per_launch = alg_mulmods(d, k, "total") * count / launches_per_step
    else:
        bytes_per_launch = alg_bytes_kind(d, k, kinds[dom], esz) * count / launches_per_step
        mulmods_per_launch = alg_mulmods(d, k, kinds[dom]) * count / launches_per_step
    ach_slots = slots_per_launch / avg_launch_s
    ach_gbs = bytes_per_launch / avg_launch_s / 1e9
    int_peak = slot_peak / IMAD_PER_MULMOD / 1e9                 # G mulmod/s (r01 unit, 272 slots)
    mulmod_rate = mulmods_per_launch / avg_launch_s / 1e9
    t_alu = slots_per_launch / slot_peak
    t_hbm = bytes_per_launch / (hbm_peak * 1e9)
    total_alg = alg_mulmods(d, k, "total") * count
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        # DRAM bytes per launch of the dominant kernel from one `ncu --set full` capture of the same
        # command, if it was taken on this workload and build
        with open(tpath) as f:
            tj = json.load(f)
        for e in (tj if isinstance(tj, list) else [tj]):
            if e.get("config") == args.config and e.get("kernel_kind") == dom and e.get("batch") == count:
                traffic = e["dram_bytes_per_launch"]
    if t_alu >= t_hbm and not gl:
        roofline = {"bound": "alu", "kernel": dom, "achieved": round(ach_slots / 1e12, 3),
                    "peak": round(slot_peak / 1e12, 3), "unit": "T IMAD-slot/s",
                    "frac": round(ach_slots / slot_peak, 4), "traffic": traffic,
                    "peak_source": f"guide unit counts: {SMS} SMs x {IMAD_PER_CLK_SM} fma-heavy slots/clk x "
                                   f"{sm_max_mhz:.0f} MHz ({peak_src} max clock); achieved = the kernel's product "
                                   "slots per launch on the integer pipe (fixmul fold 164, unreduced 256x256 product "
                                   "128, Montgomery product 272; products summed on the tensor cores excluded; "
                                   "DESIGN.md sec. 6) / CUDA-event launch time",
                    "tensor_core_sums": dict(zip(("round1", "fused"), tc_rounds(d, gl)))}
    else:
        roofline = {"bound": "hbm", "kernel": dom, "achieved": round(ach_gbs, 1), "peak": hbm_peak, "unit": "GB/s",
                    "frac": round(ach_gbs / hbm_peak, 4), "traffic": traffic,
                    "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_src}); achieved = algorithmic bytes per "
                                   "launch / CUDA-event launch time"}
    roofline.update({"alg_bytes_per_launch": bytes_per_launch, "imad_slots_per_launch": slots_per_launch,
                     "alu_time_at_peak_ms": round(t_alu * 1000, 4), "hbm_time_at_peak_ms": round(t_hbm * 1000, 4),
                     # (Goldilocks: 64-bit products, not the BN254 slot counts of imad_slots)
                     "imad_frac": None if gl else round(ach_slots / slot_peak, 4), "hbm_frac": round(ach_gbs / hbm_peak, 4),
                     "mulmod_equiv": {"achieved": round(mulmod_rate, 2), "peak": round(int_peak, 2),
                                      "unit": "Gmulmod/s (272-slot schoolbook unit, r01)",
                                      "frac": round(mulmod_rate / int_peak, 4)},
                     "step_mulmod_frac": round(total_alg / (ms_per_step / 1000.0) / 1e9 / int_peak, 4),
                     "step_hbm_alg_frac": round(d * (1 << k) * esz * count / (ms_per_step / 1000.0) / 1e9 / hbm_peak, 4),
                     "hbm_peak_gbs": hbm_peak})

    # both round kernels against the HBM roof (the dominant one is `roofline` above): round 1 reads
    # only, so it can exceed the copy-bandwidth peak
    per_kernel = {}
    for pname, pkind in (("round1_eval", "round1"), ("fused_fold_eval", "fused")):
        p_ms, p_cnt = prof.get(pname, (0.0, 0))
        if p_cnt and kinds[dom] in ("round1", "fused"):
            p_lps = max(1.0, p_cnt / args.steps)
            p_avg_s = p_ms / p_cnt / 1000.0
            p_bytes = alg_bytes_kind(d, k, pkind, esz) * count / p_lps
            per_kernel[pname] = {"launches_per_step": p_lps, "avg_launch_ms": round(p_avg_s * 1000.0, 4),
                                 "alg_bytes_per_launch": p_bytes, "achieved_gbs": round(p_bytes / p_avg_s / 1e9, 1),
                                 "hbm_frac": round(p_bytes / p_avg_s / 1e9 / hbm_peak, 4)}
    if per_kernel:
        roofline["per_kernel_hbm"] = per_kernel

    kernel_ms = {n: round(v[0] / args.steps, 3) for n, v in prof.items() if v[1]}
    line = {"metric": METRIC, "value": round(value, 2), "unit": "proofs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": True,
            "scaling": "strong" if strong else "weak", "vs_baseline": None, "dtype": "u64" if gl else "u32",
            "data": "synthetic",
            "config": {"workload": desc, "batch_per_gpu": count, "global_batch": global_B, "d": d, "k": k,
                       "order": "LSB" if order == 0 else "MSB", "field": "Goldilocks" if gl else "BN254 Fr",
                       "waves_per_gpu": len(waves), "wave_size": wave,
                       "l2": "inputs larger than L2 (%.0f GiB vs 126 MB); no flush" % (wave * d * (1 << k) * esz / 2**30)},
            "gpu_launches": launches, "gpu_launches_per_step": launches / args.steps,
            "kernel_ms_per_step": kernel_ms, "ms_per_step_kernel_by_kernel": round(sum(step_ms_prof) / args.steps, 3),
            "roofline": roofline, "clocks": clocks,
            "digest_rank0": digests[0], "digests_per_rank": len(digests)}
    if dist:
        line["dist"] = {"backend": dist.get_backend(), "world_size": dist.get_world_size(),
                        "nccl_version": ".".join(map(str, torch.cuda.nccl.version())) if dist.get_backend() == "nccl"
                        else None, "data_path_collectives": 0}
    if args.config in ("m0", "m0lit"):
        line["context"] = ("paper Table 4 (P:268-276): 5.622 proofs/ms at N = 2^20 on GH200 for Alg. 1 "
                           "(single multilinear, pre-seeded challenges); 1.461 / 2.884 / 10.610 / 19.753 at "
                           "2^22 / 2^21 / 2^19 / 2^18 -- other hardware, context only")
    if gathered:
        line["proofs_gathered"] = gathered
    if gold:
        line["golden_check"] = gold

    # ---------------- e2e: host (pinned) tables in, host outputs out, through bzk_prove
    if not args.no_e2e and args.config != "c3":
        del tables
        torch.cuda.empty_cache()
        # pinned host memory is shared by all ranks of the node: cap each rank's e2e batch at 40 % of
        # the available host memory / world (same metric, proofs/s, on a smaller host-resident batch)
        try:
            avail = os.sysconf("SC_AVPHYS_PAGES") * os.sysconf("SC_PAGE_SIZE")
        except (ValueError, OSError):
            avail = 1 << 40
        proof_bytes = d * (1 << k) * esz
        Be = int(max(1, min(wave, 0.4 * avail / world // proof_bytes)))
        host_t = torch.empty(tshape(Be), dtype=torch.int64, pin_memory=True)
        chunk = max(1, Be // 16)
        tmp = torch.empty(tshape(chunk), dtype=torch.int64, device="cuda")
        for c0 in range(0, Be, chunk):
            n = min(chunk, Be - c0)
            bzk.bzk_generate(tmp, n, d, k, first + c0, gen_dist, stream=stream)
            stream.synchronize()
            host_t[c0:c0 + n].copy_(tmp[:n])
        del tmp
        torch.cuda.empty_cache()
        out_h = (bzk.Prover.alloc_outputs_gl if gl else bzk.Prover.alloc_outputs)(Be, k, d, device="cpu", pin=True)
        if given:
            out_h["challenges"].copy_(out["challenges"][:Be])
        hb = prover.batch(host_t, k, d, order, None, first,
                          flags & (bzk.BZK_F_GIVEN_CHALLENGES | bzk.BZK_F_FIELD_GOLDILOCKS), out_h)
        bzk.bzk_prove(prover.ctx, hb, stream)   # warm-up (allocates staging)
        barrier()
        t0 = time.perf_counter()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(args.e2e_steps):
            bzk.bzk_prove(prover.ctx, hb, stream)   # host tables + host outputs: returns after D2H
        e1.record(stream)
        stream.synchronize()
        barrier()
        wall = time.perf_counter() - t0
        e2e_ms = shard.max_over_ranks(e0.elapsed_time(e1), dist, device="cuda")
        out_bytes = sum(v.numel() * 8 for v in out_h.values())
        same = all(torch.equal(out_h[key], out[key][:Be].cpu()) for key in out_h)
        line["e2e"] = {"value": round(Be * world * args.e2e_steps / (e2e_ms / 1000.0), 2), "unit": "proofs/s",
                       "batch_per_gpu": Be,
                       "h2d_bytes_per_step": int(host_t.numel() * 8), "d2h_bytes_per_step": int(out_bytes),
                       "steps": args.e2e_steps, "wall_s": round(wall, 3), "matches_device_run": bool(same),
                       "path": "bzk_prove(tables_mem=HOST pinned, outputs_mem=HOST): side-stream H2D waves "
                               "overlapping compute"}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(args.config, max_proofs=args.ref_proofs)
    if rank == 0:
        print(json.dumps(line), flush=True)
    prover.close()
    if dist:
        dist.destroy_process_group()


CHAIN_METRIC = "section-4 chain proofs/s (encode + Merkle commit + root of roots + sum-check, NEXT-4)"
CHAIN_SEGMENTS, CHAIN_LOG_N = 4, 18


def run_chain(args, rank, world, local):
    """NEXT-4: bzk_commit_prove over a batch -- per proof S segments encoded, each codeword committed
    (Merkle tree over its 64-byte blocks), the S roots combined by a root-of-roots tree, and a sum-check
    (d = 2, k = 20) seeded with the final root, all in one stream-ordered library call."""
    import torch

    from paper_conf_asplos_lucw0cz25_b200 import bzk, inputs
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        backend = os.environ.get("BZK_DIST_BACKEND", "nccl")
        if backend == "nccl":
            init_pg_quiet(dist, "nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    B, d, k, order, _, desc = CONFIGS[args.config]
    if args.batch:
        B = args.batch
    S, log_n = CHAIN_SEGMENTS, CHAIN_LOG_N
    n = 1 << log_n
    first, _ = shard.weak_range(B, rank)
    code = inputs.gen_code(log_n, 6)
    enc = bzk.Encoder(code, local)
    stream = torch.cuda.Stream()
    msgs = torch.empty((B * S, 1, n, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(msgs, B * S, 1, log_n, first * S, "uniform", data_seed=0x42415443485A4B53, stream=stream)
    codes = torch.empty((B, S, 2 * n, 4), dtype=torch.int64, device="cuda")
    roots = torch.empty((B, S, 32), dtype=torch.uint8, device="cuda")
    fin = torch.empty((B, 32), dtype=torch.uint8, device="cuda")
    tables = torch.empty((B, d, 1 << k, 4), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(tables, B, d, k, first, "uniform", stream=stream)
    out = bzk.Prover.alloc_outputs(B, k, d)
    stream.synchronize()
    commit = bzk.bzk_commit(S, bzk.BZK_MERKLE_COMPRESS, codes.data_ptr(), roots.data_ptr(), None, fin.data_ptr())
    sb = bzk.make_batch(k, d, order, bzk.BZK_F_PRESERVE_INPUT, B, first, None, tables, bzk.BZK_MEM_DEVICE,
                        bzk.BZK_MEM_DEVICE, out["round_evals"], out["challenges"], out["final_evals"], out["claims"])

    def reset():
        with torch.cuda.stream(stream):       # untimed: every step encodes the same messages
            codes.view(B * S, 2 * n, 4)[:, :n].copy_(msgs[:, 0])

    def barrier():
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    for _ in range(args.warmup):
        reset()
        bzk.bzk_commit_prove(enc.ctx, enc.enc, commit, sb, stream)
    stream.synchronize()

    def timed(profile):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        bzk.bzk_profile_enable(enc.ctx, profile)
        bzk.bzk_profile_read(enc.ctx, reset=True)
        bzk.bzk_launch_count(enc.ctx, reset=True)
        barrier()
        with ClockSampler(local) as clk:
            for i in range(args.steps):
                reset()
                ev[i][0].record(stream)
                bzk.bzk_commit_prove(enc.ctx, enc.enc, commit, sb, stream)
                ev[i][1].record(stream)
            stream.synchronize()
            barrier()
        launches = bzk.bzk_launch_count(enc.ctx, reset=True)
        prof = bzk.bzk_profile_read(enc.ctx, reset=True)
        bzk.bzk_profile_enable(enc.ctx, False)
        return float(sum(a.elapsed_time(b) for a, b in ev)), launches, prof, clk.summary()

    my_ms, launches, _, clocks = timed(False)
    _, _, prof, _ = timed(True)
    max_ms = shard.max_over_ranks(my_ms, dist, device="cuda")
    digest = shard.output_digest([fin.cpu()] + [out[key].cpu() for key in ("round_evals", "challenges", "final_evals",
                                                                           "claims")])
    digests = [x.hex() for x in shard.gather_bytes(bytes.fromhex(digest), dist, device="cuda")]
    ms_per_step = max_ms / args.steps
    value = B * world * args.steps / (max_ms / 1000.0)
    kernel_ms = {nm: round(v[0] / args.steps, 3) for nm, v in prof.items() if v[1]}
    # roofline of the dominant kernel kind (encoder products: IMAD; Merkle stages: ALU; sum-check rounds)
    hbm_peak, sm_max_mhz, peak_src = peaks()
    dom = max(kernel_ms, key=kernel_ms.get)
    edges = enc_edges(code)
    roof = {"kernel": dom}
    if dom == "encoder_spmv":
        ach = B * S * edges / (kernel_ms[dom] / 1000.0) / 1e9
        peak = SMS * IMAD_PER_CLK_SM * sm_max_mhz * 1e6 / IMAD_PER_EDGE_PRODUCT / 1e9
        roof.update({"bound": "alu", "achieved": round(ach, 2), "peak": round(peak, 2), "unit": "Gproduct/s",
                     "frac": round(ach / peak, 4), "traffic": None,
                     "peak_source": f"guide unit counts: {SMS} SMs x {IMAD_PER_CLK_SM} IMAD/clk x {sm_max_mhz:.0f} MHz "
                                    f"/ {IMAD_PER_EDGE_PRODUCT} IMAD slots per edge product"})
    elif dom == "merkle_stage":
        hashes = B * S * (2 * n - 1) + B * (S - 1)
        ach = hashes / (kernel_ms[dom] / 1000.0) / 1e9
        peak = SMS * ALU_PER_CLK_SM * sm_max_mhz * 1e6 / ALU_OPS_PER_COMPRESSION / 1e9
        roof.update({"bound": "alu", "achieved": round(ach, 3), "peak": round(peak, 3), "unit": "Ghash/s",
                     "frac": round(ach / peak, 4), "traffic": None})
    else:
        slots = (imad_slots(d, k, "round1") + imad_slots(d, k, "fused")) * B
        t_all = (kernel_ms.get("round1_eval", 0) + kernel_ms.get("fused_fold_eval", 0)) / 1000.0
        ach = slots / t_all
        peak = SMS * IMAD_PER_CLK_SM * sm_max_mhz * 1e6
        roof.update({"bound": "alu", "achieved": round(ach / 1e12, 3), "peak": round(peak / 1e12, 3),
                     "unit": "T IMAD-slot/s", "frac": round(ach / peak, 4), "traffic": None})
    line = {"metric": CHAIN_METRIC, "value": round(value, 2), "unit": "proofs/s", "n_gpus": world,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u32", "data": "synthetic",
            "config": {"workload": desc, "proofs_per_gpu": B, "segments": S, "segment_log_n": log_n, "d": d, "k": k,
                       "edges_per_codeword": edges, "l2": "codewords + tables larger than L2; no flush"},
            "gpu_launches": launches, "gpu_launches_per_step": launches / args.steps, "kernel_ms_per_step": kernel_ms,
            "roofline": roof, "clocks": clocks, "digest_rank0": digests[0], "digests_per_rank": len(digests)}
    if rank == 0:
        print(json.dumps(line), flush=True)
    enc.close()
    if dist:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="c2", choices=sorted(CONFIGS))
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--batch", type=int, default=None, help="override proofs (trees) per GPU")
    ap.add_argument("--log-blocks", type=int, default=None, help="Merkle configs: override n (2^n blocks per tree)")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu", action="store_true")
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--ref-proofs", type=int, default=None, help="oracle sample (default min(B, 4 x cores))")
    ap.add_argument("--vml-chunk", type=int, default=0, help="c4: images per job group (0 = all)")
    ap.add_argument("--wave", type=int, default=1024, help="c5: proofs per wave on each GPU (<= 1024)")
    ap.add_argument("--k", type=int, default=None, help="sum-check configs: override k (size sweeps)")
    args = ap.parse_args()

    rank = int(os.environ.get("RANK", 0))
    world = int(os.environ.get("WORLD_SIZE", 1))
    local = int(os.environ.get("LOCAL_RANK", 0))
    # BZK_BENCH_DEVICE pins every rank to one GPU and BZK_DIST_BACKEND=gloo swaps the collective
    # backend: together they smoke-test the multi-rank path on a single-GPU box
    if os.environ.get("BZK_BENCH_DEVICE") is not None:
        local = int(os.environ["BZK_BENCH_DEVICE"])

    if args.impl == "reference":
        run_reference(args, rank, world)
        return
    if args.config == "c4":
        run_vml(args, rank, world)
        return
    if CONFIGS[args.config][4] == "blocks":
        run_merkle(args, rank, world)
        return
    if CONFIGS[args.config][4] == "code":
        run_encoder(args, rank, world)
        return
    if CONFIGS[args.config][4] == "chain":
        run_chain(args, rank, world, local)
        return

    run_sumcheck(args, rank, world, local)

if __name__ == "__main__":
    main()
