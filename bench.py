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
                                          "--format=csv,noheader,nounits", "-lms", "100"],
                                         stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.t = threading.Thread(target=self._read, daemon=True)
            self.t.start()
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


def cpu_baseline(cfg, max_proofs=8):
    """The oracle as it stands on this box's host cores: a bounded sample of the same workload."""
    import numpy as np  # noqa: F401

    import oracle
    from paper_conf_asplos_lucw0cz25_b200 import inputs
    B, d, k, order, dist, _ = CONFIGS[cfg]
    cores = len(os.sched_getaffinity(0))
    n = max(1, min(max_proofs, cores, B))
    oracle.build()
    if dist == "code":
        code = inputs.gen_code(k, 6)
        ms = inputs.gen_tables(n, 1, k, 0)[:, 0]
        t0 = time.perf_counter()
        oracle.encode_batch(code, ms, nthreads=n)
        dt = time.perf_counter() - t0
        return {"value": n / dt, "unit": "codes/s", "cores": n, "kind": "oracle",
                "sample": f"{n} codewords of {cfg} (2^{k} elements), one per thread, {dt:.1f} s wall "
                          f"= {n * dt:.0f} CPU-seconds"}
    if dist == "blocks":
        blocks = inputs.gen_blocks(n, k, 0)
        t0 = time.perf_counter()
        oracle.merkle_batch(blocks, k, d, nodes=True, nthreads=n)
        dt = time.perf_counter() - t0
        return {"value": n / dt, "unit": "trees/s", "cores": n, "kind": "oracle",
                "sample": f"{n} trees of {cfg} (2^{k} blocks, hash mode {d}), one per thread, {dt:.1f} s wall "
                          f"= {n * dt:.0f} CPU-seconds"}
    if dist == "gl":
        import concurrent.futures as cf
        tabs = inputs.gen_tables_gl(n, d, k, 0)
        t0 = time.perf_counter()
        with cf.ThreadPoolExecutor(n) as ex:     # ctypes releases the GIL: one proof per thread
            list(ex.map(lambda b: oracle.gl_prove(tabs[b], k, d, order, inputs.DEFAULT_SEED, b), range(n)))
        dt = time.perf_counter() - t0
    else:
        tabs = inputs.gen_tables(n, d, k, 0, dist)
        t0 = time.perf_counter()
        oracle.prove_batch(tabs, k, d, order, inputs.DEFAULT_SEED, 0, nthreads=n)
        dt = time.perf_counter() - t0
    return {"value": n / dt, "unit": "proofs/s", "cores": n, "kind": "oracle",
            "sample": f"{n} proofs of {cfg} (d={d}, k={k}), one per thread, {dt:.1f} s wall "
                      f"= {n * dt:.0f} CPU-seconds"}


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
        times.append(cb["cores"] / cb["value"])
    nproofs = cb["cores"]
    value = nproofs * len(times) / sum(times)
    unit = cb["unit"]
    metric = {"blocks": MERKLE_METRIC, "code": ENC_METRIC}.get(dist, METRIC)
    line = {"impl": "reference", "metric": metric, "value": value,
            "unit": unit, "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1000 * sum(times) / len(times),
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u64",
            "data": "synthetic", "config": {"workload": desc, "batch_sampled": nproofs, "d": d, "k": k},
            "cpu_baseline": {"value": value, "unit": unit, "cores": nproofs, "kind": "oracle",
                             "sample": cb["sample"]},
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
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
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
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
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
    ap.add_argument("--ref-proofs", type=int, default=8)
    ap.add_argument("--vml-chunk", type=int, default=0, help="c4: images per job group (0 = all)")
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

    import numpy as np
    import torch

    from paper_conf_asplos_lucw0cz25_b200 import bzk
    torch.cuda.set_device(local)
    dist = None
    if world > 1:
        import torch.distributed as dist
        backend = os.environ.get("BZK_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)

    B, d, k, order, gen_dist, desc = CONFIGS[args.config]
    if args.batch:
        B = args.batch
    first, _ = shard.weak_range(B, rank)
    consume = args.config == "c3"
    gl = gen_dist == "gl"
    esz = 8 if gl else 32
    flags = 0 if consume else bzk.BZK_F_PRESERVE_INPUT
    if gl:
        flags |= bzk.BZK_F_FIELD_GOLDILOCKS

    def tshape(n):
        return (n, d, 1 << k) if gl else (n, d, 1 << k, 4)
    if args.config == "m0lit":
        flags |= bzk.BZK_F_GIVEN_CHALLENGES
    stream = torch.cuda.Stream()
    tables = torch.empty(tshape(B), dtype=torch.int64, device="cuda")
    bzk.bzk_generate(tables, B, d, k, first, gen_dist, stream=stream)
    prover = bzk.Prover(local)
    out = (bzk.Prover.alloc_outputs_gl if gl else bzk.Prover.alloc_outputs)(B, k, d)
    if flags & bzk.BZK_F_GIVEN_CHALLENGES:
        # pre-seeded challenges (the paper's PRG output): any canonical values < 2^253
        kk = max(1, (k - 1).bit_length())          # generator tables have 2^kk >= k entries
        g = torch.empty((B, 1, 1 << kk, 4), dtype=torch.int64, device="cuda")
        bzk.bzk_generate(g, B, 1, kk, first, "uniform", data_seed=0x5052470000000000, stream=stream)
        with torch.cuda.stream(stream):          # ordered after the generator on the same stream
            out["challenges"].copy_(g[:, 0, :k, :])
        stream.synchronize()
    batch = prover.batch(tables, k, d, order, None, first, flags, out)

    batch_g = prover.batch(tables, k, d, order, None, first, flags | bzk.BZK_F_GRAPH, out)

    def step(b):
        if consume:
            # consume mode destroys the input: regenerate it (untimed) before every step
            bzk.bzk_generate(tables, B, d, k, first, gen_dist, stream=stream)
        bzk.bzk_prove(prover.ctx, b, stream)

    for _ in range(args.warmup):
        step(batch_g)        # the first call captures the CUDA graph of the whole step
    stream.synchronize()

    def barrier():
        if dist:
            dist.barrier()
        torch.cuda.synchronize()

    def timed_region(b, profile):
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
        bzk.bzk_profile_enable(prover.ctx, profile)
        bzk.bzk_profile_read(prover.ctx, reset=True)
        bzk.bzk_launch_count(prover.ctx, reset=True)
        barrier()
        with ClockSampler(local) as clk:
            for i in range(args.steps):
                if consume:
                    bzk.bzk_generate(tables, B, d, k, first, gen_dist, stream=stream)
                ev[i][0].record(stream)
                bzk.bzk_prove(prover.ctx, b, stream)
                ev[i][1].record(stream)
            stream.synchronize()
            barrier()
        launches = bzk.bzk_launch_count(prover.ctx, reset=True)
        prof = bzk.bzk_profile_read(prover.ctx, reset=True)
        bzk.bzk_profile_enable(prover.ctx, False)
        return [a.elapsed_time(b_) for a, b_ in ev], launches, prof, clk.summary()

    # timed region 1 (the headline value): the whole step replayed as one CUDA graph
    step_ms, launches, _, clocks = timed_region(batch_g, False)
    # timed region 2 (roofline): the same steps launched kernel by kernel with CUDA events around
    # every launch on the launch stream (per-kernel device time)
    step_ms_prof, _, prof, _ = timed_region(batch, True)
    my_ms = float(sum(step_ms))

    # output digest (for cross-GPU-count comparisons) -- outside the timed region
    digest = shard.output_digest([out[key].cpu() for key in ("round_evals", "challenges", "final_evals", "claims")])

    max_ms = shard.max_over_ranks(my_ms, dist, device="cuda")
    digests = [x.hex() for x in shard.gather_bytes(bytes.fromhex(digest), dist, device="cuda")]
    # the proofs themselves are gathered to rank 0 over NCCL (NVLink) after the timed region
    # (north star: "NCCL is used only to gather proofs and timing"); rank 0 digests the global batch
    gathered = None
    if dist:
        torch.cuda.synchronize()
        g0 = time.perf_counter()
        allp = shard.gather_outputs({k_: out[k_] for k_ in ("round_evals", "challenges", "final_evals", "claims")},
                                    dist, dst=0)
        torch.cuda.synchronize()
        g_ms = (time.perf_counter() - g0) * 1000.0
        if rank == 0:
            gbytes = sum(v.numel() * v.element_size() for v in allp.values())
            gathered = {"proofs": B * world, "bytes": int(gbytes), "ms": round(g_ms, 3),
                        "backend": dist.get_backend(),
                        "global_digest": shard.output_digest([allp[k_].cpu() for k_ in
                                                              ("round_evals", "challenges", "final_evals", "claims")])}

    total_proofs = B * world * args.steps
    value = total_proofs / (max_ms / 1000.0)
    ms_per_step = max_ms / args.steps

    # ---------------- roofline of the dominant kernel (ALU-bound: integer pipe)
    hbm_peak, sm_max_mhz, peak_src = peaks()
    kinds = {"round1_eval": "round1", "fused_fold_eval": "fused"}
    dom = max(kinds, key=lambda n: prof[n][0])
    dom_ms, dom_cnt = prof[dom]
    mulmods_per_launch = alg_mulmods(d, k, kinds[dom]) * B / max(1, dom_cnt / args.steps)
    avg_launch_s = dom_ms / max(1, dom_cnt) / 1000.0
    achieved = mulmods_per_launch / avg_launch_s / 1e9
    int_peak = SMS * IMAD_PER_CLK_SM * sm_max_mhz * 1e6 / IMAD_PER_MULMOD / 1e9
    total_alg = alg_mulmods(d, k, "total") * B
    step_gmulmod = total_alg / (ms_per_step / 1000.0) / 1e9
    # HBM: algorithmic bytes (read each input once) and the streaming schedule's bytes
    alg_bytes = d * (1 << k) * esz * B
    traffic = None
    tpath = os.path.join(ROOT, "profiles", "traffic.json")
    if os.path.exists(tpath):
        # DRAM bytes per launch of the dominant kernel from one `ncu --set full` capture of the same
        # command (scripts/ncu_traffic.sh), if it was taken on this workload
        with open(tpath) as f:
            tj = json.load(f)
        for e in (tj if isinstance(tj, list) else [tj]):
            if e.get("config") == args.config and e.get("kernel_kind") == dom and e.get("batch") == B:
                traffic = e["dram_bytes_per_launch"]
    bytes_per_launch = alg_bytes_kind(d, k, kinds[dom], esz) * B / max(1, dom_cnt / args.steps)
    roofline = {"bound": "alu", "kernel": dom, "achieved": round(achieved, 2), "peak": round(int_peak, 2),
                "unit": "Gmulmod/s", "frac": round(achieved / int_peak, 4), "traffic": traffic,
                "alg_bytes_per_launch": bytes_per_launch,
                "peak_source": f"guide unit counts: {SMS} SMs x {IMAD_PER_CLK_SM} IMAD/clk x {sm_max_mhz:.0f} MHz "
                               f"({peak_src} max clock) / {IMAD_PER_MULMOD} IMAD per mulmod",
                "step_frac": round(step_gmulmod / int_peak, 4),
                "hbm_alg_frac": round(alg_bytes / (ms_per_step / 1000.0) / 1e9 / hbm_peak, 4),
                "hbm_peak_gbs": hbm_peak}
    # the dominant kernel's bound: the larger of its algorithmic IMAD time and HBM time at the peaks
    # (d = 1 fused rounds move 192 B per 2 products: HBM-bound; d >= 2 BN254 rounds: IMAD-bound)
    t_alu = mulmods_per_launch / (int_peak * 1e9)
    t_hbm = bytes_per_launch / (hbm_peak * 1e9)
    ach_gbs = bytes_per_launch / avg_launch_s / 1e9
    roofline["alu_time_at_peak_ms"] = round(t_alu * 1000, 4)
    roofline["hbm_time_at_peak_ms"] = round(t_hbm * 1000, 4)
    if not gl and t_hbm > t_alu:
        roofline.update({"bound": "hbm", "achieved": round(ach_gbs, 1), "peak": hbm_peak, "unit": "GB/s",
                         "frac": round(ach_gbs / hbm_peak, 4),
                         "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_src}); this kernel's algorithmic "
                                        "HBM time exceeds its IMAD time at the roofs",
                         "alu_gmulmod_s": round(achieved, 2), "alu_frac": round(achieved / int_peak, 4)})
    if gl:
        # Goldilocks (8-byte elements): the dominant kernel streams; its roof is HBM bandwidth
        roofline.update({"bound": "hbm", "achieved": round(ach_gbs, 1), "peak": hbm_peak, "unit": "GB/s",
                         "frac": round(ach_gbs / hbm_peak, 4),
                         "peak_source": f"MEASURED_PEAKS.json hbm_gbs ({peak_src}); achieved = algorithmic bytes per "
                                        "launch (reads 4dh + writes 2dh elements per proof for a fused round, 2dh "
                                        "reads for round 1) / CUDA-event launch time",
                         "alu_gmulmod_s": round(achieved, 2)})

    kernel_ms = {n: round(v[0] / args.steps, 3) for n, v in prof.items() if v[1]}
    line = {"metric": METRIC, "value": round(value, 2), "unit": "proofs/s", "n_gpus": world, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": round(ms_per_step, 3), "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "u64" if gl else "u32", "data": "synthetic",
            "config": {"workload": desc, "batch_per_gpu": B, "global_batch": B * world, "d": d, "k": k,
                       "order": "LSB" if order == 0 else "MSB", "field": "Goldilocks" if gl else "BN254 Fr",
                       "l2": "inputs larger than L2 (%.0f GiB vs 126 MB); no flush" % (B * d * (1 << k) * esz / 2**30)},
            "gpu_launches": launches, "gpu_launches_per_step": launches / args.steps,
            "kernel_ms_per_step": kernel_ms, "ms_per_step_kernel_by_kernel": round(sum(step_ms_prof) / args.steps, 3),
            "roofline": roofline, "clocks": clocks,
            "digest_rank0": digests[0], "digests_per_rank": len(digests)}
    if gathered:
        line["proofs_gathered"] = gathered

    # ---------------- e2e: host (pinned) tables in, host outputs out, through bzk_prove
    if not args.no_e2e and not consume:
        del tables
        torch.cuda.empty_cache()
        # pinned host memory is shared by all ranks of the node: cap each rank's e2e batch at 40 % of
        # the available host memory / world (same metric, proofs/s, on a smaller host-resident batch)
        try:
            avail = os.sysconf("SC_AVPHYS_PAGES") * os.sysconf("SC_PAGE_SIZE")
        except (ValueError, OSError):
            avail = 1 << 40
        proof_bytes = d * (1 << k) * esz
        Be = int(max(1, min(B, 0.4 * avail / world // proof_bytes)))
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
        if flags & bzk.BZK_F_GIVEN_CHALLENGES:
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
        e2e_ms = e0.elapsed_time(e1)
        e2e_ms = shard.max_over_ranks(e2e_ms, dist, device="cuda")
        out_bytes = sum(v.numel() * 8 for v in out_h.values())
        same = all(torch.equal(out_h[key], out[key][:Be].cpu()) for key in out_h)
        line["e2e"] = {"value": round(Be * world * args.e2e_steps / (e2e_ms / 1000.0), 2), "unit": "proofs/s",
                       "batch_per_gpu": Be,
                       "h2d_bytes_per_step": int(host_t.numel() * 8), "d2h_bytes_per_step": int(out_bytes),
                       "steps": args.e2e_steps, "wall_s": round(wall, 3), "matches_device_run": bool(same),
                       "path": "bzk_prove(tables_mem=HOST pinned, outputs_mem=HOST): side-stream H2D waves "
                               "overlapping compute"}
    if rank == 0 and world == 1 and not args.no_cpu:
        line["cpu_baseline"] = cpu_baseline(args.config)
    if rank == 0:
        print(json.dumps(line), flush=True)
    prover.close()
    if dist:
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
