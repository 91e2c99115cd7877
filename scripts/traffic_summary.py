"""Summarise scripts/ncu_traffic2.sh captures into profiles/traffic.json (per config, per kernel kind:
average DRAM bytes per launch) -- the `traffic` field of bench.py's roofline object."""
import csv
import json
import sys
from collections import defaultdict

BATCH = {"c2": 1024, "c3": 256, "g2": 1024, "m0": 1024, "m0lit": 1024, "enc20": 256}   # bench.py default batches


def kind_of(name):
    if "k_spmv" in name:
        return "encoder_spmv"
    if "k_multi" in name:
        return "multi_round"
    if "k_small" in name:
        return "small_cluster"
    if "k_round1_tc" in name:
        return "round1_eval"
    if "k_fused_tc" in name:   # k_fused_tc<D, ORDER, FIRST, NW>
        first = name.split("<", 1)[1].split(">")[0].split(",")[2].strip()
        return "round1_eval" if first in ("1", "true") else "fused_fold_eval"
    args = name.split("<", 1)[1].split(">")[0].split(",")      # k_round<D, ORDER, FIRST, TMA>, k_gl_round<D, ORDER, FIRST>
    first = args[2].strip()
    return "round1_eval" if first in ("1", "true") else "fused_fold_eval"


def main(out_path, files):
    entries = []
    for f in files:
        cfg = f.split("traffic2_")[-1].split(".")[0]
        rows = list(csv.reader(open(f)))
        h = next(i for i, r in enumerate(rows) if "Metric Name" in r)
        H = rows[h]
        ki, mi, vi, ii = H.index("Kernel Name"), H.index("Metric Name"), H.index("Metric Value"), H.index("ID")
        ui = H.index("Metric Unit")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}
        per = defaultdict(dict)
        for r in rows[h + 1:]:
            if len(r) > vi:
                per[(r[ii], r[ki])][r[mi]] = float(r[vi].replace(",", "")) * scale.get(r[ui], 1)
        agg = defaultdict(lambda: [0, 0.0, 0.0, 0.0])
        for (_, name), m in per.items():
            a = agg[kind_of(name)]
            a[0] += 1
            a[1] += m.get("dram__bytes_read.sum", 0)
            a[2] += m.get("dram__bytes_write.sum", 0)
            a[3] += m.get("gpu__time_duration.sum", 0)
        for kind, (n, rd, wr, t) in agg.items():
            entries.append({"config": cfg, "kernel_kind": kind, "launches": n, "batch": BATCH.get(cfg),
                            "dram_bytes_per_launch": int((rd + wr) / n), "dram_read_per_launch": int(rd / n),
                            "dram_write_per_launch": int(wr / n),
                            "source": f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum (one bench step, "
                                      f"default batch) -> {f}"})
    json.dump(entries, open(out_path, "w"), indent=1)
    for e in entries:
        print(e["config"], e["kernel_kind"], e["launches"], e["dram_bytes_per_launch"] / 1e9, "GB/launch")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2:])
