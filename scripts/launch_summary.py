"""Summarise an ncu --metrics gpu__time_duration.sum launch list (CSV): per-kernel launches, total
time and share of the step (cold-cache, serialised launches: compare SHARES, not absolutes)."""
import csv, sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = next(i for i, r in enumerate(rows) if 'Kernel Name' in r)
h = rows[hdr]
ki, vi = h.index('Kernel Name'), h.index('Metric Value')
tot = {}
for r in rows[hdr + 1:]:
    if len(r) > vi:
        tot.setdefault(r[ki], []).append(float(r[vi].replace(',', '')) / 1e6)
T = sum(sum(v) for k, v in tot.items() if 'generate' not in k)
print(f"# {sys.argv[1]}: ncu --metrics gpu__time_duration.sum --clock-control none; k_generate is setup (untimed)")
for k, v in tot.items():
    share = 0 if 'generate' in k else sum(v) / T * 100
    print(f"{k[:70]:70s} launches={len(v):3d} total_ms={sum(v):9.3f} share={share:5.1f}%")
