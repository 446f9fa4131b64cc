"""Join `ncu --metrics ... --csv` of tools/ncu_c3_points.py (launches in order) with its JSON lines:
issue-active %, warp instructions per root, model and hardware busy fractions per (tau0, D, policy).
usage: python tools/ncu_c3_table.py <ncu.csv> <points.jsonl>"""
import csv
import json
import sys

rows = {}
for r in csv.DictReader([l for l in open(sys.argv[1]) if l.startswith('"')]):
    rows.setdefault(int(r["ID"]), {})[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
runs = [json.loads(l) for l in open(sys.argv[2]) if l.startswith("{") and '"policy"' in l]
ids = sorted(rows)
assert len(ids) == len(runs), (len(ids), len(runs))
print(f"{'tau0':>5} {'D_us':>5} {'policy':<16} {'issue%':>7} {'inst/root':>10} {'model_af':>9} {'hw_busy':>8} {'misses':>7}")
for i, r in zip(ids, runs):
    m = rows[i]
    print(f"{r['tau0_ns']:>5} {r['D_us']:>5} {r['policy']:<16} {m['smsp__issue_active.avg.pct_of_peak_sustained_active']:>7.2f} "
          f"{m['smsp__inst_executed.sum'] / r['roots']:>10.1f} {r['active_fraction']:>9.4f} {r['hw_busy_fraction']:>8.4f} {r['misses']:>7}")
