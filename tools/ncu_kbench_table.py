"""Per-stage table from an `ncu --metrics ... --csv` log of tools/stage_bench.py (K-BENCH kernels):
the last launch of each stage, its duration, DRAM bytes, GB/s and fraction of the measured HBM peak,
issue-active and SM throughput, plus the algorithmic bytes stage_bench.py prints.
usage: python tools/ncu_kbench_table.py <ncu.csv> <stage_bench.jsonl>"""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
    PK = json.load(f)["hbm_gbs"]
rows = {}
with open(sys.argv[1]) as f:
    lines = [l for l in f if l.startswith('"')]
for r in csv.DictReader(lines):
    rows.setdefault(int(r["ID"]), {})[r["Metric Name"]] = (r["Metric Value"].replace(",", ""), r["Metric Unit"])
algo = [json.loads(l) for l in open(sys.argv[2]) if l.startswith("{")]
ids = sorted(rows)
per_stage = [ids[2 * s + 1] for s in range(len(ids) // 2)]   # stage_bench: a warm-up and one timed launch per stage
names = ["S0 seed lookup", "S1 hit enumeration", "S2 window filter", "S3 X-drop"]
print(f"{'stage':<20}{'inputs':>12}{'us':>10}{'dram_MB':>10}{'GB/s':>9}{'frac_hbm':>10}{'issue%':>8}{'sm%':>7}"
      f"{'alg_MB':>9}{'alg_GB/s':>10}")
for s, i in enumerate(per_stage):
    m = rows[i]
    ns = float(m["gpu__time_duration.sum"][0]) * (1e3 if m["gpu__time_duration.sum"][1] == "usecond" else
                                                  1e6 if m["gpu__time_duration.sum"][1] == "msecond" else 1)
    def mb(k):
        v, u = m[k]
        return float(v) * {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1, "Gbyte": 1e3}[u]
    dram = mb("dram__bytes_read.sum") + mb("dram__bytes_write.sum")
    a = algo[s] if s < len(algo) else {}
    amb = a.get("algorithmic_bytes", 0) / 1e6
    print(f"{names[s]:<20}{a.get('inputs', 0):>12}{ns / 1e3:>10.1f}{dram:>10.1f}{dram * 1e6 / ns:>9.1f}"
          f"{dram * 1e6 / ns / PK:>10.2e}{float(m['smsp__issue_active.avg.pct_of_peak_sustained_active'][0]):>8.2f}"
          f"{float(m['sm__throughput.avg.pct_of_peak_sustained_elapsed'][0]):>7.2f}{amb:>9.1f}{amb * 1e6 / ns:>10.1f}")
print(f"# HBM peak {PK} GB/s (MEASURED_PEAKS.json)")
