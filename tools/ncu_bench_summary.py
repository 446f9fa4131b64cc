"""profiles/ncu_summary_<workload>.json for bench.py's `roofline.traffic` and `issue` fields, from
one `ncu --set full` capture of the headline kernel (tools/gpurun/r02_evidence.sh) and the util pass
(enforced vs monolithic at the same tau0, D).

usage: python tools/ncu_bench_summary.py <full.ncu-rep> <util.csv> <roots_per_launch> <alg_bytes> <out.json>"""
import csv
import io
import json
import subprocess
import sys

rep, util, roots, alg, out = sys.argv[1], sys.argv[2], float(sys.argv[3]), float(sys.argv[4]), sys.argv[5]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, r = rows[0], rows[1], rows[2]
SC = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1}


def g(k):
    i = hdr.index(k)
    return float(r[i].replace(",", "")) * SC.get(units[i], 1)


inst = g("smsp__inst_executed.sum")
res = {"kernel": r[hdr.index("Kernel Name")], "source": rep.split("/")[-1],
       "duration_s": g("gpu__time_duration.sum"),
       "dram_bytes_per_launch": g("dram__bytes_read.sum") + g("dram__bytes_write.sum"),
       "algorithmic_bytes_per_launch": alg,
       "issue_active_pct": g("smsp__issue_active.avg.pct_of_peak_sustained_active"),
       "sm_throughput_pct": g("sm__throughput.avg.pct_of_peak_sustained_elapsed"),
       "warp_inst_per_launch": inst, "warp_inst_per_root": inst / roots}
res["traffic_over_algorithmic"] = res["dram_bytes_per_launch"] / alg
# enforced vs monolithic at the same (tau0, D): issue-active and instructions
u = list(csv.reader(open(util)))
h = next(i for i, x in enumerate(u) if x and x[0] == "ID")
cmp = {}
for x in u[h + 1:]:
    d = dict(zip(u[h], x))
    name = "enforced" if "enforced" in d["Kernel Name"] else "monolithic"
    cmp.setdefault(name, {})[d["Metric Name"]] = float(d["Metric Value"].replace(",", ""))
res["util_same_rate"] = {k: {"issue_active_pct": v.get("smsp__issue_active.avg.pct_of_peak_sustained_active"),
                             "warp_inst_per_root": v.get("smsp__inst_executed.sum", 0) / roots,
                             "sm_throughput_pct": v.get("sm__throughput.avg.pct_of_peak_sustained_elapsed")}
                         for k, v in cmp.items()}
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(res, indent=1))
