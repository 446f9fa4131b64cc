"""Join an ncu source page (SASS) with nvdisasm line info of the in-tree library.

usage: python tools/ncu_sass.py <report.ncu-rep> <kernel-mangled-substring> [per_unit]
Prints per-source-line warp-instructions executed (divided by per_unit, e.g. the number
of firings x warps) and stall samples, in source order."""
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, kname = sys.argv[1], sys.argv[2]
per = float(sys.argv[3]) if len(sys.argv) > 3 else 1.0
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
data = [r for r in rows[2:] if len(r) == len(hdr)]
base = int(data[0][0], 16)
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath("paper_conf_icppw_planob21_b200/libplgpu.so")],
               cwd=d, capture_output=True)
cub = [f for f in os.listdir(d) if f.startswith("executor")][0]
dis = subprocess.run(["nvdisasm", "-g", os.path.join(d, cub)], capture_output=True, text=True).stdout
lines, fn, cur = {}, None, None
for l in dis.split("\n"):
    m = re.match(r"\.text\.(\S+):", l)
    if m:
        fn = m.group(1)
        continue
    m = re.search(r'line (\d+)', l)
    if "## File" in l and m:
        f = l.split('"')[1].split("/")[-1] if '"' in l else "?"
        cur = (f if "executor" not in f else "", int(m.group(1)))
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/", l)
    if m and fn and kname in fn:
        lines[int(m.group(1), 16)] = cur


def g(r, k):
    try:
        return float(r[ix[k]])
    except (ValueError, KeyError):
        return 0.0


agg = {}
stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
for r in data:
    ln = lines.get(int(r[0], 16) - base, ("?", 0))
    a = agg.setdefault(ln, {"inst": 0.0, "samp": 0.0, "st": {}})
    a["inst"] += g(r, "Instructions Executed")
    a["samp"] += g(r, "Warp Stall Sampling (All Samples)")
    for s in stall_cols:
        a["st"][s] = a["st"].get(s, 0) + g(r, s)
src = open("paper_conf_icppw_planob21_b200/csrc/executor.cu").read().split("\n")
tot_i = sum(a["inst"] for a in agg.values())
tot_s = sum(a["samp"] for a in agg.values())
print(f"total warp-inst {tot_i:.0f} ({tot_i / per:.1f} per unit), samples {tot_s:.0f}")
for ln in sorted(agg, key=lambda x: (x[0], x[1])):
    a = agg[ln]
    if a["inst"] / per < 0.5 and a["samp"] < tot_s * 0.003:
        continue
    top = sorted(a["st"].items(), key=lambda kv: -kv[1])[:3]
    txt = src[ln[1] - 1].strip()[:60] if ln[0] == "" and 0 < ln[1] <= len(src) else ln[0]
    print(f"{ln[0] or 'exec'}:{ln[1]:5d} inst/u {a['inst'] / per:7.1f} samp {a['samp']:6.0f}  "
          f"{' '.join(f'{k[6:]}={v:.0f}' for k, v in top if v)}  | {txt}")
