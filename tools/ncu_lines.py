"""Map ncu per-SASS stall samples to CUDA source lines (via nvdisasm -g of the in-tree .so).
usage: python tools/ncu_lines.py <report.ncu-rep> <kernel-mangled-name-substring> [top]"""
import csv
import io
import os
import re
import subprocess
import sys
import tempfile

rep, kname = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = rows[1]
ix = {h: i for i, h in enumerate(hdr)}
data = rows[2:]
stalls = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
base = int(data[0][0], 16)
# line table from nvdisasm
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(os.path.join("paper_conf_icppw_planob21_b200", "libplgpu.so"))],
               cwd=d, capture_output=True)
cub = [f for f in os.listdir(d) if f.startswith("executor")][0]
dis = subprocess.run(["nvdisasm", "-g", os.path.join(d, cub)], capture_output=True, text=True).stdout
lines = {}
cur_fn = None
cur_line = None
for l in dis.split("\n"):
    m = re.match(r"\.text\.(\S+):", l)
    if m:
        cur_fn = m.group(1)
        continue
    m = re.search(r'line (\d+)', l)
    if "## File" in l and m:
        cur_line = int(m.group(1))
        continue
    m = re.match(r"\s+/\*([0-9a-f]{4,})\*/", l)
    if m and cur_fn and kname in cur_fn:
        lines[int(m.group(1), 16)] = cur_line
src = open("paper_conf_icppw_planob21_b200/csrc/executor.cu").read().split("\n")
agg = {}
tot = 0
for r in data:
    off = int(r[0], 16) - base
    ln = lines.get(off)
    def g(k):
        try:
            return int(r[ix[k]])
        except (ValueError, KeyError):
            return 0
    samp = g("Warp Stall Sampling (All Samples)") - g("stall_barrier") - g("stall_sleep")
    tot += samp
    a = agg.setdefault(ln, [0, {}])
    a[0] += samp
    for s in stalls:
        if s not in ("stall_barrier", "stall_sleep"):
            a[1][s] = a[1].get(s, 0) + g(s)
print("non-barrier/sleep samples:", tot)
for ln, (v, st) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    best = sorted(st.items(), key=lambda x: -x[1])[:2]
    text = src[ln - 1].strip()[:80] if ln else "?"
    print(f"{str(ln):>5s} {v:6d} {v / max(1, tot):6.3f}  {text:80s} {[(k[6:], c) for k, c in best]}")
