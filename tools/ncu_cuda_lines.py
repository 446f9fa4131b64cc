"""Per-CUDA-source-line stall samples and warp instructions from an ncu report captured with
--import-source on (ncu's own cuda,sass correlation; no nvdisasm needed).
usage: python tools/ncu_cuda_lines.py <report.ncu-rep> [top] [inst]   (inst: sort by warp instructions)"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and r[0] == "Line No")
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
agg, src, cur = {}, {}, None
for r in rows:
    if not r:
        continue
    if r[0].isdigit():
        cur = int(r[0])
        src[cur] = ",".join(r[1:2])[:70]
        continue
    if r[0] == "" and len(r) > 7 and r[2].startswith("0x") and cur is not None:
        a = agg.setdefault(cur, [0, 0, {}])
        a[0] += int(r[6] or 0)
        a[1] += int(r[7] or 0)
        if len(r) == len(hdr):
            for i in stall_cols:
                v = int(r[i] or 0)
                if v:
                    a[2][hdr[i][6:]] = a[2].get(hdr[i][6:], 0) + v
tot = sum(a[0] for a in agg.values())
print(f"samples {tot}, warp-inst {sum(a[1] for a in agg.values())}")
key = 1 if len(sys.argv) > 3 and sys.argv[3] == "inst" else 0
for ln, a in sorted(agg.items(), key=lambda kv: -kv[1][key])[:top]:
    st = " ".join(f"{k}={v}" for k, v in sorted(a[2].items(), key=lambda kv: -kv[1])[:3])
    print(f"{ln:5d} samp {a[0]:6d} ({100 * a[0] / max(1, tot):4.1f}%) inst {a[1]:10d}  {st:45s} | {src.get(ln, '')}")
