"""Where a kernel issues: per-CUDA-source-line 'selected' warp-stall samples (a sample whose warp
was issuing) from an ncu report captured with --import-source on, with each line's share.
usage: python tools/ncu_issue_lines.py <report.ncu-rep> [top]"""
import csv
import io
import subprocess
import sys

raw = subprocess.run(["ncu", "-i", sys.argv[1], "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
rows = list(csv.reader(io.StringIO(raw)))
hdr = next(r for r in rows if r and r[0] == "Line No")
S = hdr.index("stall_selected")
agg, src, cur = {}, {}, None
for r in rows:
    if not r:
        continue
    if r[0].isdigit():
        cur = int(r[0])
        src[cur] = r[1][:100]
        continue
    if r[0] == "" and len(r) == len(hdr) and r[2].startswith("0x") and cur is not None:
        agg[cur] = agg.get(cur, 0) + int(r[S] or 0)
tot = sum(agg.values())
print(f"selected (issuing) samples {tot}")
acc = 0
for ln, v in sorted(agg.items(), key=lambda kv: -kv[1])[:top]:
    acc += v
    print(f"{ln:5d} {v:6d} {100 * v / tot:5.1f}% cum {100 * acc / tot:5.1f}% | {src.get(ln, '')}")
