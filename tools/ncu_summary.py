"""Summarise an ncu --set full report into profiles/ (text + JSON).

usage: python tools/ncu_summary.py <report.ncu-rep> <out_prefix> [algorithmic_bytes_per_launch]
"""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum", "sm__cycles_elapsed.avg",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "lts__t_bytes.sum", "launch__registers_per_thread",
        "launch__shared_mem_per_block_dynamic", "launch__grid_size", "launch__block_size",
        "smsp__pcsamp_warps_issue_stalled_barrier", "smsp__pcsamp_warps_issue_stalled_sleeping",
        "smsp__pcsamp_warps_issue_stalled_wait", "smsp__pcsamp_warps_issue_stalled_no_instructions",
        "smsp__pcsamp_warps_issue_stalled_short_scoreboard", "smsp__pcsamp_warps_issue_stalled_long_scoreboard",
        "smsp__pcsamp_warps_issue_stalled_branch_resolving", "smsp__pcsamp_warps_issue_stalled_selected"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1}


def main():
    rep, out = sys.argv[1], sys.argv[2]
    alg = float(sys.argv[3]) if len(sys.argv) > 3 else None
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k)
                d[k] = (r[i], units[i])
        res.append(d)
    lines = []
    js = []
    for d in res:
        lines.append(f"kernel: {d['kernel']}")
        for k in KEYS:
            if k in d:
                lines.append(f"  {k:62s} {d[k][0]:>16s} {d[k][1]}")
        def val(k):
            v, u = d[k]
            return float(v.replace(",", "")) * SCALE.get(u, 1)
        rb, wb, t = val("dram__bytes_read.sum"), val("dram__bytes_write.sum"), val("gpu__time_duration.sum")
        e = {"kernel": d["kernel"], "duration_s": t, "dram_bytes_per_launch": rb + wb, "dram_read": rb, "dram_write": wb}
        if alg:
            e["algorithmic_bytes_per_launch"] = alg
            e["traffic_over_algorithmic"] = (rb + wb) / alg
            lines.append(f"  algorithmic bytes/launch {alg:.0f}; traffic/algorithmic {(rb + wb) / alg:.2f}")
        js.append(e)
    open(out + ".txt", "w").write("\n".join(lines) + "\n")
    json.dump(js[0] if len(js) == 1 else js, open(out + ".json", "w"), indent=1)
    print("\n".join(lines))


if __name__ == "__main__":
    main()
