# one gpurun call: ncu issue-active / instructions of enforced waiting vs monolithic at c3 points (tools/ncu_c3_points.py)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 900 python tools/ncu_c3_points.py > gpurun_out/c3u_plain.jsonl 2> gpurun_out/c3u_plain.err; echo plain=$?
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed
timeout 1500 ncu --nvtx --nvtx-include "measure/" --metrics $M --clock-control none --csv --log-file gpurun_out/c3u_ncu.csv python tools/ncu_c3_points.py > gpurun_out/c3u_ncu.jsonl 2> gpurun_out/c3u_ncu.err; echo ncu=$?
python tools/ncu_c3_table.py gpurun_out/c3u_ncu.csv gpurun_out/c3u_ncu.jsonl > gpurun_out/c3u_table.txt 2>&1; cat gpurun_out/c3u_table.txt
