# one gpurun call: final default bench (full line), a second short run, then the ncu evidence of the final build:
# headline kernel util (enforced vs monolithic) + full capture at the bench's operating point, K-BENCH per stage
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null 2>&1; echo build_rc=$?
timeout 1500 python bench.py > gpurun_out/h_bench1.json 2> gpurun_out/h_bench1.err; echo bench1=$?
timeout 1200 python bench.py --no-side --no-stages > gpurun_out/h_bench2.json 2> gpurun_out/h_bench2.err; echo bench2=$?
tail -1 gpurun_out/h_bench1.json > gpurun_out/h_bench_line.json
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg
timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec -c 2 --csv --log-file gpurun_out/h_ncu_util.csv python tools/ncu_headline.py gpurun_out/h_bench_line.json > gpurun_out/h_ncu_util.log 2>&1; echo util_rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:pl_exec_enforced -c 1 -o gpurun_out/h_ncu_full python tools/ncu_headline.py gpurun_out/h_bench_line.json > gpurun_out/h_ncu_full.log 2>&1; echo full_rc=$?
M2=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M2 --clock-control none -k regex:kbench --csv --log-file gpurun_out/h_kb_ncu.csv python tools/stage_bench.py 104857600 1 > gpurun_out/h_kb_ncu.jsonl 2>&1; echo kb_rc=$?
python tools/ncu_kbench_table.py gpurun_out/h_kb_ncu.csv gpurun_out/h_kb_ncu.jsonl
