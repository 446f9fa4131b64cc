# one gpurun call: the K-BENCH per-stage kernels (full-occupancy rewrite): parity, c2/c4 rates, ncu per stage
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 600 python -m pytest tests/test_gpu_stage_batch.py -m gpu -q > gpurun_out/kb_tests.log 2>&1; echo tests=$?; tail -1 gpurun_out/kb_tests.log
timeout 300 python tools/stage_bench.py 1048576 5 > gpurun_out/kb_c2.jsonl 2> gpurun_out/kb_c2.err; echo c2=$?
timeout 600 python tools/stage_bench.py 104857600 5 > gpurun_out/kb_c4.jsonl 2> gpurun_out/kb_c4.err; echo c4=$?
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M --clock-control none -k regex:kbench --csv --log-file gpurun_out/kb_ncu_c4.csv python tools/stage_bench.py 104857600 1 > gpurun_out/kb_ncu_c4.jsonl 2>&1; echo ncu=$?
python tools/ncu_kbench_table.py gpurun_out/kb_ncu_c4.csv gpurun_out/kb_ncu_c4.jsonl > gpurun_out/kb_table_c4.txt 2>&1; cat gpurun_out/kb_table_c4.txt
timeout 900 ncu --set full --clock-control none --import-source on -k regex:kbench -c 8 -o gpurun_out/kb_full_c4 python tools/stage_bench.py 104857600 1 > gpurun_out/kb_full_c4.log 2>&1; echo full=$?
