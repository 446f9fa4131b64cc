# one gpurun call: K-BENCH parity tests, c4 stage rates, ncu per stage (table), ncu --set full of the S0 kernel
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 600 python -m pytest tests/test_gpu_stage_batch.py -m gpu -q > gpurun_out/kb3_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/kb3_tests.log
timeout 300 python tools/stage_bench.py 104857600 5 > gpurun_out/kb3_c4.jsonl 2>&1; timeout 300 python tools/stage_bench.py 1048576 5 > gpurun_out/kb3_c2.jsonl 2>&1
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum
timeout 900 ncu --metrics $M --clock-control none -k regex:kbench --csv --log-file gpurun_out/kb3_ncu_c4.csv python tools/stage_bench.py 104857600 1 > gpurun_out/kb3_ncu_c4.jsonl 2>&1
python tools/ncu_kbench_table.py gpurun_out/kb3_ncu_c4.csv gpurun_out/kb3_ncu_c4.jsonl
