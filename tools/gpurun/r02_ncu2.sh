python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg
timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec -c 2 --csv --log-file gpurun_out/r02_ncu_c4_util.csv python tools/ncu_headline.py > gpurun_out/r02_ncu_c4_util.log 2>&1; echo util_rc=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:stage_batch -c 8 -o gpurun_out/r02_ncu_stages_c4 python tools/stage_bench.py 104857600 1 > gpurun_out/r02_ncu_stages_c4.log 2>&1; echo stages_rc=$?
