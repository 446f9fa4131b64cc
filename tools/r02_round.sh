# one gpurun call: GPU tests, the hardware-utilisation ncu pass (enforced vs monolithic), the bench
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 600 python -m pytest tests -m gpu -x -q > gpurun_out/r02_gputests_$TAG.log 2>&1; echo tests_rc=$?; tail -1 gpurun_out/r02_gputests_$TAG.log
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg
timeout 600 ncu --metrics $M --clock-control none -k regex:pl_exec -c 2 --csv --log-file gpurun_out/r02_ncu_util_$TAG.csv python tools/ncu_headline.py > gpurun_out/r02_ncu_util_$TAG.log 2>&1; echo util_rc=$?
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/r02_bench_$TAG.json 2> gpurun_out/r02_bench_$TAG.log; echo bench_rc=$? elapsed=$(( $(date +%s) - s ))
