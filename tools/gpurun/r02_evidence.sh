# one gpurun call: ncu evidence for the c4 headline (parameters from $SRC, default profiles/r02_bench_c4_latest.json)
#  1. hardware utilisation, enforced (THRESHOLD_SLACK) vs MONOLITHIC at the same (tau0, D)
#  2. ncu --set full of the headline kernel (traffic, issue, stalls) -> ncu_summary_c4.json
#  3. the launch list of a short bench run (per-launch durations, cold and serialised)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg
timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec -c 2 --csv --log-file gpurun_out/r02_ncu_util_$TAG.csv python tools/ncu_headline.py ${SRC:-profiles/r02_bench_c4_latest.json} > gpurun_out/r02_ncu_util_$TAG.log 2>&1; echo util_rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:pl_exec_enforced -c 1 -o gpurun_out/r02_ncu_full_$TAG python tools/ncu_headline.py ${SRC:-profiles/r02_bench_c4_latest.json} > gpurun_out/r02_ncu_full_$TAG.log 2>&1; echo full_rc=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r02_launches_$TAG.csv python bench.py --steps 3 --warmup 3 --no-side --no-e2e --no-cpu-baseline > gpurun_out/r02_launches_$TAG.json 2> gpurun_out/r02_launches_$TAG.log; echo launches_rc=$?
