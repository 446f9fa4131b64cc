# one gpurun call: the whole GPU suite, smoke, the default bench, then the ncu evidence of the bench's kernel
# at the bench's own operating point (util enforced vs monolithic, full capture) -> ncu_summary inputs
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null 2>&1; echo build_rc=$?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/f_gputests.log 2>&1; echo gpu_rc=$?; tail -2 gpurun_out/f_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/f_smoke.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/f_smoke.log
timeout 1500 python bench.py > gpurun_out/f_bench.json 2> gpurun_out/f_bench.err; echo bench_rc=$?
tail -1 gpurun_out/f_bench.json > gpurun_out/f_bench_line.json
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg
timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec -c 2 --csv --log-file gpurun_out/f_ncu_util.csv python tools/ncu_headline.py gpurun_out/f_bench_line.json > gpurun_out/f_ncu_util.log 2>&1; echo util_rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:pl_exec_enforced -c 1 -o gpurun_out/f_ncu_full python tools/ncu_headline.py gpurun_out/f_bench_line.json > gpurun_out/f_ncu_full.log 2>&1; echo full_rc=$?
