# one gpurun call: agreement tests (incl. the bench kernel's match-set digest), then the ncu
# evidence of the current build (util enforced vs monolithic, full capture of the headline kernel)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 900 python -m pytest tests/test_gpu_agreement.py -m gpu -q -rs -s > gpurun_out/r02_agree_$TAG.log 2>&1; echo agree_rc=$?; tail -1 gpurun_out/r02_agree_$TAG.log
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed,sm__warps_active.avg.pct_of_peak_sustained_active,dram__bytes_read.sum,dram__bytes_write.sum,sm__cycles_elapsed.avg
timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec -c 2 --csv --log-file gpurun_out/r02_ncu_util_$TAG.csv python tools/ncu_headline.py > gpurun_out/r02_ncu_util_$TAG.log 2>&1; echo util_rc=$?
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:pl_exec_enforced -c 1 -o gpurun_out/r02_ncu_full_$TAG python tools/ncu_headline.py > gpurun_out/r02_ncu_full_$TAG.log 2>&1; echo full_rc=$?
