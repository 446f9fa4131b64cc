# one gpurun call: the N3 co-runner GPU test, then an ncu util A/B of leader-paced node 0 (PL_VARIANT=1)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 600 python -m pytest tests/test_gpu_corunner.py -m gpu -q -s > gpurun_out/r02_corunner_$TAG.log 2>&1; echo corun_rc=$?; tail -1 gpurun_out/r02_corunner_$TAG.log
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
PL_VARIANT=1 timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec_enforced -c 1 --csv --log-file gpurun_out/r02_ncu_util_v1_$TAG.csv python tools/ncu_headline.py > gpurun_out/r02_ncu_util_v1_$TAG.log 2>&1; echo v1_rc=$?
