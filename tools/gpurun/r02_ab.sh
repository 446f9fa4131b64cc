# one gpurun call: co-runner test, then bench A/B (leader-paced node 0; non-overloaded budget probe)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 600 python -m pytest tests/test_gpu_corunner.py -m gpu -q -s > gpurun_out/r02_corunner_$TAG.log 2>&1; echo corun_rc=$?; tail -1 gpurun_out/r02_corunner_$TAG.log
PL_VARIANT=1 timeout 900 python bench.py --no-side --no-e2e --no-cpu-baseline > gpurun_out/r02_bench_v1_$TAG.json 2> gpurun_out/r02_bench_v1_$TAG.log; echo v1_rc=$?
timeout 900 python bench.py --no-side --no-e2e --no-cpu-baseline --probe-t 20000 > gpurun_out/r02_bench_p20k_$TAG.json 2> gpurun_out/r02_bench_p20k_$TAG.log; echo p20k_rc=$?
