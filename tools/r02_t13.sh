# one gpurun call: injection + agreement GPU tests, then the bench with injected-stall rate search
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_agreement.py -m gpu -x -q -s > gpurun_out/r02_gputests_$TAG.log 2>&1; echo tests_rc=$?; tail -1 gpurun_out/r02_gputests_$TAG.log
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/r02_bench_$TAG.json 2> gpurun_out/r02_bench_$TAG.log; echo bench_rc=$? elapsed=$(( $(date +%s) - s ))
