# one gpurun call: the whole -m gpu suite, smoke(), then the bench
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/r02_gputests_$TAG.log 2>&1; echo tests_rc=$?; tail -1 gpurun_out/r02_gputests_$TAG.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r02_smoke_$TAG.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/r02_smoke_$TAG.log
s=$(date +%s); timeout 1500 python bench.py > gpurun_out/r02_bench_$TAG.json 2> gpurun_out/r02_bench_$TAG.log; echo bench_rc=$? elapsed=$(( $(date +%s) - s ))
