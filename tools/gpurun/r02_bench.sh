# one gpurun call: the bench (default c4 headline)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}; shift
s=$(date +%s); timeout 1500 python bench.py "$@" > gpurun_out/r02_bench_$TAG.json 2> gpurun_out/r02_bench_$TAG.log; echo bench_rc=$? elapsed=$(( $(date +%s) - s ))
