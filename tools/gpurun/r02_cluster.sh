# one gpurun call: N4 cluster-variant GPU tests (+ live regression)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 600 python -m pytest tests/test_gpu_cluster.py -m gpu -x -q -s > gpurun_out/r02_cluster_$TAG.log 2>&1; echo cluster_rc=$?; tail -1 gpurun_out/r02_cluster_$TAG.log
timeout 600 python -m pytest tests/test_gpu_live.py tests/test_gpu_parity.py -m gpu -x -q > gpurun_out/r02_reg_$TAG.log 2>&1; echo reg_rc=$?; tail -1 gpurun_out/r02_reg_$TAG.log
