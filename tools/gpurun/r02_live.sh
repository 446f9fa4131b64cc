# one gpurun call: live-ingest GPU tests (+ the agreement tests)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
TAG=${1:-x}
timeout 900 python -m pytest tests/test_gpu_live.py -m gpu -x -q -s > gpurun_out/r02_live_$TAG.log 2>&1; echo live_rc=$?; tail -1 gpurun_out/r02_live_$TAG.log
timeout 600 python -m pytest tests/test_gpu_agreement.py -m gpu -x -q -s > gpurun_out/r02_agree_$TAG.log 2>&1; echo agree_rc=$?; tail -1 gpurun_out/r02_agree_$TAG.log
