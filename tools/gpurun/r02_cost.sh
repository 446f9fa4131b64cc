# one gpurun call: per-firing cost of the in-tree build (both node-0 pacing modes) + parity regression
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
  timeout 300 python tools/bisect_fire.py in-tree
  PL_VARIANT=0 timeout 300 python tools/bisect_fire.py in-tree-v0
done
timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_cluster.py tests/test_gpu_live.py -m gpu -q > gpurun_out/r02_reg_cost.log 2>&1; echo reg_rc=$? >&2; tail -1 gpurun_out/r02_reg_cost.log >&2
