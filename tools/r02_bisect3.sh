# one gpurun call: per-firing cost, current tree vs pre-live build, plus live/cluster regression tests
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
  PLGPU_LIB=_variants/v_81e5c17.so timeout 300 python tools/bisect_fire.py v_81e5c17
  timeout 300 python tools/bisect_fire.py in-tree
  PL_VARIANT=0 timeout 300 python tools/bisect_fire.py in-tree-v0
  PLGPU_LIB=_variants/x_nomask.so timeout 300 python tools/bisect_fire.py x_nomask
done
timeout 900 python -m pytest tests/test_gpu_live.py tests/test_gpu_cluster.py -m gpu -q > gpurun_out/r02_reg3.log 2>&1; echo reg_rc=$? >&2; tail -1 gpurun_out/r02_reg3.log >&2
