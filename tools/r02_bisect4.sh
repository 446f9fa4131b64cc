# one gpurun call: per-firing cost, watchdog placement
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
  PLGPU_LIB=_variants/v_81e5c17.so timeout 300 python tools/bisect_fire.py v_81e5c17
  timeout 300 python tools/bisect_fire.py in-tree
  PL_VARIANT=0 timeout 300 python tools/bisect_fire.py in-tree-v0
  PLGPU_LIB=_variants/x_nowd2.so timeout 300 python tools/bisect_fire.py x_nowd2
done
