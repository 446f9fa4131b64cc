# one gpurun call: per-firing cost across builds (tools/bisect_fire.py)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for v in d2863c6 636ad4b 9bfdfa5 81e5c17 5371798 f9a0b01 ce4b6ae 8df1efc; do
  PLGPU_LIB=_variants/v_$v.so timeout 300 python tools/bisect_fire.py $v
done
PL_VARIANT=0 timeout 300 python tools/bisect_fire.py in-tree-variant0
timeout 300 python tools/bisect_fire.py in-tree
