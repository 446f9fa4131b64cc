# one gpurun call: per-firing cost of experiment builds (tools/bisect_fire.py), twice each
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
for v in v_81e5c17 x_base x_wsinl x_nogate x_nowd x_noinj x_none; do
  PLGPU_LIB=_variants/$v.so timeout 300 python tools/bisect_fire.py $v
done
done
