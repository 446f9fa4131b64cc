# one gpurun call: c4 probe per build (sink spread, nap shift) -- budgets and logical time
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
  timeout 300 python tools/probe_c4.py in-tree
  PLGPU_LIB=_variants/x_spread.so timeout 300 python tools/probe_c4.py spread
done
bash tools/gpurun/r02_nap_ab.sh >&2
