# one gpurun call: the default bench without the budget refinement at the operating point (--refine 0), twice
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for r in 1 2; do timeout 1200 python bench.py --refine 0 --no-side --no-stages > gpurun_out/rf_$r.json 2> gpurun_out/rf_$r.err; echo rf_$r=$?; done
