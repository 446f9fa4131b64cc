# one gpurun call: budget margin A/B on the default bench (t_i = margin x longest probe firing + 128 ns)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for m in 1.0 1.05; do timeout 1200 python bench.py --budget-margin $m --no-side --no-stages > gpurun_out/mg_$m.json 2> gpurun_out/mg_$m.err; echo margin_$m=$?; done
