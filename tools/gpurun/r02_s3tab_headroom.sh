# one gpurun call: the default bench with the table-driven X-drop at two headrooms over the injected-stall edge
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for h in 1.15 1.25; do timeout 1200 python bench.py --headroom $h --no-side --no-stages > gpurun_out/sh_$h.json 2> gpurun_out/sh_$h.err; echo h_$h=$?; done
