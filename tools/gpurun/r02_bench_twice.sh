# one gpurun call: the default bench (c4 headline, headroom 1.08) twice on one box
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for r in 1 2; do timeout 1200 python bench.py > gpurun_out/r02_bench_h108_$r.json 2> gpurun_out/r02_bench_h108_$r.err; echo bench_$r=$?; done
