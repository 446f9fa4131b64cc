# one gpurun call: the whole GPU suite and smoke on the final build, the default bench, two more short bench runs
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null 2>&1; echo build_rc=$?
timeout 900 python -m pytest tests -m gpu -q > gpurun_out/g_gputests.log 2>&1; echo gpu_rc=$?; tail -2 gpurun_out/g_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/g_smoke.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/g_smoke.log
timeout 1500 python bench.py > gpurun_out/g_bench1.json 2> gpurun_out/g_bench1.err; echo bench1=$?
for r in 2 3; do timeout 1200 python bench.py --no-side --no-stages > gpurun_out/g_bench$r.json 2> gpurun_out/g_bench$r.err; echo bench$r=$?; done
