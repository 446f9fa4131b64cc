python paper_conf_icppw_planob21_b200/build.py --force >/dev/null 2>&1; echo build_rc=$?
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/v_gputests.log 2>&1; echo gpu_rc=$?; tail -2 gpurun_out/v_gputests.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/v_smoke.log 2>&1; echo smoke_rc=$?; tail -2 gpurun_out/v_smoke.log
timeout 1500 python bench.py > gpurun_out/v_bench.json 2> gpurun_out/v_bench.err; echo bench_rc=$?; tail -c 600 gpurun_out/v_bench.json
