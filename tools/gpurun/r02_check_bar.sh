# one gpurun call: synccheck/memcheck over tools/sanitize_run.py, per-firing cost, nap A/B
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 1200 compute-sanitizer --tool synccheck python tools/sanitize_run.py > gpurun_out/r02_synccheck2.txt 2>&1; echo synccheck_rc=$?
timeout 1200 compute-sanitizer --tool memcheck --leak-check full python tools/sanitize_run.py > gpurun_out/r02_memcheck2.txt 2>&1; echo memcheck_rc=$?
for rep in 1 2; do timeout 300 python tools/bisect_fire.py in-tree-syncwarp; done
