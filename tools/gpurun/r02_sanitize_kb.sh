# one gpurun call: compute-sanitizer memcheck + synccheck over tools/sanitize_run.py (K-BENCH kernels added)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 1500 compute-sanitizer --tool memcheck --leak-check full python tools/sanitize_run.py > gpurun_out/r02_memcheck_kb.txt 2>&1; echo memcheck_rc=$?; tail -3 gpurun_out/r02_memcheck_kb.txt
timeout 1500 compute-sanitizer --tool synccheck python tools/sanitize_run.py > gpurun_out/r02_synccheck_kb.txt 2>&1; echo synccheck_rc=$?; tail -3 gpurun_out/r02_synccheck_kb.txt
