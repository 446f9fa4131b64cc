# one gpurun call: synccheck with win_step inlined vs out of line
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
PLGPU_LIB=_variants/x_wsinl.so timeout 1200 compute-sanitizer --tool synccheck python tools/sanitize_run.py > gpurun_out/r02_synccheck_wsinl.txt 2>&1; echo wsinl_rc=$?
tail -2 gpurun_out/r02_synccheck_wsinl.txt
