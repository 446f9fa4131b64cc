# one gpurun call: ncu --set full of the K-BENCH S3 kernel on c4 (source-level view of the X-drop walk)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 900 ncu --set full --import-source on --clock-control none -k regex:kbench_kernel -s 7 -c 1 -o gpurun_out/s3_full python tools/stage_bench.py 104857600 1 > gpurun_out/s3_full.log 2>&1; echo rc=$?
