# one gpurun call: ncu --set full of THRESHOLD_SLACK and MONOLITHIC at the c3 point (50 ns, 350 us)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
timeout 1200 ncu --set full --import-source on --nvtx --nvtx-include "measure/" --clock-control none -k regex:pl_exec_enforced -c 1 -o gpurun_out/c3_full_thr python tools/ncu_c3_points.py 50:350 > gpurun_out/c3_full_thr.log 2>&1; echo thr=$?
timeout 1200 ncu --set full --import-source on --nvtx --nvtx-include "measure/" --clock-control none -k regex:pl_exec_monolithic -c 1 -o gpurun_out/c3_full_mono python tools/ncu_c3_points.py 50:350 > gpurun_out/c3_full_mono.log 2>&1; echo mono=$?
