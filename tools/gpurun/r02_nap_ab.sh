# one gpurun call: ncu instruction counts of the headline kernel, nap shift 2 (default) vs 1
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec_enforced -c 1 --csv --log-file gpurun_out/r02_nap_s2.csv python tools/ncu_headline.py > gpurun_out/r02_nap_s2.log 2>&1; echo s2=$?
PLGPU_LIB=_variants/x_nap1.so timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec_enforced -c 1 --csv --log-file gpurun_out/r02_nap_s1.csv python tools/ncu_headline.py > gpurun_out/r02_nap_s1.log 2>&1; echo s1=$?
