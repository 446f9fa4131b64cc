# one gpurun call: node-0 pacing mode (PL_VARIANT 0 = every warp paces, 1 = leader paces) on the
# current build -- c4 probe, c2 probe, and ncu instructions of the c4 headline kernel
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for v in 0 1; do
  PL_VARIANT=$v timeout 300 python tools/probe_c4.py v$v
  PL_VARIANT=$v timeout 300 python tools/bisect_fire.py c2-v$v
  M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum
  PL_VARIANT=$v timeout 900 ncu --metrics $M --clock-control none -k regex:pl_exec_enforced -c 1 --csv --log-file gpurun_out/r02_pace_v$v.csv python tools/ncu_headline.py > /dev/null 2>&1
done
