# one gpurun call: PL_NAP_HALF A/B -- c3 issue counts (ncu), the c4 budget probe, and the default bench with the variant
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed
for v in base naphalf; do
  if [ $v = base ]; then L=; else L=_variants/$v.so; fi
  PLGPU_LIB=$L timeout 900 ncu --nvtx --nvtx-include "measure/" --metrics $M --clock-control none --csv --log-file gpurun_out/nh_ncu_$v.csv python tools/ncu_c3_points.py > gpurun_out/nh_pts_$v.jsonl 2> gpurun_out/nh_pts_$v.err
  python tools/ncu_c3_table.py gpurun_out/nh_ncu_$v.csv gpurun_out/nh_pts_$v.jsonl > gpurun_out/nh_table_$v.txt 2>&1; echo "== $v"; cat gpurun_out/nh_table_$v.txt
  PLGPU_LIB=$L timeout 300 python tools/probe_c4.py $v >> gpurun_out/nh_probe.jsonl 2>/dev/null
done
cat gpurun_out/nh_probe.jsonl
PLGPU_LIB=_variants/naphalf.so timeout 1200 python bench.py --no-side --no-stages > gpurun_out/nh_bench.json 2> gpurun_out/nh_bench.err; echo bench=$?
