# one gpurun call: PL_NAP_LEAD A/B (lead of a waiting node's nap before its earliest possible firing):
# c3 issue counts (ncu), the c4 budget probe, and the default bench with lead 256
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed
for v in base lead256 lead64; do
  if [ $v = base ]; then L=; else L=_variants/$v.so; fi
  PLGPU_LIB=$L timeout 900 ncu --nvtx --nvtx-include "measure/" --metrics $M --clock-control none --csv --log-file gpurun_out/ld_ncu_$v.csv python tools/ncu_c3_points.py > gpurun_out/ld_pts_$v.jsonl 2> gpurun_out/ld_pts_$v.err
  python tools/ncu_c3_table.py gpurun_out/ld_ncu_$v.csv gpurun_out/ld_pts_$v.jsonl > gpurun_out/ld_table_$v.txt 2>&1; echo "== $v"; cat gpurun_out/ld_table_$v.txt
  PLGPU_LIB=$L timeout 300 python tools/probe_c4.py $v >> gpurun_out/ld_probe.jsonl 2>/dev/null
done
cat gpurun_out/ld_probe.jsonl
PLGPU_LIB=_variants/lead256.so timeout 1200 python bench.py --no-side --no-stages > gpurun_out/ld_bench256.json 2> gpurun_out/ld_bench256.err; echo bench=$?
