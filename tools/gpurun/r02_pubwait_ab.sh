# one gpurun call: PL_PUB_WAIT A/B (waiting leaders sleep on the input edge's mbarrier, woken by the producer's
# publication): c3 issue counts (ncu), the c4 budget probe, the physical-clock parity tests and the bench with it
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
M=gpu__time_duration.sum,smsp__issue_active.avg.pct_of_peak_sustained_active,smsp__inst_executed.sum,sm__throughput.avg.pct_of_peak_sustained_elapsed
for v in base pubwait; do
  if [ $v = base ]; then L=; else L=_variants/$v.so; fi
  PLGPU_LIB=$L timeout 900 ncu --nvtx --nvtx-include "measure/" --metrics $M --clock-control none --csv --log-file gpurun_out/pw_ncu_$v.csv python tools/ncu_c3_points.py > gpurun_out/pw_pts_$v.jsonl 2> gpurun_out/pw_pts_$v.err
  python tools/ncu_c3_table.py gpurun_out/pw_ncu_$v.csv gpurun_out/pw_pts_$v.jsonl > gpurun_out/pw_table_$v.txt 2>&1; echo "== $v"; cat gpurun_out/pw_table_$v.txt
  PLGPU_LIB=$L timeout 300 python tools/probe_c4.py $v >> gpurun_out/pw_probe.jsonl 2>/dev/null
done
cat gpurun_out/pw_probe.jsonl
PLGPU_LIB=_variants/pubwait.so timeout 900 python -m pytest tests/test_gpu_fullsize.py tests/test_gpu_agreement.py tests/test_gpu_parity.py tests/test_gpu_live.py tests/test_gpu_window.py -m gpu -q > gpurun_out/pw_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/pw_tests.log
PLGPU_LIB=_variants/pubwait.so timeout 1200 python bench.py --no-side --no-stages > gpurun_out/pw_bench.json 2> gpurun_out/pw_bench.err; echo bench=$?
