# one gpurun call: PL_S3_TAB2 A/B (left and right table walks advanced together): K-BENCH S3, the c4 probe,
# the DNA parity tests with the variant, and the default bench with it
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for v in base s3tab2; do
  if [ $v = base ]; then L=; else L=_variants/$v.so; fi
  PLGPU_LIB=$L timeout 300 python tools/stage_bench.py 104857600 5 > gpurun_out/t2_kb_$v.jsonl 2>&1; echo "== $v"; tail -1 gpurun_out/t2_kb_$v.jsonl | cut -c1-110
  PLGPU_LIB=$L timeout 300 python tools/probe_c4.py $v >> gpurun_out/t2_probe.jsonl 2>/dev/null
done
cat gpurun_out/t2_probe.jsonl
PLGPU_LIB=_variants/s3tab2.so timeout 1200 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window.py tests/test_gpu_c4.py tests/test_gpu_fullsize.py tests/test_gpu_stage_batch.py tests/test_gpu_agreement.py -m gpu -q -x > gpurun_out/t2_tests.log 2>&1; echo tests=$?; tail -2 gpurun_out/t2_tests.log
PLGPU_LIB=_variants/s3tab2.so timeout 1200 python bench.py --no-side --no-stages > gpurun_out/t2_bench.json 2> gpurun_out/t2_bench.err; echo bench=$?
