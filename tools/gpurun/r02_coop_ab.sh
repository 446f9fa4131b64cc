# one gpurun call: S3 hybrid walk (PL_S3_COOP) A/B on the c4 budget probe, plus the DNA parity
# tests with the variants (tools/build_variant.py builds them into _variants/)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
  for v in in-tree coop coop_s4c4 coop_s8c8 coop_s16c2; do
    if [ $v = in-tree ]; then timeout 300 python tools/probe_c4.py $v; else PLGPU_LIB=_variants/$v.so timeout 300 python tools/probe_c4.py $v; fi
  done
done > gpurun_out/r02_coop_ab.jsonl 2> gpurun_out/r02_coop_ab.err
for v in coop coop_s4c4 coop_s16c2; do
  PLGPU_LIB=_variants/$v.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window.py tests/test_gpu_c4.py -m gpu -q -x > gpurun_out/r02_coop_parity_$v.log 2>&1; echo parity_$v=$?; tail -1 gpurun_out/r02_coop_parity_$v.log
done
