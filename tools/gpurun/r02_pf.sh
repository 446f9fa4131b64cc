# one gpurun call: S3 prefetch A/B on the c4 probe, plus its parity (DNA tests) with the variant
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for rep in 1 2; do
  timeout 300 python tools/probe_c4.py in-tree
  PLGPU_LIB=_variants/x_pf.so timeout 300 python tools/probe_c4.py prefetch
done
PLGPU_LIB=_variants/x_pf.so timeout 900 python -m pytest tests/test_gpu_parity.py tests/test_gpu_window.py -m gpu -q -k "dna or window or vector" > gpurun_out/r02_pf_parity.log 2>&1; echo pf_parity=$? >&2; tail -1 gpurun_out/r02_pf_parity.log >&2
