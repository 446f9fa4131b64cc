# one gpurun call: c4 rate vs the platform-stall allowance SG (D = 3.5 ms), injected-stall criterion
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
for sg in 2200000 3000000; do
  timeout 900 python bench.py --no-side --no-e2e --no-cpu-baseline --stall-guard-ns $sg --steps 10 > gpurun_out/r02_bench_sg$sg.json 2> gpurun_out/r02_bench_sg$sg.log; echo sg$sg rc=$?
done
