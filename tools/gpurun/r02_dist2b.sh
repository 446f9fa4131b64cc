# one gpurun call: bench.py's N>1 path on the final build (2 ranks sharing the one GPU, gloo), c2 and the reference arm
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
PL_BENCH_SHARE_GPU=1 PL_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 3 --warmup 3 --workload c2 --no-side \
  --no-cpu-baseline > gpurun_out/r02_dist2b.json 2> gpurun_out/r02_dist2b.log; echo dist_rc=$?; tail -c 400 gpurun_out/r02_dist2b.json
timeout 600 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/r02_ref.json 2> gpurun_out/r02_ref.log; echo ref_rc=$?; tail -c 300 gpurun_out/r02_ref.json
