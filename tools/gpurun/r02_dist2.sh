# one gpurun call: bench.py's N>1 path (2 ranks sharing the one GPU, gloo for the collectives)
python paper_conf_icppw_planob21_b200/build.py --force >/dev/null
PL_BENCH_SHARE_GPU=1 PL_DIST_BACKEND=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 \
  --master-addr 127.0.0.1 --master-port 29517 bench.py --gpus 2 --steps 3 --warmup 3 --workload c2 --no-side \
  --no-cpu-baseline > gpurun_out/r02_dist2.json 2> gpurun_out/r02_dist2.log; echo dist_rc=$?
timeout 600 python -m pytest tests/test_gpu_agreement.py -m gpu -q -rs -s > gpurun_out/r02_agree_rs.log 2>&1; echo agree_rc=$?
