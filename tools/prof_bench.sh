set -x
timeout 600 python bench.py --steps 20 --warmup 5 > gpurun_out/bench_v8.log 2>&1
tail -1 gpurun_out/bench_v8.log > gpurun_out/bench_v8.json
# bench parameters for the captures
P=$(python - <<'PY'
import json
d=json.load(open("gpurun_out/bench_v8.json"))
c=d["config"]
print(c["tau0_ns"], *c["budgets_ns"], *c["w_ns"], c["deadline_ns"], 0, 0, 1)
PY
)
echo "params $P"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_v8.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline > gpurun_out/bench_under_ncu.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:pl_exec_enforced -c 1 -o gpurun_out/exec_v8 python tools/run_bench_cfg.py $P > gpurun_out/ncu_full.log 2>&1
