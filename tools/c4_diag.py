"""c4 headline diagnostics: the bench's THRESHOLD_SLACK schedule run repeatedly at a fixed tau0,
with per-run per-node statistics, under variants (window size, queue capacity).
argv: tau0_ns budgets(comma) [runs] [variant ...] where a variant is name=key:value,... over
pl_config fields (e.g. win128=window_words:32768 q16k=queue_capacity:16384)."""
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime
from paper_conf_icppw_planob21_b200._pl import PL_FIXED_SERVICE

tau = int(sys.argv[1])
budgets = tuple(int(x) for x in sys.argv[2].split(","))
runs = int(sys.argv[3]) if len(sys.argv) > 3 else 6
variants = [("base", {})]
for v in sys.argv[4:]:
    name, kv = v.split("=", 1)
    variants.append((name, {k: int(x) for k, x in (p.split(":") for p in kv.split(","))}))
D, SG = 2_500_000, 1_700_000
base = C.c4()
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
gains = (0.04995395898599429, 8.946504731148144, 0.560928702174972)
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B,
                   slack_guard=max(budgets) + SG, policy=1)
w, th, T = realtime.solve_at(cfg.replace(deadline=D - SG), tau)
cfg = cfg.replace(interarrival=tau, wait_time=tuple(w), wait_threshold=tuple(th))
for name, over in variants:
    for r in range(runs):
        pl = Pipeline(cfg, wl, flags=PL_FIXED_SERVICE, match_capacity=1 << 25, spill_capacity=1 << 19, **over)
        pl.bind_device(db.data_ptr(), wl.db_len)
        pl.launch()
        st = pl.stats()
        pl.close()
        print(json.dumps({"variant": name, "run": r, "misses": st["miss_events_ns"], "outliers": st["latency_outliers"],
                          "lateness": st["max_lateness_ns"], "max_fire": st["max_fire_ns"], "max_loop": st["max_loop_ns"],
                          "overruns": st["overruns"], "spilled": st["spilled"], "max_queue": st["max_queue"],
                          "refills": st["window_refills"], "wall_ms": st["wall_ns"] / 1e6}), flush=True)
