"""Per-node firing durations of one library build on c2 (the budget probe of bench.py: every node
fires full vectors at a generous period, 148 streams, physical clock), for bisecting per-firing
cost across commits: PLGPU_LIB=_variants/<build>.so python tools/bisect_fire.py <label>.
Prints one JSON line: max firing (min over 3 runs) and mean firing per node, and a logical-clock
c2 run's wall time."""
import json
import os
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

base = C.c2(n_streams=148)
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
b, st = realtime.calibrate_budgets(base, wl, db.data_ptr(), reps=3, margin=1.0, slack_ns=0)
mean = [round(st["busy_ns"][i] / max(1, st["firings"][i])) for i in range(4)]
lg = base.replace(wait_time=(993, 2422, 965, 1628))
walls = []
for _ in range(3):
    pl = Pipeline(lg, wl)
    pl.bind_device(db.data_ptr(), wl.db_len)
    pl.drain()
    walls.append(pl.stats()["wall_ns"])
    pl.close()
print(json.dumps({"build": sys.argv[1] if len(sys.argv) > 1 else os.environ.get("PLGPU_LIB", "in-tree"),
                  "variant_env": os.environ.get("PL_VARIANT"), "max_fire_ns": list(b), "mean_fire_ns": mean,
                  "logical_wall_us": min(walls) / 1e3}), flush=True)
