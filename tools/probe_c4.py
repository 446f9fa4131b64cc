"""c4 budget probe of one library build (bench.py's calibration: every node overloaded, budgets of
1 us at tau0 = 20 ns, 148 streams): per-node max and mean firing times, plus the time of a
logical-clock c4 run.  PLGPU_LIB=<build>.so python tools/probe_c4.py <label>"""
import json
import os
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

base = C.c4()
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
b, st = realtime.calibrate_budgets(base, wl, db.data_ptr(), reps=3, margin=1.0, slack_ns=0, probe_t=1000,
                                   probe_tau=20, over=over)
mean = [round(st["busy_ns"][i] / max(1, st["firings"][i])) for i in range(4)]
walls = []
for _ in range(2):
    pl = Pipeline(base.replace(wait_time=(993, 2422, 965, 1628)), wl, **over)
    pl.bind_device(db.data_ptr(), wl.db_len)
    pl.drain()
    walls.append(pl.stats()["wall_ns"])
    pl.close()
print(json.dumps({"build": sys.argv[1] if len(sys.argv) > 1 else "in-tree", "max_fire_ns": list(b),
                  "mean_fire_ns": mean, "logical_wall_ms": min(walls) / 1e6}), flush=True)
