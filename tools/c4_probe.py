"""Service-time probes on c4: per-node firing durations (max and mean) with every node firing full
vectors at a generous period (probe_t, the default calibration) and with every node overloaded
(probe_t small: each node fires back to back, so all four share the SM -- the 1/N processor
share at which PAPER.md L69 defines t_i).  argv: probe_t_ns[,probe_t_ns...] [reps]"""
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import realtime

ts = [int(x) for x in (sys.argv[1] if len(sys.argv) > 1 else "20000,1000").split(",")]
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 2
base = C.c4()
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
for pt in ts:
    b, st = realtime.calibrate_budgets(base, wl, db.data_ptr(), over=over, probe_t=pt, probe_tau=20, margin=1.1,
                                       slack_ns=128, reps=reps)
    print(json.dumps({"probe_t": pt, "budgets": b, "max_fire_runs": st["max_fire_ns_runs"],
                      "mean_fire": [round(st["busy_ns"][i] / max(1, st["firings"][i])) for i in range(4)],
                      "max_loop": st["max_loop_ns"], "spilled": st["spilled"], "lateness": st["max_lateness_ns"],
                      "wall_ms": st["wall_ns"] / 1e6}), flush=True)
