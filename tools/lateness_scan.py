"""Node-0 lateness vs tau0 at the bench's budgets (physical clock, c2, eager drain): for each
tau0, Fig. 1's waits, `reps` launches, the max node-0 lateness (ns) and loop time per launch.
A node whose loop exceeds its period P_0 falls behind: the lateness grows with tau0 shrinking.
argv: t0 t1 t2 t3 tau0,... [reps] [db_len]"""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

t = tuple(int(x) for x in sys.argv[1:5])
taus = [int(x) for x in sys.argv[5].split(",")]
reps = int(sys.argv[6]) if len(sys.argv) > 6 else 3
dbl = int(sys.argv[7]) if len(sys.argv) > 7 else 1 << 20
base = C.c2(n_streams=148, dna=dict(db_len=dbl, q_len=1024, n_planted=64 * dbl // (1 << 20)))
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
import os
gains = (tuple(float(x) for x in os.environ["GAINS"].split(",")) if os.environ.get("GAINS")
         else realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, db.data_ptr()))
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=t, gain=gains, deadline=350_000, b=C.PAPER_B,
                   eager_drain=True)
for tau in taus:
    w, th, T = realtime.solve_at(cfg, tau)
    c = cfg.replace(interarrival=tau, wait_time=tuple(w))
    lat, loop, miss = [], [], 0
    for _ in range(reps):
        pl = Pipeline(c, wl, flags=0)
        pl.bind_device(db.data_ptr(), wl.db_len)
        pl.drain()
        s = pl.stats()
        pl.close()
        lat.append(s["max_lateness_ns"][0])
        loop.append(s["max_loop_ns"][0])
        miss += s["miss_events_ns"]
    print(json.dumps({"tau0": tau, "w0": w[0], "lateness0": lat, "max_loop0": loop, "misses": miss}), flush=True)
