"""Hardware utilisation of enforced waiting vs the monolithic baseline at the same (tau0, D)
(SURVEY §8(d) "Hardware utilisation"): one physical-clock launch of each policy on the c2
workload with the bench's B200 budgets; run it under
  ncu --metrics <list> -k regex:pl_exec python tools/hw_util.py tau0 [D]
and summarise with tools/ncu_summary.py.  Without ncu it prints each run's model-level
statistics (active fraction, measured busy fraction, misses)."""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

tau = int(sys.argv[1]) if len(sys.argv) > 1 else 27
D = int(sys.argv[2]) if len(sys.argv) > 2 else 350_000
budgets = (1642, 2768, 3121, 12167)
gains = (0.22344, 1.14693, 0.07856)
base = C.c2(n_streams=148).replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D,
                                    b=C.PAPER_B, eager_drain=True, interarrival=tau)
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
sol = realtime.solve_at(base, tau)
mono = realtime.monolithic_at(base, tau)
runs = []
if sol is not None:
    runs.append(("enforced", base.replace(wait_time=tuple(sol[0]))))
if mono is not None:
    runs.append(("monolithic", base.replace(policy=C.MONOLITHIC, block_size=mono[0])))
for name, cfg in runs:
    pl = Pipeline(cfg, wl, flags=0)
    pl.bind_device(db.data_ptr(), wl.db_len)
    pl.drain()
    s = pl.stats()
    pl.close()
    print(json.dumps({"policy": name, "tau0_ns": tau, "D_ns": D, "active_fraction": s["active_fraction"],
                      "hw_busy_fraction": s["hw_busy_fraction"], "wall_us": s["wall_ns"] / 1e3,
                      "misses": s["miss_events_ns"], "M": mono[0] if name == "monolithic" else None}), flush=True)
