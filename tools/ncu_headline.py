"""One launch each of the bench's c4 headline kernel (THRESHOLD_SLACK, PL_FIXED_SERVICE) and of the
MONOLITHIC baseline at the same (tau0, D), for `ncu --set full` (hardware utilisation of enforced
waiting vs the no-wait baseline; SURVEY 8(d) "Hardware utilisation").
Parameters come from the committed bench line (profiles/r02_bench_c4_v1.json) unless given.
argv: [bench_json] [--streams S]  (S < 148 shortens nothing: every stream is full length)"""
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime
from paper_conf_icppw_planob21_b200._pl import PL_FIXED_SERVICE

src = sys.argv[1] if len(sys.argv) > 1 else "profiles/r02_bench_c4_inject.json"
b = json.load(open(src))["config"]
budgets, tau, D, SG, gains = tuple(b["budgets_ns"]), b["tau0_ns"], b["deadline_ns"], b["stall_guard_ns"], tuple(b["gains"])
base = C.c4()
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B)
w, th, T = realtime.solve_at(cfg.replace(deadline=D - SG), tau)
thr = cfg.replace(interarrival=tau, wait_time=tuple(w), wait_threshold=tuple(th), policy=1,
                  slack_guard=max(budgets) + SG)
M, _ = realtime.monolithic_at(cfg.replace(deadline=D - SG, policy=2), tau)
mono = cfg.replace(interarrival=tau, policy=2, block_size=M)
for name, c, fl in (("threshold_slack", thr, PL_FIXED_SERVICE), ("monolithic", mono, 0)):
    pl = Pipeline(c, wl, flags=fl, **over)
    pl.bind_device(db.data_ptr(), wl.db_len)
    pl.launch()
    st = pl.stats()
    pl.close()
    print(json.dumps({"policy": name, "tau0_ns": tau, "roots": st["roots"], "matches": st["matches"],
                      "misses": st["miss_events_ns"], "active_fraction": st["active_fraction"],
                      "hw_busy_fraction": st["hw_busy_fraction"], "wall_ms": st["wall_ns"] / 1e6,
                      "algorithmic_bytes": 0.25 * st["roots"] + 24 * st["matches"]}), flush=True)
