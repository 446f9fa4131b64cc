"""A/B of catch-up batching (executor.cu peek_next) on c4 at FIXED budgets: the bench's procedure
(gains, overloaded 1 us probe, THRESHOLD_SLACK, D = 3.5 ms, SG = 2.7 ms) and its injected-stall
rate search, once with batching (PL_VARIANT=1, the default) and once without (PL_VARIANT=9), with
the same budgets, so that only the executor differs.  Prints one JSON line per variant."""
import json
import os
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import realtime
from paper_conf_icppw_planob21_b200._pl import PL_FIXED_SERVICE

D, SG = 3_500_000, 2_700_000
INJECT = (100_000_000, 1_800_000)
base = C.c4()
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, db.data_ptr(), over=over)
budgets, _ = realtime.calibrate_budgets(base, wl, db.data_ptr(), margin=1.1, slack_ns=128, probe_tau=20, over=over,
                                        probe_t=1000)
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B,
                   slack_guard=int(max(budgets)) + SG)
print(json.dumps({"budgets_ns": list(budgets), "gains": list(gains)}), flush=True)
for name, var in (("batching", "1"), ("no_batching", "9"), ("batching_again", "1")):
    os.environ["PL_VARIANT"] = var
    tau, w, th, T, st = realtime.find_rate(cfg, wl, db.data_ptr(), policy=1, over=over, max_lateness_ns=None,
                                           grow=1.5, tries=16, flags=PL_FIXED_SERVICE, solve_deadline=D - SG,
                                           inject=INJECT)
    print(json.dumps({"variant": name, "PL_VARIANT": var, "tau0_ns": tau, "items_per_s": 148e9 / tau,
                      "batched_firings": st["batched_firings"][:4], "max_lateness_ns": st["max_lateness_ns"],
                      "overruns": st["overruns"]}), flush=True)
