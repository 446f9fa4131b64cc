"""Hardware utilisation of enforced waiting vs the no-wait baseline where the paper says enforced
waiting should win (fast arrivals, loose deadlines; SURVEY 8(d) "Hardware
utilisation"; north_star "enforced waiting below the baseline's SM utilisation").  The c3 DNA
workload of tools/sweep_c3_dna.py (c2's pipeline, 148 streams x 50,000 roots, budgets calibrated on
this GPU), one physical launch per policy at each (tau0, D) point -- THRESHOLD_SLACK (Fig. 1 thetas),
FIXED_WAIT (Fig. 1 waits) and MONOLITHIC (Fig. 2's M) -- each inside an NVTX range "measure" so
that `ncu --nvtx --nvtx-include "measure/"` captures exactly these launches (issue-active, warp
instructions; ncu_c3_table.py joins them with the JSON lines printed here).
argv: [tau0_ns:D_us ...]   (default 50:350 100:700 200:1000)"""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

PTS = [tuple(int(x) for x in a.split(":")) for a in sys.argv[1:]] or [(50, 350), (100, 700), (200, 1000)]
S, X = 148, 50_000
base = C.c2(n_streams=S)
L = S * X + base.stages[0].iparam[0] - 1
base = base.replace(dna=dict(base.dna, db_len=L, n_planted=base.dna["n_planted"] * L // (1 << 20)))
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
ptr = db.data_ptr()
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr)
budgets, _ = realtime.calibrate_budgets(base, wl, ptr, margin=1.10, slack_ns=128)
cfg0 = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, b=C.PAPER_B)
print(json.dumps({"streams": S, "roots_per_stream": X, "gains": gains, "budgets_ns": budgets}), flush=True)

for tau, D_us in PTS:
    cfg = cfg0.replace(interarrival=tau, deadline=D_us * 1000)
    runs = []
    sol = realtime.solve_at(cfg, tau)
    if sol is not None:
        w, th, T = sol
        runs.append(("threshold_slack", cfg.replace(wait_threshold=tuple(th), policy=1, slack_guard=int(max(budgets))),
                     {"theta": list(th)}))
        runs.append(("fixed_wait", cfg.replace(wait_time=tuple(w), policy=0), {"w_ns": list(w), "fig1_T": T}))
    Mm = realtime.monolithic_at(cfg, tau)
    if Mm is not None:
        runs.append(("monolithic", cfg.replace(policy=2, block_size=Mm[0]), {"M": Mm[0], "fig2_objective": Mm[1]}))
    for name, c, extra in runs:
        pl = Pipeline(c, wl, flags=0)
        pl.bind_device(ptr, wl.db_len)
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_push("measure")
        pl.launch()
        torch.cuda.synchronize()
        torch.cuda.nvtx.range_pop()
        st = pl.stats()
        pl.close()
        print(json.dumps({"tau0_ns": tau, "D_us": D_us, "policy": name, "roots": st["roots"],
                          "active_fraction": st["active_fraction"], "hw_busy_fraction": st["hw_busy_fraction"],
                          "misses": st["miss_events_ns"], "max_latency_us": st["max_latency_ns"] / 1e3, **extra}),
              flush=True)
