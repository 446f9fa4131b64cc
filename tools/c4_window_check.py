"""Is c4's FIXED_WAIT lateness a window-cap effect?  c4's recipe (heavy-tailed repeat islands)
at two DB sizes: per-stream length inside the 64 KB smem window (200 kbp) and the full c4
(708 kbp, window capped: S0 beyond it reads HBM).  Physical clock, D = 1 ms, paper b, slow
arrival rates; per node: max lateness, overruns; misses; max latency.
argv: [per_stream_bases,...]"""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

sizes = [int(x) for x in sys.argv[1].split(",")] if len(sys.argv) > 1 else [200_000, 708_497]
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
for per in sizes:
    base = C.c4()
    L = per * 148
    base = base.replace(dna=dict(base.dna, db_len=L, n_planted=max(64, base.dna["n_planted"] * L // base.dna["db_len"])))
    wl = G.make_dna(base.seed, **base.dna)
    db = torch.from_numpy(wl.db.view("int32")).cuda()
    ptr = db.data_ptr()
    gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr, over=over)
    budgets, cal = realtime.calibrate_budgets(base, wl, ptr, over=over, probe_tau=20)
    cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=1_000_000,
                       b=C.PAPER_B, eager_drain=True)
    for tau in (5000, 20000):
        sol = realtime.solve_at(cfg, tau)
        if sol is None:
            print(json.dumps({"per_stream": per, "tau0": tau, "fig1": "infeasible"}), flush=True)
            continue
        c = cfg.replace(interarrival=tau, wait_time=tuple(sol[0]))
        pl = Pipeline(c, wl, flags=0, **over)
        pl.bind_device(ptr, wl.db_len)
        pl.drain()
        s = pl.stats()
        pl.close()
        print(json.dumps({"per_stream": per, "tau0": tau, "budgets": budgets, "gains": [round(g, 3) for g in gains],
                          "lateness": s["max_lateness_ns"], "overruns": s["overruns"], "misses": s["miss_events_ns"],
                          "max_latency_ns": s["max_latency_ns"], "max_fire": s["max_fire_ns"],
                          "stalls": s["stalls"], "spilled": s["spilled"]}), flush=True)
    del db
