"""Threshold slack-guard sweep: THRESHOLD_SLACK at guards {0, 2e4, 6e4} on the physical clock."""
import json, sys
sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime
base = C.c2(n_streams=148)
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda(); ptr = db.data_ptr()
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr)
budgets, _ = realtime.calibrate_budgets(base, wl, ptr)
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=350_000, b=C.PAPER_B)
for guard in (0, 20000, 60000):
    for tau in (25, 40, 80, 160):
        sol = realtime.solve_at(cfg, tau)
        if sol is None: continue
        w, th, T = sol
        for logical in (False, True):
            c = cfg.replace(interarrival=tau, wait_threshold=tuple(th), policy=1, slack_guard=guard,
                            clock=0 if logical else 1)
            if logical:
                c = c.replace(service_time=budgets)
            pl = Pipeline(c, wl, flags=1)
            pl.bind_device(ptr, wl.db_len)
            pl.drain()
            st = pl.stats()
            pl.close()
            print(json.dumps({"guard": guard, "tau": tau, "logical": logical, "theta": th, "misses": st["misses"],
                              "miss_ns": st["miss_events_ns"], "sched_miss": st["miss_events"],
                              "maxlat": st["max_latency"], "maxlat_ns": st["max_latency_ns"],
                              "stalls": st["stalls"], "late": st["max_lateness_ns"], "firings": st["firings"]}), flush=True)
