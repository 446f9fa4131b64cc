"""Executor throughput vs streams per GPU (1 or 2 CTAs per SM), c2 workload."""
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime, solve_enforced_waits

base0 = C.c2()
wl = G.make_dna(base0.seed, **base0.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
for S in (148, 296, 444):
    base = base0.replace(n_streams=S)
    w, th, T, Tc = solve_enforced_waits(base.replace(gain=C.TABLE1_G))
    pl = Pipeline(base.replace(wait_time=tuple(w)), wl, flags=0)
    pl.bind_device(db.data_ptr(), wl.db_len)
    for _ in range(3):
        pl.launch()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record()
    for _ in range(5):
        pl.launch()
    e1.record()
    torch.cuda.synchronize()
    st = pl.stats()
    pl.close()
    ms = e0.elapsed_time(e1) / 5
    budgets, cal = realtime.calibrate_budgets(base, wl, db.data_ptr())
    print(json.dumps({"streams": S, "logical_ms": ms, "logical_items_per_s": st["roots"] / ms * 1e3,
                      "cal_max_fire": cal["max_fire_ns"], "mean_fire": [round(cal["busy_ns"][i] / max(1, cal["firings"][i])) for i in range(4)],
                      "budgets": budgets, "sustained_bound": S * 128e9 / budgets[0]}), flush=True)
