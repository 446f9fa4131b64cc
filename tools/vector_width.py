"""Physical budgets and the sustained-rate bound (streams * v / t_0) vs the vector width v."""
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import realtime

base0 = C.c2(n_streams=148)
wl = G.make_dna(base0.seed, **base0.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
for v in (64, 128, 256):
    base = base0.replace(vector_width=v)
    budgets, cal = realtime.calibrate_budgets(base, wl, db.data_ptr(), probe_tau=50)
    mean = [round(cal["busy_ns"][i] / max(1, cal["firings"][i])) for i in range(4)]
    print(json.dumps({"v": v, "budgets": budgets, "max_fire": cal["max_fire_ns"], "mean_fire": mean,
                      "sustained_bound_items_per_s": 148 * v * 1e9 / budgets[0],
                      "per_item_ns_node0": budgets[0] / v}), flush=True)
