"""c4: 100 Mbp heavy-tailed DB, one stream per SM (148), logical then physical clock.
Reports spills, misses and items/s; physical rate found as in bench.py."""
import json
import sys
import time

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime, solve_enforced_waits

D = int(sys.argv[1]) if len(sys.argv) > 1 else 350_000
import subprocess
smi = subprocess.Popen(["nvidia-smi", "--query-gpu=clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active",
                        "--format=csv,noheader", "-lms", "500"], stdout=open("gpurun_out/c4_clocks.csv", "w"))
base = C.c4()
t0 = time.time()
wl = G.make_dna(base.seed, **base.dna)
print(json.dumps({"gen_s": time.time() - t0, "db_len": wl.db_len, "planted": len(wl.planted)}), flush=True)
db = torch.from_numpy(wl.db.view("int32")).cuda()
ptr = db.data_ptr()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
w, th, T, Tc = solve_enforced_waits(base.replace(gain=C.TABLE1_G))
lc = base.replace(wait_time=tuple(w))
pl = Pipeline(lc, wl, flags=0, **over)
pl.bind_device(ptr, wl.db_len)
for _ in range(2):
    pl.launch()
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
pl.launch()
e1.record()
torch.cuda.synchronize()
st = pl.stats()
ms = e0.elapsed_time(e1)
pl.close()
print(json.dumps({"mode": "logical", "ms": ms, "roots": st["roots"], "items_per_s": st["roots"] / ms * 1e3,
                  "consumed": st["consumed"], "produced": st["produced"], "spilled": st["spilled"],
                  "matches": st["matches"], "misses": st["miss_events"], "errors": st["errors"]}), flush=True)
gains = tuple(st["produced"][i] / max(1, st["consumed"][i]) for i in range(3))
budgets, cal = realtime.calibrate_budgets(base, wl, ptr, over=over, probe_tau=2000)
print(json.dumps({"gains": gains, "budgets": budgets, "cal_max_fire": cal["max_fire_ns"],
                  "cal_spilled": cal["spilled"], "cal_errors": cal["errors"]}), flush=True)
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B)
try:
    tau, w, th, T, st = realtime.find_rate(cfg, wl, ptr, log=lambda d: print(json.dumps(d), flush=True), over=over, grow=2.0, tries=14)
    rc = cfg.replace(interarrival=tau, wait_time=tuple(w))
    pl = Pipeline(rc, wl, flags=0, **over)
    pl.bind_device(ptr, wl.db_len)
    pl.launch()
    torch.cuda.synchronize()
    e0.record()
    pl.launch()
    e1.record()
    torch.cuda.synchronize()
    st = pl.stats()
    ms = e0.elapsed_time(e1)
    pl.close()
    print(json.dumps({"mode": "physical", "D": D, "tau0": tau, "ms": ms, "items_per_s": st["roots"] / ms * 1e3,
                      "sustained": 148e9 / tau, "misses": st["miss_events"], "overruns": st["overruns"],
                      "spilled": st["spilled"], "max_latency_ns": st["max_latency_ns"], "errors": st["errors"],
                      "active_fraction": st["active_fraction"], "hw_busy": st["hw_busy_fraction"]}), flush=True)
except RuntimeError as ex:
    print(json.dumps({"physical": "failed", "why": str(ex)}), flush=True)

smi.terminate()
