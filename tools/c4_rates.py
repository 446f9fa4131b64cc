"""c4 (BASELINE configs[3]) rate search, round 2: the 100 Mbp heavy-tailed DB, 148 full-length
streams (708 K roots each) through the sliding smem window, physical clock.

Budgets from the full-vector probe (realtime.calibrate_budgets), then for each policy the fastest
miss-free tau0 (no lateness bound: runs this long meet the platform's ~1.6 ms SM stalls,
profiles/r02_pause_control.txt).  argv: D_ns [policies, e.g. "thr,mono,fixed"] [slack_guard_extra_ns]
"""
import json
import sys
import time

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

D = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
POL = (sys.argv[2] if len(sys.argv) > 2 else "thr,mono").split(",")
EXTRA = int(sys.argv[3]) if len(sys.argv) > 3 else 0
log = lambda d: print(json.dumps(d), flush=True)
t_start = time.time()
base = C.c4()
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
ptr = db.data_ptr()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr, over=over)
budgets, cal = realtime.calibrate_budgets(base, wl, ptr, over=over, probe_tau=20, margin=1.1, slack_ns=128)
log({"gains": gains, "budgets_ns": budgets, "cal_max_fire_ns": cal["max_fire_ns"], "refills": cal["window_refills"],
     "cal_spilled": cal["spilled"], "t": round(time.time() - t_start, 1)})
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B,
                   eager_drain=True)


def timed(c):
    pl = Pipeline(c, wl, flags=0, **over)
    pl.bind_device(ptr, wl.db_len)
    pl.launch()
    pl.summary()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    pl.launch()
    e1.record()
    torch.cuda.synchronize()
    st = pl.stats()
    pl.close()
    ms = e0.elapsed_time(e1)
    return {"ms": ms, "items_per_s": st["roots"] / ms * 1e3, "misses_ns": st["miss_events_ns"],
            "overruns": st["overruns"], "spilled": st["spilled"], "max_latency_ns": st["max_latency_ns"],
            "max_lateness_ns": st["max_lateness_ns"], "max_fire_ns": st["max_fire_ns"],
            "active_fraction": st["active_fraction"], "hw_busy": st["hw_busy_fraction"], "matches": st["matches"],
            "refills": st["window_refills"], "errors": st["errors"]}


if "thr" in POL:
    ct = cfg.replace(slack_guard=int(max(budgets)) + EXTRA)
    try:
        tau, w, th, T, st = realtime.find_rate(ct, wl, ptr, over=over, grow=1.5, tries=16, policy=1,
                                               max_lateness_ns=None,
                                               log=lambda d: log(dict(d, search="threshold_slack")))
        log({"result": "threshold_slack", "D": D, "theta": list(th), "tau0": tau, "sustained": 148e9 / tau,
             **timed(ct.replace(interarrival=tau, wait_threshold=tuple(th), policy=1)),
             "t": round(time.time() - t_start, 1)})
    except RuntimeError as ex:
        log({"result": "threshold_slack", "failed": str(ex)})

if "fixed" in POL:
    cf = cfg.replace(deadline=D - EXTRA)
    try:
        tau, w, th, T, st = realtime.find_rate(cf, wl, ptr, over=over, grow=1.5, tries=16, max_lateness_ns=None,
                                               log=lambda d: log(dict(d, search="fixed_wait")))
        log({"result": "fixed_wait", "D": D, "w": list(w), "tau0": tau, "sustained": 148e9 / tau,
             **timed(cf.replace(interarrival=tau, wait_time=tuple(w))), "t": round(time.time() - t_start, 1)})
    except RuntimeError as ex:
        log({"result": "fixed_wait", "failed": str(ex)})

if "mono" in POL:
    tau = realtime.min_feasible_tau(cfg) or 1
    found, bad = None, None
    for _ in range(20):
        Mm = realtime.monolithic_at(cfg.replace(deadline=D - EXTRA), tau)
        if Mm is not None:
            r = timed(cfg.replace(interarrival=tau, policy=2, block_size=Mm[0]))
            log(dict(r, search="monolithic", tau0=tau, M=Mm[0]))
            if r["misses_ns"] == 0 and r["errors"] == 0:
                found = (tau, Mm[0], r)
                break
            bad = tau
        tau = int(tau * 1.3) + 1
    if found:
        log({"result": "monolithic", "D": D, "tau0": found[0], "M": found[1], "sustained": 148e9 / found[0],
             **found[2], "t": round(time.time() - t_start, 1)})
    else:
        log({"result": "monolithic", "failed": "no miss-free tau0 found"})
