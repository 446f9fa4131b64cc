"""c4 (BASELINE configs[3]): 100 Mbp heavy-tailed DB, 148 streams, physical clock.
Budgets from a full-vector probe (probe tau0 = 20 ns: node 0 always fires full vectors and
the repeat islands drive node 1 to full vectors with up to u = 16 outputs each), R-DRAIN end
of stream, the fastest miss-free rate with the paper's b, then with b calibrated on the
device from the streams' input-queue peaks (realtime.calibrate_b).
argv: [deadline_ns] [max_lateness_ns or "none"] (runs longer than ~1 s meet ~1.7 ms platform
pauses, profiles/r01_globaltimer_pauses.txt, so long c4 runs need D well above that and no
lateness bound)"""
import json
import sys
import time

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

D = int(sys.argv[1]) if len(sys.argv) > 1 else 1_000_000
ML = None if len(sys.argv) > 2 and sys.argv[2] == "none" else (int(sys.argv[2]) if len(sys.argv) > 2 else 5000)
log = lambda d: print(json.dumps(d), flush=True)
base = C.c4()
t0 = time.time()
wl = G.make_dna(base.seed, **base.dna)
log({"gen_s": round(time.time() - t0, 1), "db_len": wl.db_len, "planted": len(wl.planted)})
db = torch.from_numpy(wl.db.view("int32")).cuda()
ptr = db.data_ptr()
over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr, over=over)
budgets, cal = realtime.calibrate_budgets(base, wl, ptr, over=over, probe_tau=20)
log({"gains": gains, "budgets_ns": budgets, "cal_max_fire_ns": cal["max_fire_ns"], "cal_stalls": cal["stalls"],
     "cal_spilled": cal["spilled"]})
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
            "overruns": st["overruns"], "stalls": st["stalls"], "spilled": st["spilled"],
            "max_latency_ns": st["max_latency_ns"], "active_fraction": st["active_fraction"],
            "hw_busy": st["hw_busy_fraction"], "matches": st["matches"], "errors": st["errors"]}


for label, c in (("paper_b", cfg),):
    try:
        tau, w, th, T, st = realtime.find_rate(c, wl, ptr, over=over, grow=1.6, tries=14, max_lateness_ns=ML,
                                               log=lambda d: log(dict(d, search=label)))
        log({"result": label, "D": D, "b": list(c.b), "tau0": tau, "w": list(w), "sustained": 148e9 / tau,
             **timed(c.replace(interarrival=tau, wait_time=tuple(w)))})
    except RuntimeError as ex:
        log({"result": label, "failed": str(ex)})

# b calibrated on the device at 1.5x the Fig. 1 feasibility limit of b = 1
tau_c = int(1.5 * realtime.min_feasible_tau(cfg.replace(b=(1,) * 4)))
cb = realtime.calibrate_b(cfg.replace(interarrival=tau_c), wl, ptr, target=1.0, quantile=1.0, max_iter=8, over=over,
                          log=lambda d: log(dict(d, calib_tau0=tau_c)))
log({"calibrated_b": list(cb["b"]), "miss_free": cb["miss_free"], "iterations": cb["iterations"]})
c2 = cfg.replace(b=tuple(cb["b"]))
try:
    tau, w, th, T, st = realtime.find_rate(c2, wl, ptr, over=over, grow=1.6, tries=14, max_lateness_ns=ML,
                                           log=lambda d: log(dict(d, search="calibrated_b")))
    log({"result": "calibrated_b", "D": D, "b": list(c2.b), "tau0": tau, "w": list(w), "sustained": 148e9 / tau,
         **timed(c2.replace(interarrival=tau, wait_time=tuple(w)))})
except RuntimeError as ex:
    log({"result": "calibrated_b", "failed": str(ex)})

# THRESHOLD_SLACK (the north_star rule; theta from Fig. 1, slack guard = the largest budget):
# it fires on queue size or deadline slack, so it can absorb the repeat islands' bursts
ct = cfg.replace(slack_guard=int(max(budgets)))
try:
    tau, w, th, T, st = realtime.find_rate(ct, wl, ptr, over=over, grow=1.6, tries=14, policy=1, max_lateness_ns=ML,
                                           log=lambda d: log(dict(d, search="threshold_slack")))
    log({"result": "threshold_slack", "D": D, "theta": list(th), "tau0": tau, "sustained": 148e9 / tau,
         **timed(ct.replace(interarrival=tau, wait_threshold=tuple(th), policy=1))})
except RuntimeError as ex:
    log({"result": "threshold_slack", "failed": str(ex)})

# MONOLITHIC (Fig. 2's block size M; no internal waiting): the fastest miss-free tau0
tau = realtime.min_feasible_tau(cfg) or 1
found = None
for _ in range(16):
    Mm = realtime.monolithic_at(cfg, tau)
    if Mm is not None:
        r = timed(cfg.replace(interarrival=tau, policy=2, block_size=Mm[0]))
        log(dict(r, search="monolithic", tau0=tau, M=Mm[0]))
        if r["misses_ns"] == 0 and r["errors"] == 0:
            found = (tau, Mm[0], r)
            break
    tau = int(tau * 1.6) + 1
if found:
    log({"result": "monolithic", "D": D, "tau0": found[0], "M": found[1], "sustained": 148e9 / found[0], **found[2]})
else:
    log({"result": "monolithic", "failed": "no miss-free tau0 found"})
