"""N4 on c4 (the verdict's "c4 rate comparison"): the cluster executor (one node
per CTA of a 4-CTA cluster, PL_CLUSTER_NODES) against the one-CTA-per-stream executor, both by
bench.py's procedure -- gains from a logical run, budgets from an overloaded physical probe of
the same kernel, THRESHOLD_SLACK with Fig. 1 thresholds at D - SG, and the fastest tau0 with zero
measured misses across 1.8 ms stalls injected every 100 ms (R-STALL).

The same 100 Mbp heavy-tailed DB is split into 148 streams for the one-CTA executor (one SM per
stream, its four nodes sharing it) and into 37 streams for N4 (four SMs per stream, one per
node): items/s per GPU and per SM are the comparable numbers.
Prints one JSON line per variant; argv: [--quick]."""
import json
import sys
import time

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import realtime
from paper_conf_icppw_planob21_b200._pl import PL_CLUSTER_NODES, PL_FIXED_SERVICE

D, SG = 3_500_000, 2_700_000
INJECT = (100_000_000, 1_800_000)


def evaluate(name, streams, extra_flags, wl, db_ptr, over):
    t0 = time.time()
    base = C.c4(n_streams=streams)
    gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, db_ptr, over=over)
    budgets, cal = realtime.calibrate_budgets(base, wl, db_ptr, margin=1.1, slack_ns=128, probe_tau=20, over=over,
                                              probe_t=1000, flags=extra_flags)
    cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B,
                       slack_guard=int(max(budgets)) + SG)
    log = lambda d: print(json.dumps(dict(variant=name, **d)), file=sys.stderr, flush=True)
    tau, w, th, T, st = realtime.find_rate(cfg, wl, db_ptr, log=log, policy=1, over=over, max_lateness_ns=None,
                                           grow=1.5, tries=16, flags=PL_FIXED_SERVICE | extra_flags,
                                           solve_deadline=D - SG, inject=INJECT)
    # one clean run at the operating point (no injection): misses, utilisation, per-node firing times
    run = cfg.replace(interarrival=tau, wait_time=tuple(w), wait_threshold=tuple(th), policy=1)
    sx = realtime._run(run, db_ptr, wl.db_len, wl, flags=PL_FIXED_SERVICE | extra_flags, over=over)
    sms = streams * (4 if extra_flags & PL_CLUSTER_NODES else 1)
    return {"variant": name, "streams": streams, "sms_used": min(sms, 148), "budgets_ns": list(budgets),
            "probe_max_fire_ns": cal["max_fire_ns_runs"], "tau0_ns": tau, "theta": list(th),
            "items_per_s": streams * 1e9 / tau, "items_per_s_per_sm": streams * 1e9 / tau / min(sms, 148),
            "check_run": {"misses": sx["miss_events_ns"], "errors": sx["errors"],
                          "max_latency_ns": sx["max_latency_ns"], "max_fire_ns": sx["max_fire_ns"],
                          "mean_fire_ns": [round(sx["busy_ns"][i] / max(1, sx["firings"][i])) for i in range(4)],
                          "hw_busy_fraction": sx["hw_busy_fraction"], "active_fraction": sx["active_fraction"],
                          "stalled": realtime.stalled(sx)},
            "search_s": round(time.time() - t0, 1)}


def main():
    base = C.c4()
    wl = G.make_dna(base.seed, **base.dna)
    db = torch.from_numpy(wl.db.view("int32")).cuda()
    over = dict(match_capacity=1 << 25, spill_capacity=1 << 19)
    for name, streams, fl in (("one_cta_per_stream", 148, 0), ("n4_cluster", 37, PL_CLUSTER_NODES)):
        print(json.dumps(evaluate(name, streams, fl, wl, db.data_ptr(), over)), flush=True)


if __name__ == "__main__":
    main()
