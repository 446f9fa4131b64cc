"""c3 on the DNA pipeline itself (BASELINE configs[2]: "same pipeline swept over arrival rate and
deadline D to map where enforced waiting beats the no-wait baseline"), on the physical clock of
a B200: the BLAST seed -> enumerate -> window -> X-drop pipeline of c2, 148 streams of 50,000
roots each (the paper's stream length, L230), budgets t_i calibrated on this GPU
(realtime.calibrate_budgets: the longest firing x 1.1 + 128 ns), gains measured by a logical
run, b = (1, 3, 9, 6) (L230).

Per grid point (tau0 ns, D us), one physical launch per policy:
  FIXED_WAIT       w_i from Fig. 1 (L139-L151)              -- enforced waiting, the paper's method
  THRESHOLD_SLACK  theta_i from Fig. 1, slack guard = max t_i -- the north_star's firing rule
  MONOLITHIC       M from Fig. 2 (L165-L180)                 -- the no-internal-wait baseline
and reports the model active fraction (L75; enforced: (1/N) sum_i active_i / H, monolithic:
busy / H), the hardware busy fraction of the persistent CTAs, measured deadline misses and the
largest measured latency.  "infeasible" = the optimiser has no feasible point (Fig. 1 / Fig. 2).
Prints one JSON line per point, then the difference surface (enforced - monolithic active
fraction at points where both are miss-free), the paper's Fig. 4 analogue (L249).
argv: [streams] [roots_per_stream]"""
import json
import sys
import time

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

TAUS = (15, 20, 30, 50, 100, 200, 400)
DS_US = (50, 100, 200, 350, 700, 1000)
S = int(sys.argv[1]) if len(sys.argv) > 1 else 148
X = int(sys.argv[2]) if len(sys.argv) > 2 else 50_000

base = C.c2(n_streams=S)
L = S * X + base.stages[0].iparam[0] - 1
base = base.replace(dna=dict(base.dna, db_len=L, n_planted=base.dna["n_planted"] * L // (1 << 20)))
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
ptr = db.data_ptr()
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr)
budgets, cal = realtime.calibrate_budgets(base, wl, ptr, margin=1.10, slack_ns=128)
cfg0 = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, b=C.PAPER_B)
print(json.dumps({"streams": S, "roots_per_stream": X, "gains": gains, "budgets_ns": budgets,
                  "b": list(C.PAPER_B)}), flush=True)


def run(c):
    pl = Pipeline(c, wl, flags=0)
    pl.bind_device(ptr, wl.db_len)
    t0 = time.perf_counter()
    pl.drain()
    dt = time.perf_counter() - t0
    st = pl.stats()
    pl.close()
    return {"active_fraction": round(st["active_fraction"], 4),
            "hw_busy_fraction": round(st["hw_busy_fraction"], 4),
            "misses": int(st["miss_events_ns"]), "max_latency_us": round(st["max_latency_ns"] / 1e3, 1),
            "max_lateness_us": round(max(st["max_lateness_ns"]) / 1e3, 1), "wall_s": round(dt, 3)}


rows = []
for tau in TAUS:
    for D_us in DS_US:
        cfg = cfg0.replace(interarrival=tau, deadline=D_us * 1000)
        rec = {"tau0_ns": tau, "D_us": D_us}
        sol = realtime.solve_at(cfg, tau)
        if sol is None:
            rec["enforced"] = rec["threshold"] = "infeasible"
        else:
            w, th, T = sol
            rec["enforced"] = {"fig1_T": round(T, 4), "w_ns": list(w), **run(cfg.replace(wait_time=tuple(w), policy=0))}
            rec["threshold"] = {"theta": list(th), **run(cfg.replace(wait_threshold=tuple(th), policy=1,
                                                                   slack_guard=int(max(budgets))))}
        Mm = realtime.monolithic_at(cfg, tau)
        if Mm is None:
            rec["monolithic"] = "infeasible"
        else:
            rec["monolithic"] = {"M": Mm[0], "fig2_objective": round(Mm[1], 4),
                                 **run(cfg.replace(policy=2, block_size=Mm[0]))}
        rows.append(rec)
        print(json.dumps(rec), flush=True)


def cell(r, key):
    x = r[key]
    if not isinstance(x, dict):
        return "   -  "
    return f"{x['active_fraction']:.3f}" + ("*" if x["misses"] else " ")


print("\nmodel active fraction (enforced / threshold / monolithic; * = deadline misses)")
print("tau0\\D(us) " + "".join(f"{d:>24}" for d in DS_US))
for tau in TAUS:
    line = f"{tau:>9}  "
    for D_us in DS_US:
        r = next(x for x in rows if x["tau0_ns"] == tau and x["D_us"] == D_us)
        line += f"  {cell(r, 'enforced')}/{cell(r, 'threshold')}/{cell(r, 'monolithic')}"
    print(line)
print("\nenforced - monolithic active fraction where both are miss-free "
      "(negative = enforced waiting uses less of the SM; E = only enforced is feasible and miss-free)")
print("tau0\\D(us) " + "".join(f"{d:>8}" for d in DS_US))
for tau in TAUS:
    line = f"{tau:>9}  "
    for D_us in DS_US:
        r = next(x for x in rows if x["tau0_ns"] == tau and x["D_us"] == D_us)
        e, m = r["enforced"], r["monolithic"]
        eok = isinstance(e, dict) and e["misses"] == 0
        mok = isinstance(m, dict) and m["misses"] == 0
        line += f"{e['active_fraction'] - m['active_fraction']:>+8.3f}" if eok and mok else (
            f"{'E':>8}" if eok else f"{'M':>8}" if mok else f"{'-':>8}")
    print(line)
