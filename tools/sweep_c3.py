"""c3 / paper Figs. 3-4 on the GPU: enforced waiting (Fig. 1) vs monolithic (Fig. 2) over the
(tau0, D) grid on the paper-faithful random-gain BLAST model (Table 1), logical clock.
Each grid point: 100 streams x 50,000 items (= the paper's 100 seeds x 50,000-input streams,
L227-L230) for each policy, one executor launch each.  Prints one JSON line per point and a
summary table; the optimiser's predicted fractions are printed beside the simulated ones."""
import json
import sys
import time

sys.path.insert(0, ".")
from plgen import configs as C
from paper_conf_icppw_planob21_b200 import Pipeline, solve_enforced_waits, solve_monolithic

TAUS = (3, 5, 10, 20, 50, 100)
DS = (20_000, 25_000, 50_000, 100_000, 200_000, 350_000)
S, X = 100, 50_000


def run(cfg):
    pl = Pipeline(cfg, None, flags=1)
    pl.push(None, cfg.n_roots)
    t0 = time.perf_counter()
    pl.drain()
    dt = time.perf_counter() - t0
    st = pl.stats()
    lat, _ = pl.latency()
    pl.close()
    per_stream = lat.reshape(cfg.n_streams, -1)
    miss_free = int(((per_stream > cfg.deadline).sum(axis=1) == 0).sum())
    return st, miss_free, dt


rows = []
for tau in TAUS:
    for D in DS:
        base = C.gain_model_blast(interarrival=tau, deadline=D, n_streams=S, n_roots=X, seed=7)
        rec = {"tau0": tau, "D": D}
        try:
            w, th, T, Tc = solve_enforced_waits(base)
            st, mf, dt = run(base.replace(wait_time=tuple(w)))
            rec["enforced"] = {"fig1_T": T, "active_fraction": st["active_fraction"], "miss_free_streams": mf,
                               "missed_items": st["misses"], "max_latency": st["max_latency"], "wall_s": dt}
        except RuntimeError:
            rec["enforced"] = None
        try:
            M, Tm = solve_monolithic(base)
            st, mf, dt = run(base.replace(policy=C.MONOLITHIC, block_size=M))
            rec["monolithic"] = {"M": M, "fig2_objective": Tm, "active_fraction": st["active_fraction"],
                                 "miss_free_streams": mf, "missed_items": st["misses"], "wall_s": dt}
        except RuntimeError:
            rec["monolithic"] = None
        rows.append(rec)
        print(json.dumps(rec), flush=True)

print("\ntau0\\D  " + "".join(f"{d:>22d}" for d in DS))
for tau in TAUS:
    line = f"{tau:6d}  "
    for D in DS:
        r = next(x for x in rows if x["tau0"] == tau and x["D"] == D)
        e = f"{r['enforced']['active_fraction']:.3f}" if r["enforced"] else "inf"
        m = f"{r['monolithic']['active_fraction']:.3f}" if r["monolithic"] else "inf"
        line += f"{e + ' / ' + m:>22s}"
    print(line)
