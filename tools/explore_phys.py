"""Exploration: physical-clock behaviour of the executor on the c2 workload (B200)."""
import json
import math
import sys
import time

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, solve_enforced_waits, solve_monolithic


def run(cfg, wl, flags=0, reps=1, **over):
    pl = Pipeline(cfg, wl, flags=flags, **over)
    pl.push(wl.db, wl.db_len)
    ts = []
    for r in range(reps):
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        pl.launch()
        pl.drain()
        ts.append(time.perf_counter() - t0)
        pl.rewind()
        pl.push(wl.db, wl.db_len)
    st = pl.stats()
    pl.close()
    return st, min(ts)


def main():
    cfg0 = C.c2(n_streams=148)
    wl = G.make_dna(cfg0.seed, **cfg0.dna)
    # logical, Table-1 timing, paper tau0/D
    w, th, T, Tc = solve_enforced_waits(cfg0.replace(gain=C.TABLE1_G))
    cfgL = cfg0.replace(wait_time=tuple(w))
    st, dt = run(cfgL, wl, reps=3)
    g = [st["produced"][i] / max(1, st["consumed"][i]) for i in range(3)]
    print(json.dumps(dict(mode="logical", wall_s=dt, roots=st["roots"], items_per_s=st["roots"] / dt,
                          misses=st["miss_events"], af=st["active_fraction"], gains=g,
                          firings=st["firings"], sched_cycles=st["sched_cycles"], spilled=st["spilled"],
                          matches=st["matches"])), flush=True)
    for mode in (C.THRESHOLD_SLACK, C.MONOLITHIC):
        c = cfgL.replace(policy=mode, wait_threshold=tuple(th), block_size=2688)
        st, dt = run(c, wl, reps=3)
        print(json.dumps(dict(mode=f"logical-{mode}", wall_s=dt, items_per_s=st["roots"] / dt,
                              misses=st["miss_events"], af=st["active_fraction"])), flush=True)
    # physical calibration with generous budgets
    for tb in (20000, 5000):
        cfgP = cfg0.replace(clock=C.CLOCK_GLOBALTIMER, service_time=(tb,) * 4, wait_time=(0, 0, 0, 0),
                            interarrival=200, deadline=10**8)
        st, dt = run(cfgP, wl)
        mean = [st["busy_ns"][i] / max(1, st["firings"][i]) for i in range(4)]
        print(json.dumps(dict(mode="phys-calib", budget=tb, wall_s=dt, max_fire=st["max_fire_ns"], mean_fire=mean,
                              late=st["max_lateness_ns"], overruns=st["overruns"], wall_ns=st["wall_ns"],
                              hw_busy=st["hw_busy_fraction"], errors=st["errors"])), flush=True)
    tcal = [int(math.ceil(1.3 * x)) + 64 for x in st["max_fire_ns"]]
    print("calibrated t", tcal, flush=True)
    for D in (50_000, 100_000, 350_000):
        for tau in (4, 6, 8, 10, 15, 20, 40, 100):
            c = cfg0.replace(clock=C.CLOCK_GLOBALTIMER, service_time=tuple(tcal), interarrival=tau, deadline=D,
                             gain=tuple(g))
            try:
                w, th, T, Tc = solve_enforced_waits(c)
            except Exception as e:
                print(json.dumps(dict(D=D, tau=tau, infeasible=True)), flush=True)
                continue
            st, dt = run(c.replace(wait_time=tuple(w)), wl, flags=1)
            print(json.dumps(dict(D=D, tau=tau, w=w, T=T, wall_s=dt, misses=st["misses"], miss_ev=st["miss_events"],
                                  maxlat=st["max_latency"], maxlat_ns=st["max_latency_ns"],
                                  late=st["max_lateness_ns"], overruns=st["overruns"], max_fire=st["max_fire_ns"],
                                  af=st["active_fraction"], hw_busy=st["hw_busy_fraction"], wall_ns=st["wall_ns"],
                                  items_per_s=st["roots"] / dt, spilled=st["spilled"], errors=st["errors"])), flush=True)
            try:
                M, Tm = solve_monolithic(c)
                st, dt = run(c.replace(policy=C.MONOLITHIC, block_size=M), wl, flags=1)
                print(json.dumps(dict(D=D, tau=tau, mono_M=M, Tm=Tm, misses=st["misses"], maxlat_ns=st["max_latency_ns"],
                                      af=st["active_fraction"], hw_busy=st["hw_busy_fraction"], wall_ns=st["wall_ns"],
                                      errors=st["errors"])), flush=True)
            except Exception as e:
                print(json.dumps(dict(D=D, tau=tau, mono="infeasible")), flush=True)


if __name__ == "__main__":
    main()
