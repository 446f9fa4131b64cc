"""Per-phase cycles per firing of the executor (leader lane clock64), c2 workload."""
import json
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, solve_enforced_waits

NAMES = ["decide", "bar1", "load+stage+scan", "records+reserve", "writes", "publish"]


def show(tag, st):
    out = {"tag": tag}
    for i in range(st["n_stages"]):
        f = max(1, st["firings"][i])
        out[f"node{i}"] = {n: round(st["phase_cycles"][i][k] / f) for k, n in enumerate(NAMES)}
        out[f"node{i}"]["firings"] = st["firings"][i]
        out[f"node{i}"]["mean_fire_ns"] = round(st["busy_ns"][i] / f) if st["busy_ns"][i] else None
        out[f"node{i}"]["max_fire_ns"] = st["max_fire_ns"][i]
    print(json.dumps(out), flush=True)


cfg0 = C.c2(n_streams=148)
wl = G.make_dna(cfg0.seed, **cfg0.dna)
w, th, T, Tc = solve_enforced_waits(cfg0.replace(gain=C.TABLE1_G))
for S in (148, 1):
    for clock, t, tau, ww in ((C.CLOCK_LOGICAL, C.TABLE1_T, 10, tuple(w)), (C.CLOCK_GLOBALTIMER, (20000,) * 4, 200, (0, 0, 0, 0))):
        cfg = cfg0.replace(n_streams=S, clock=clock, service_time=t, interarrival=tau, wait_time=ww, deadline=10**8)
        pl = Pipeline(cfg, wl, flags=0)
        pl.push(wl.db, wl.db_len)
        pl.drain()
        show(f"S={S} clock={clock}", pl.stats())
        pl.close()
