"""Node 0's per-firing loop (leader clock64 cycles per firing, excluding the pacing wait:
decide / firing phases / publish+bookkeeping) at the bench configuration, with the other
nodes firing on their schedule vs parked (huge waits: they fire once at T=0 and then only
in the drain), and the measured max loop time / max firing time in ns.
argv: tau0 t0 t1 t2 t3 w0 w1 w2 w3"""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

a = [int(x) for x in sys.argv[1:]] or [16, 1976, 3616, 3816, 16336, 72, 5549, 4174, 25088]
tau, t, w = a[0], tuple(a[1:5]), tuple(a[5:9])
base = C.c2(n_streams=148).replace(clock=1, ns_per_unit=1.0, service_time=t, interarrival=tau,
                                    deadline=10 ** 9, b=C.PAPER_B, eager_drain=True)
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
for tag, ww in (("all nodes", w), ("others parked", (w[0], 10 ** 9, 10 ** 9, 10 ** 9))):
    cfg = base.replace(wait_time=ww)
    for _ in range(2):
        pl = Pipeline(cfg, wl, flags=0)
        pl.bind_device(db.data_ptr(), wl.db_len)
        pl.drain()
        s = pl.stats()
        pl.close()
    f = s["firings"][0]
    ph = [round(x / f) for x in s["phase_cycles"][0]]
    print(json.dumps({"case": tag, "node0_cycles_per_firing": sum(ph), "phases": ph,
                      "max_loop_ns": s["max_loop_ns"][0], "max_fire_ns": s["max_fire_ns"][0],
                      "mean_fire_ns": round(s["busy_ns"][0] / f), "max_lateness_ns": s["max_lateness_ns"][0]}))
