"""One physical executor launch at the bench configuration (for ncu --set full).
argv: tau0_ns t0 t1 t2 t3 w0 w1 w2 w3 [deadline_ns] [policy] [M] [eager_drain 0/1]"""
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

a = [int(x) for x in sys.argv[1:]]
tau, t, w = a[0], tuple(a[1:5]), tuple(a[5:9])
D = a[9] if len(a) > 9 else 350_000
policy = a[10] if len(a) > 10 else 0
M = a[11] if len(a) > 11 else 0
eager = bool(a[12]) if len(a) > 12 else False
cfg = C.c2(n_streams=148).replace(clock=1, ns_per_unit=1.0, service_time=t, wait_time=w, interarrival=tau,
                                   deadline=D, b=C.PAPER_B, policy=policy, block_size=M,
                                   eager_drain=eager)
wl = G.make_dna(cfg.seed, **cfg.dna)
pl = Pipeline(cfg, wl, flags=0)
pl.push(wl.db, wl.db_len)
pl.drain()
st = pl.stats()
print({k: st[k] for k in ("roots", "firings", "miss_events", "overruns", "max_latency_ns", "matches", "errors")})
