"""Physical-clock run where node 0 (S0 seed lookup) does nearly all the work: a 2-node
pipeline S0 -> S1 with S1 firing every 220 us.  For ncu source-level views of node 0's
firing path.  argv: [reps]"""
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

reps = int(sys.argv[1]) if len(sys.argv) > 1 else 1
base = C.c2(n_streams=148)
wl = G.make_dna(base.seed, **base.dna)
cfg = base.replace(stages=C.dna_stages()[:2], service_time=(20000, 20000), b=(1, 1), clock=C.CLOCK_GLOBALTIMER,
                   interarrival=150, wait_time=(0, 200000), deadline=10**9)
pl = Pipeline(cfg, wl, flags=0)
for r in range(reps):
    pl.push(wl.db, wl.db_len)
    pl.drain()
    st = pl.stats()
    pl.rewind()
print({k: st[k] for k in ("firings", "busy_ns", "phase_cycles")})
