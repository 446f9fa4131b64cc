import sys
sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline
base = C.c2(n_streams=148)
wl = G.make_dna(base.seed, **base.dna)
for flags in (8, 15, 0, 7):
    cfg = base.replace(clock=1, service_time=(5000, 6000, 7000, 20000), interarrival=60, wait_time=(0, 20000, 30000, 50000), deadline=10**8)
    pl = Pipeline(cfg, wl, flags=flags)
    pl.push(wl.db, wl.db_len); pl.drain(); st = pl.stats(); pl.close()
    print(flags, [round(st["busy_ns"][i] / max(1, st["firings"][i])) for i in range(4)], st["firings"], st["overruns"], st["max_fire_ns"])
