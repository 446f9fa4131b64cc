import sys
sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline
cfg0 = C.c2(n_streams=148)
wl = G.make_dna(cfg0.seed, **cfg0.dna)
cfg = cfg0.replace(stages=C.dna_stages()[:1], service_time=C.TABLE1_T[:1], b=(1,), wait_time=(993,))
pl = Pipeline(cfg, wl, flags=0)
pl.push(wl.db, wl.db_len)
pl.drain()
print(pl.stats()["firings"])
