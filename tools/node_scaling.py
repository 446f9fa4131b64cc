"""Node-0 per-firing phase cycles as a function of how many pipeline nodes run beside it."""
import json
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

NAMES = ["decide", "bar1", "load+stage+scan", "records", "writes", "publish"]
cfg0 = C.c2(n_streams=148)
wl = G.make_dna(cfg0.seed, **cfg0.dna)
for N in (1, 2, 4):
    st = C.dna_stages()[:N]
    cfg = cfg0.replace(stages=st, service_time=C.TABLE1_T[:N], b=C.PAPER_B[:N], wait_time=(993, 2422, 965, 1628)[:N])
    pl = Pipeline(cfg, wl, flags=0)
    pl.push(wl.db, wl.db_len)
    pl.drain()
    s = pl.stats()
    pl.close()
    f = s["firings"][0]
    print(json.dumps({"N": N, "node0": {n: round(s["phase_cycles"][0][k] / f) for k, n in enumerate(NAMES)},
                      "wall_us": s["wall_ns"] / 1e3}), flush=True)
