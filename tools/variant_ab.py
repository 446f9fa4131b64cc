"""A/B of executor experiment bits (PL_VARIANT) on the physical c2 run: per-node phase
cycles and firing times.  usage: python tools/variant_ab.py 0 1 2 3"""
import json
import os
import subprocess
import sys

CHILD = r'''
import json, sys
sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline
NAMES = ["decide", "bar1", "load+stage+scan", "records", "writes", "publish"]
cfg0 = C.c2(n_streams=148)
wl = G.make_dna(cfg0.seed, **cfg0.dna)
out = {"variant": int(sys.argv[1])}
for tau in (150, 25):
    cfg = cfg0.replace(clock=C.CLOCK_GLOBALTIMER, service_time=(20000,) * 4, interarrival=tau,
                       wait_time=(0, 0, 0, 0), deadline=10**8)
    best = None
    for rep in range(3):
        pl = Pipeline(cfg, wl, flags=0)
        pl.push(wl.db, wl.db_len)
        pl.drain()
        st = pl.stats()
        pl.close()
        f0 = max(1, st["firings"][0])
        m = st["busy_ns"][0] / f0
        if best is None or m < best[0]:
            best = (m, st)
    st = best[1]
    r = {}
    for i in range(st["n_stages"]):
        f = max(1, st["firings"][i])
        r[f"node{i}"] = {n: round(st["phase_cycles"][i][k] / f) for k, n in enumerate(NAMES)}
        r[f"node{i}"]["mean_fire_ns"] = round(st["busy_ns"][i] / f)
        r[f"node{i}"]["max_fire_ns"] = st["max_fire_ns"][i]
        r[f"node{i}"]["firings"] = st["firings"][i]
        r[f"node{i}"]["loop"] = sum(st["phase_cycles"][i][k] for k in range(6)) // f
    out[f"tau{tau}"] = r
print(json.dumps(out), flush=True)
'''

for v in sys.argv[1:]:
    env = dict(os.environ, PL_VARIANT=v)
    r = subprocess.run([sys.executable, "-c", CHILD, v], env=env, capture_output=True, text=True)
    print(r.stdout.strip() or r.stderr[-2000:], flush=True)
