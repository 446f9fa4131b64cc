"""One executor launch on the c2 workload (for ncu).  argv: clock(0/1) policy(0/1/2) streams"""
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, solve_enforced_waits

clock = int(sys.argv[1]) if len(sys.argv) > 1 else 0
policy = int(sys.argv[2]) if len(sys.argv) > 2 else 0
S = int(sys.argv[3]) if len(sys.argv) > 3 else 148
reps = int(sys.argv[4]) if len(sys.argv) > 4 else 1
cfg = C.c2(n_streams=S)
wl = G.make_dna(cfg.seed, **cfg.dna)
w, th, T, Tc = solve_enforced_waits(cfg.replace(gain=C.TABLE1_G))
if clock == 0:
    cfg = cfg.replace(wait_time=tuple(w), wait_threshold=tuple(th), policy=policy, block_size=2688)
else:
    cfg = cfg.replace(clock=1, service_time=(20000,) * 4, interarrival=200, wait_time=(0, 0, 0, 0),
                      deadline=10**8, policy=policy, wait_threshold=(128, 64, 64, 8), block_size=1024)
pl = Pipeline(cfg, wl, flags=0)
pl.push(wl.db, wl.db_len)
for r in range(reps):
    pl.launch()
    pl.drain()
    pl.rewind()
    pl.push(wl.db, wl.db_len)
print(pl.stats()["firings"])
