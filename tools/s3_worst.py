"""Worst-case extension vectors for the S3 (X-drop) node: a 1 Mbp DB made of back-to-back
planted query copies (256 bases, 5 % substitutions), so nearly every S3 input extends a
whole planted diagonal.  Logical clock (runs as fast as the executor can); reports per
node the mean leader-clock cycles per firing of each phase (decide / B1 / load+stage+scan /
records / writes / publish) and the mean inputs per firing.  PL_VARIANT selects experiments."""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, solve_enforced_waits

n_pl = int(sys.argv[1]) if len(sys.argv) > 1 else 3500
base = C.c2(n_streams=148)
wl = G.make_dna(base.seed, db_len=1 << 20, q_len=1024, n_planted=n_pl, min_len=256, max_len=256)
w, th, T, Tc = solve_enforced_waits(base.replace(gain=C.TABLE1_G))
cfg = base.replace(wait_time=tuple(w), gain=C.TABLE1_G)
db = torch.from_numpy(wl.db.view("int32")).cuda()
for rep in range(2):
    pl = Pipeline(cfg, wl, flags=0)
    pl.bind_device(db.data_ptr(), wl.db_len)
    pl.drain()
    s = pl.stats()
    pl.close()
N = cfg.n_stages
out = {"planted": len(wl.planted), "consumed": s["consumed"], "firings": s["firings"],
       "items_per_firing": [round(s["consumed"][i] / max(1, s["firings"][i]), 1) for i in range(N)],
       "phase_cycles_per_firing": [[round(x / max(1, s["firings"][i])) for x in s["phase_cycles"][i]] for i in range(N)],
       "matches": s["matches"]}
print(json.dumps(out))
