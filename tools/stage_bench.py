"""Per-stage batch kernels (pl_stage_batch) on the c2 / c4 DB: items/s, bytes moved and GB/s
per stage (SURVEY K-BENCH; north_star: per-stage HBM GB/s).  argv: db_len [reps]"""
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

db_len = int(sys.argv[1]) if len(sys.argv) > 1 else (1 << 20)
reps = int(sys.argv[2]) if len(sys.argv) > 2 else 5
heavy = db_len > (1 << 24)
cfg = C.c2(n_streams=1, dna=dict(db_len=db_len, q_len=1024, n_planted=max(64, db_len >> 14), heavy_tailed=heavy),
           wait_time=(0, 0, 0, 0))
wl = G.make_dna(cfg.seed, **cfg.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
pl = Pipeline(cfg, wl, flags=0)
pl.bind_device(db.data_ptr(), db_len)
R = db_len - 5
cap = int(R * 0.5) * 2 + (1 << 20)
a = torch.empty((cap, 2), dtype=torch.int32, device="cuda")
b = torch.empty((cap, 2), dtype=torch.int32, device="cuda")
import os
with open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "MEASURED_PEAKS.json")) as _f:
    pk = json.load(_f)["hbm_gbs"]
out = []
srcs = [(0, R), None, None, None]
n_in = R
bufin, bufout = 0, a.data_ptr()
for st in range(4):
    in_ptr = 0 if st == 0 else bufin
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    pl.stage_batch(st, in_ptr, n_in, 0, bufout if st < 3 else 0, cap if st < 3 else 0)   # warm-up
    torch.cuda.synchronize()
    ev0.record()
    for _ in range(reps):
        n_out, cyc = pl.stage_batch(st, in_ptr, n_in, 0, bufout if st < 3 else 0, cap if st < 3 else 0)
    ev1.record()
    torch.cuda.synchronize()
    ms = ev0.elapsed_time(ev1) / reps
    in_bytes = 0.25 * n_in if st == 0 else 8.0 * n_in
    out_bytes = (8.0 if st < 3 else 24.0) * n_out
    gbs = (in_bytes + out_bytes) / (ms * 1e-3) / 1e9
    rec = {"stage": st, "inputs": n_in, "outputs": n_out, "ms": ms, "items_per_s": n_in / (ms * 1e-3),
           "algorithmic_bytes": in_bytes + out_bytes, "GB_per_s": gbs, "frac_of_hbm_peak": gbs / pk,
           "max_vector_cycles": cyc}
    out.append(rec)
    print(json.dumps(rec), flush=True)
    n_in = n_out
    bufin = bufout
    bufout = b.data_ptr() if bufout == a.data_ptr() else a.data_ptr()
pl.close()
