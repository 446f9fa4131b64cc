"""N1: the paper's b calibration on the GPU for the random-gain BLAST model (Table 1),
100 streams x 50,000 items per launch, at several (tau0, D) points; compare with the
paper's b = (1, 3, 9, 6) (L230)."""
import json
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from paper_conf_icppw_planob21_b200 import realtime

for tau, D in ((10, 50_000), (10, 100_000), (20, 100_000), (50, 200_000), (100, 350_000), (5, 350_000)):
    cfg = C.gain_model_blast(interarrival=tau, deadline=D, n_streams=100, n_roots=50_000, seed=21)
    r = realtime.calibrate_b(cfg)
    print(json.dumps({"tau0": tau, "D": D, "b": r["b"], "miss_free": r["miss_free"], "T": r["T"],
                      "iterations": r["iterations"], "history": r["history"]}), flush=True)
