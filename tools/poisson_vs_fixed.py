"""N2: Poisson vs fixed-rate arrivals on the random-gain BLAST model (100 streams x 50,000
items): b from the on-device calibration, Fig. 1 objective, simulated active fraction."""
import json
import sys

sys.path.insert(0, ".")
from plgen import arrivals as A
from plgen import configs as C
from paper_conf_icppw_planob21_b200 import Pipeline, realtime

for tau, D in ((10, 50_000), (20, 100_000), (50, 200_000), (100, 350_000)):
    cfg = C.gain_model_blast(interarrival=tau, deadline=D, n_streams=100, n_roots=50_000, seed=23)
    out = {"tau0": tau, "D": D}
    for name, arr in (("fixed", None), ("poisson", A.poisson(23, [50_000] * 100, tau))):
        r = realtime.calibrate_b(cfg, arrivals=arr, max_iter=12)
        af = None
        if r.get("w"):
            pl = Pipeline(cfg.replace(b=r["b"], wait_time=r["w"]), None, flags=0, arrivals=arr)
            pl.push(None, cfg.n_roots)
            pl.drain()
            af = pl.stats()["active_fraction"]
            pl.close()
        out[name] = {"b": r["b"], "miss_free": r["miss_free"], "fig1_T": r["T"], "active_fraction": af,
                     "iterations": r["iterations"]}
    print(json.dumps(out), flush=True)
