"""Where a bench step's time goes (bench configuration, physical clock): the stream's arrival
window H = X*tau0, the logical drain tail (t_end - H, averaged over streams), the kernel-side
CTA runtime (wall_ns, max over CTAs), and the CUDA-event time of a launch (after an L2 flush,
back to back, and from an idle stream).  argv: tau0 t0 t1 t2 t3 w0 w1 w2 w3 [eager 0/1]"""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

a = [int(x) for x in sys.argv[1:]] or [16, 1976, 3616, 3816, 16336, 72, 5549, 4174, 25088, 1]
tau, t, w = a[0], tuple(a[1:5]), tuple(a[5:9])
eager = bool(a[9]) if len(a) > 9 else True
import os
dbl = int(os.environ.get("DB_LEN", str(1 << 20)))   # longer streams: does the lateness stay bounded?
cfg = C.c2(n_streams=148, dna=dict(db_len=dbl, q_len=1024, n_planted=64 * dbl // (1 << 20))).replace(clock=1, ns_per_unit=1.0, service_time=t, wait_time=w, interarrival=tau,
                                   deadline=350_000, b=C.PAPER_B, eager_drain=eager)
wl = G.make_dna(cfg.seed, **cfg.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
st = torch.cuda.current_stream()
pl = Pipeline(cfg, wl, flags=0, stream=st)
pl.bind_device(db.data_ptr(), wl.db_len)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(5):
    pl.launch()
torch.cuda.synchronize()
K = 20
out = {}
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
for k in range(K):
    flush.zero_()
    ev[k][0].record(st)
    pl.launch()
    ev[k][1].record(st)
    pl.summary()
out["flush_then_launch_us"] = sum(x.elapsed_time(y) for x, y in ev) / K * 1e3
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for k in range(K):
    pl.launch()
e1.record(st)
torch.cuda.synchronize()
out["back_to_back_us"] = e0.elapsed_time(e1) / K * 1e3
s = pl.stats()
S = s["n_streams"]
out["H_us_per_stream"] = s["window"] / S / 1e3
out["t_end_us_per_stream"] = s["t_end"] / S / 1e3
out["logical_tail_us"] = (s["t_end"] - s["window"]) / S / 1e3
out["wall_us_max_cta"] = s["wall_ns"] / 1e3
out["max_latency_ns"] = s["max_latency_ns"]
out["misses"] = s["miss_events_ns"]
out["firings"] = s["firings"]
out["max_lateness_ns"] = s["max_lateness_ns"]
out["max_fire_ns"] = s["max_fire_ns"]
out["max_loop_ns"] = s["max_loop_ns"]
out["overruns"] = s["overruns"]
print(json.dumps(out))
