"""Per-step time of the bench configuration three ways: events around pl.launch() after an
L2 flush (the bench), back-to-back launches, and the same with the stream idle before each
launch -- to separate kernel time from the per-launch memsets and host enqueue."""
import json
import sys

sys.path.insert(0, ".")
import torch
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

cfg = C.c2(n_streams=148).replace(clock=1, ns_per_unit=1.0, service_time=(1936, 3656, 3856, 16376),
                                   wait_time=(112, 5509, 4134, 25048), interarrival=16, deadline=350_000,
                                   b=C.PAPER_B, eager_drain=True)
wl = G.make_dna(cfg.seed, **cfg.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
st = torch.cuda.current_stream()
pl = Pipeline(cfg, wl, flags=0, stream=st)
pl.bind_device(db.data_ptr(), wl.db_len)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
for _ in range(5):
    pl.launch()
torch.cuda.synchronize()
out = {}
K = 20
ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(K)]
for k in range(K):
    flush.zero_()
    ev[k][0].record(st)
    pl.launch()
    ev[k][1].record(st)
    pl.summary()
out["flush_then_launch_us"] = sum(a.elapsed_time(b) for a, b in ev) / K * 1e3
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record(st)
for k in range(K):
    pl.launch()
e1.record(st)
torch.cuda.synchronize()
out["back_to_back_us"] = e0.elapsed_time(e1) / K * 1e3
for k in range(K):
    torch.cuda.synchronize()
    ev[k][0].record(st)
    pl.launch()
    ev[k][1].record(st)
torch.cuda.synchronize()
out["idle_then_launch_us"] = sum(a.elapsed_time(b) for a, b in ev) / K * 1e3
s = pl.stats()
out["wall_ns_max_cta"] = s["wall_ns"]
print(json.dumps(out))
