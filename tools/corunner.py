"""N3 co-runner experiment: does the processor time that
enforced waiting yields serve other work?  A compute-bound background kernel (tools/corunner/corunner.cu,
~8 CTAs/SM) runs beside the physical-clock executor (c2, v = 64 so that the executor CTA leaves
register room on its SM) under FIXED_WAIT and under MONOLITHIC at the same (tau0, D); we time
the co-runner alone and beside each executor, and check the executor's deadline misses."""
import ctypes
import json
import sys

sys.path.insert(0, ".")
import torch

from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline, realtime
from paper_conf_icppw_planob21_b200.build import build_corunner

lib = ctypes.CDLL(build_corunner())      # the co-runner is a measurement tool, not in libplgpu.so

D = 350_000
base = C.c2(n_streams=148, vector_width=64)
wl = G.make_dna(base.seed, **base.dna)
db = torch.from_numpy(wl.db.view("int32")).cuda()
ptr = db.data_ptr()
gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, ptr)
budgets, _ = realtime.calibrate_budgets(base, wl, ptr)
cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D, b=C.PAPER_B)
tau = realtime.min_feasible_tau(cfg)
while realtime.monolithic_at(cfg, tau) is None:
    tau = int(tau * 1.1) + 1
tau = int(tau * 1.3)           # a rate both strategies sustain
w, th, T = realtime.solve_at(cfg, tau)
M, Tm = realtime.monolithic_at(cfg, tau)
sink = torch.zeros(148 * 16, dtype=torch.float32, device="cuda")
sA = torch.cuda.Stream()
sB = torch.cuda.Stream()
ITERS = 20_000
N_CTAS = 148 * 8


def corunner(stream, n_ctas=None):
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record(stream)
    assert lib.pl_corunner_launch(ctypes.c_void_p(stream.cuda_stream), n_ctas or N_CTAS, ITERS,
                                  ctypes.c_void_p(sink.data_ptr())) == 0
    e1.record(stream)
    return e0, e1


def run(policy):
    c = cfg.replace(interarrival=tau, wait_time=tuple(w), policy=policy, block_size=M)
    pl = Pipeline(c, wl, flags=0, stream=sA)
    pl.bind_device(ptr, wl.db_len)
    pl.launch()                               # warm-up
    pl.summary()
    x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    x0.record(sA)
    pl.launch()
    x1.record(sA)
    e0, e1 = corunner(sB, N_CTAS) if N_CTAS else (None, None)
    torch.cuda.synchronize()
    s = pl.summary()
    st = pl.stats()
    pl.close()
    return {"executor_ms": x0.elapsed_time(x1), "corunner_ms": e0.elapsed_time(e1) if e0 else None,
            "misses_ns": s["miss_events_ns"], "max_latency_ns": s["max_latency_ns"],
            "model_active_fraction": st["active_fraction"], "hw_busy_fraction": st["hw_busy_fraction"]}


rows = []
for per_sm in (0, 1, 2, 4, 8):
    N_CTAS = 148 * per_sm
    alone = None
    if N_CTAS:
        corunner(sB)
        torch.cuda.synchronize()
        ts = []
        for _ in range(3):
            e0, e1 = corunner(sB)
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        alone = min(ts)
    row = {"corunner_ctas_per_sm": per_sm, "corunner_alone_ms": alone}
    for name, pol in (("enforced", C.FIXED_WAIT), ("monolithic", C.MONOLITHIC)):
        r = run(pol)
        if alone:
            r["corunner_throughput_share"] = alone / r["corunner_ms"]
        row[name] = r
    rows.append(row)
    print(json.dumps(row), flush=True)
print(json.dumps({"tau0_ns": tau, "D_ns": D, "v": 64, "budgets_ns": budgets, "w_ns": w, "M": M,
                  "fig1_T": T, "fig2_objective": Tm}))
