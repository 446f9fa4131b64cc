#!/usr/bin/env python
"""bench.py — sustained items/s at zero deadline misses of the enforced-waiting executor.

Metric (BASELINE.json): "items/s at 0 deadline misses; SM utilisation vs no-wait baseline".
Workload (BASELINE.json configs[1]): the BLAST-style 4-stage pipeline
(seed lookup -> hit enumeration -> ungapped window filter -> X-drop extension) on a seeded
synthetic 1 Mbp DB with a 1 kbp query and 64 planted matches, split into 148 independent
streams (one CTA each) on one B200; the physical %globaltimer clock (1 unit = 1 ns).

One step = one executor launch over the whole c2 DB (all streams).  Before timing:
  1. gains g_i from a logical-clock run; service-time budgets t_i = 1.1 x the longest
     firing of a physical run + 128 ns, re-measured at the operating point
     (realtime.refine_budgets, never raising a budget);
  2. the deadline D (default 350 us = the paper's largest D, 3.5e5 units, L212) and
     b = (1, 3, 9, 6) (L230); Fig. 1 solved by the library for w_i;
  3. tau0 = the smallest inter-arrival (ns) whose physical run has zero deadline misses,
     no queue overflow and every firing within 5 us of its schedule (sustainability).
value = roots processed / device time of the timed launches (CUDA events on the launch
stream, L2 flushed between steps), whole job over all ranks (max-over-ranks time).
The monolithic no-internal-wait baseline (§5, Fig. 2) runs at the same D: at the
enforced tau0 when Fig. 2 is feasible there, and at the fastest tau0 both strategies sustain.
"""
from __future__ import annotations

import argparse
import json
import math
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from plgen import configs as C  # noqa: E402
from plgen import dna as G  # noqa: E402

METRIC = "items/s at 0 deadline misses; SM utilisation vs no-wait baseline"
WORKLOAD = ("c2: BLAST seed-lookup -> hit-enumeration -> ungapped-window -> x-drop, 1 Mbp synthetic DB "
            "(seed 2 + rank), 1 kbp query, 64 planted matches, 148 streams (1 CTA each) per GPU")


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--deadline-ns", type=int, default=350_000)
    ap.add_argument("--streams", type=int, default=148)
    ap.add_argument("--cpu-sample-streams", type=int, default=148)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--budget-margin", type=float, default=1.10,
                    help="t_i = margin x longest measured firing + slack (SURVEY 8(d): x1.1)")
    ap.add_argument("--budget-slack", type=int, default=128)
    ap.add_argument("--refine", type=int, default=2, help="budget refinement rounds at the operating point")
    ap.add_argument("--max-lateness-ns", type=int, default=5000,
                    help="rate search: every firing must start within this of its schedule (sustainability)")
    ap.add_argument("--drain", default="eager", choices=["eager", "periodic"],
                    help="end of stream: R-DRAIN work-conserving drain (PL_EAGER_DRAIN) or the periodic rule")
    return ap.parse_args()


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks/throttle sampling during the timed region (B200_PROFILING.md)."""
    Q = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.hw_slowdown,"
         "clocks_event_reasons.hw_thermal_slowdown,clocks_event_reasons.sw_thermal_slowdown,"
         "clocks_event_reasons.sw_power_cap")

    def __init__(self, device):
        self.device = device
        self.rows = []
        self.proc = None

    def start(self):
        try:
            self.proc = subprocess.Popen(["nvidia-smi", f"--query-gpu={self.Q}", "--format=csv,noheader,nounits",
                                          "-lms", "100", "-i", str(self.device)], stdout=subprocess.PIPE,
                                         stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except OSError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            self.rows.append([x.strip() for x in line.split(",")])

    def stop(self):
        if self.proc is None:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["nvidia-smi unavailable"]}
        time.sleep(0.25)
        self.proc.terminate()
        try:
            self.proc.wait(timeout=2)
        except subprocess.TimeoutExpired:
            self.proc.kill()
        sm = [float(r[1]) for r in self.rows if len(r) >= 8 and r[1].replace(".", "").isdigit()]
        mx = [float(r[2]) for r in self.rows if len(r) >= 8 and r[2].replace(".", "").isdigit()]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[k] for r in self.rows if len(r) >= 8 for k in range(4) if r[4 + k] == "Active"})
        return {"sm_mhz": statistics.median(sm) if sm else None, "sm_max_mhz": max(mx) if mx else None,
                "reasons": reasons, "samples": len(self.rows)}


def peaks():
    try:
        with open(os.path.join(ROOT, "MEASURED_PEAKS.json")) as f:
            return json.load(f)["hbm_gbs"], "measured (MEASURED_PEAKS.json)"
    except (OSError, KeyError, ValueError):
        return 6650.0, "fallback (B200_PROFILING.md)"


def ncu_traffic():
    """dram bytes per launch of the executor from the committed ncu --set full capture."""
    try:
        with open(os.path.join(ROOT, "profiles", "ncu_summary.json")) as f:
            return json.load(f).get("dram_bytes_per_launch")
    except (OSError, ValueError):
        return None


# --------------------------------------------------------------- oracle leg
def _oracle_stream(args):
    cfg, lo, hi = args
    from oracle import des
    wl = _ORACLE_WL
    from oracle import stages as S
    ctx = S.DnaContext(wl.db, wl.db_len, wl.query, wl.q_len, cfg.stages[0].iparam[0])
    fns = des.make_stage_fns(cfg, ctx)
    r = des.simulate_stream(cfg, fns, lo, hi)
    return hi - lo, r.lat and max(r.lat)


_ORACLE_WL = None


def oracle_rate(cfg, wl, n_streams, procs=None):
    """The oracle DES (as it stands) on `n_streams` streams of the workload, over a
    process pool on the host cores.  Returns (items/s, cores, seconds, roots)."""
    global _ORACLE_WL
    import multiprocessing as mp
    _ORACLE_WL = wl
    from oracle import des
    k = cfg.stages[0].iparam[0]
    total = wl.db_len - k + 1
    rng = des.stream_ranges(cfg, total)[:n_streams]
    cores = procs or len(os.sched_getaffinity(0))
    t0 = time.perf_counter()
    with mp.get_context("fork").Pool(cores) as pool:
        res = pool.map(_oracle_stream, [(cfg, lo, hi) for lo, hi in rng], chunksize=1)
    dt = time.perf_counter() - t0
    roots = sum(r[0] for r in res)
    return roots / dt, cores, dt, roots


def logical_cfg(base):
    from paper_conf_icppw_planob21_b200 import solve_enforced_waits
    w, th, T, Tc = solve_enforced_waits(base.replace(gain=C.TABLE1_G))
    return base.replace(wait_time=tuple(w), gain=C.TABLE1_G)


# -------------------------------------------------------------- reference arm
def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    base = C.c2(n_streams=a.streams)
    wl = G.make_dna(base.seed, **base.dna)
    cfg = logical_cfg(base)
    n = min(a.cpu_sample_streams, a.streams)
    for _ in range(a.warmup):
        oracle_rate(cfg, wl, max(1, n // 8))
    times, roots = [], 0
    for _ in range(a.steps):
        rate, cores, dt, r = oracle_rate(cfg, wl, n)
        times.append(dt)
        roots = r
    V = roots * a.steps / sum(times)
    line = {"metric": METRIC, "value": V, "unit": "items/s", "n_gpus": a.gpus, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": 1e3 * sum(times) / a.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": WORKLOAD, "policy": "FIXED_WAIT", "clock": "logical (oracle DES)"},
            "cpu_baseline": {"value": V, "unit": "items/s", "cores": cores, "kind": "oracle",
                             "sample": f"{n} of {a.streams} c2 streams ({roots} roots) per step"},
            "e2e": {"value": V, "unit": "items/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# ------------------------------------------------------------------ our arm
def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
        return
    import torch
    import torch.distributed as dist
    from paper_conf_icppw_planob21_b200 import Pipeline, realtime
    from paper_conf_icppw_planob21_b200.dist import allreduce_stats

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    # PL_BENCH_SHARE_GPU=1 / PL_DIST_BACKEND=gloo let the multi-rank path run on one GPU (tests)
    if os.environ.get("PL_BENCH_SHARE_GPU"):
        local = local % torch.cuda.device_count()
    torch.cuda.set_device(local)
    dev = torch.device("cuda", local)
    if world > 1:
        backend = os.environ.get("PL_DIST_BACKEND", "nccl")
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=dev)
        else:
            dist.init_process_group(backend)
    log = (lambda d: print(json.dumps(d), file=sys.stderr, flush=True)) if rank == 0 else (lambda d: None)

    base = C.c2(n_streams=a.streams, seed=2 + rank)
    wl = G.make_dna(base.seed, **base.dna)
    db_dev = torch.from_numpy(wl.db.view("int32")).to(dev)
    db_ptr = db_dev.data_ptr()
    stream = torch.cuda.current_stream(dev)

    # 1. gains (logical run) and budgets (physical run)
    gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, db_ptr, stream=stream)
    budgets, cal = realtime.calibrate_budgets(base, wl, db_ptr, stream=stream, margin=a.budget_margin,
                                              slack_ns=a.budget_slack)
    if a.refine:
        cfg_r = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=a.deadline_ns,
                             b=C.PAPER_B, eager_drain=a.drain == "eager")
        try:
            budgets, _ = realtime.refine_budgets(cfg_r, wl, db_ptr, budgets, margin=a.budget_margin,
                                                 slack_ns=a.budget_slack, rounds=a.refine, stream=stream, log=log)
        except RuntimeError as ex:   # no operating point for the refinement: keep the probe's budgets
            log({"refine_budgets": "skipped", "error": str(ex)})
    if world > 1:   # every rank runs the same schedule: max budgets / min gains are conservative
        t = torch.tensor(budgets, dtype=torch.int64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        budgets = tuple(int(x) for x in t.tolist())
    log({"gains": gains, "budgets_ns": budgets, "cal_max_fire_ns": cal["max_fire_ns"]})
    cfg = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=a.deadline_ns,
                       b=C.PAPER_B, eager_drain=a.drain == "eager")
    # 2./3. the fastest miss-free rate
    rate_criterion = f"zero misses, every firing within {a.max_lateness_ns} ns of its schedule"
    try:
        tau, w, th, T, st_ok = realtime.find_rate(cfg, wl, db_ptr, stream=stream, log=log,
                                                  max_lateness_ns=a.max_lateness_ns)
    except RuntimeError as ex:   # keep the driver's bench line: fall back to zero misses only
        log({"rate_search": "failed with the lateness bound", "error": str(ex)})
        tau, w, th, T, st_ok = realtime.find_rate(cfg, wl, db_ptr, stream=stream, log=log, max_lateness_ns=None)
        rate_criterion = "zero misses (the lateness bound was not met at any rate tried)"
    if world > 1:
        t = torch.tensor([tau], dtype=torch.int64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        if int(t.item()) != tau:
            tau = int(t.item())
            w, th, T = realtime.solve_at(cfg, tau)
    run_cfg = cfg.replace(interarrival=tau, wait_time=tuple(w))
    pl = Pipeline(run_cfg, wl, flags=0, stream=stream)
    pl.bind_device(db_ptr, wl.db_len)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)

    for _ in range(a.warmup):
        pl.launch()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = ClockSampler(local)
    clocks.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    misses = 0
    sched_misses = 0
    overruns = 0
    lateness = 0
    errors = 0
    roots = 0
    torch.cuda.synchronize()
    for k in range(a.steps):
        flush.zero_()                                  # L2 flush, outside the timed region
        ev[k][0].record(stream)
        pl.launch()
        ev[k][1].record(stream)
        st = pl.stats()                                # syncs; outside the timed region
        misses += st["miss_events_ns"]                 # measured on %globaltimer
        sched_misses += st["miss_events"]              # the logical schedule's own
        overruns += sum(st["overruns"])
        lateness = max(lateness, max(st["max_lateness_ns"]))
        errors |= st["errors"]
        roots += st["roots"]
    torch.cuda.synchronize()
    clk = clocks.stop()
    step_ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    tot_ms = sum(step_ms)
    if world > 1:
        dist.barrier()
    st_last = allreduce_stats(dict(st, policy=0), device=dev)
    tt = torch.tensor([tot_ms], dtype=torch.float64, device=dev)
    cnt = torch.tensor([roots, misses, overruns, sched_misses], dtype=torch.int64, device=dev)
    if world > 1:
        dist.all_reduce(tt, op=dist.ReduceOp.MAX)
        dist.all_reduce(cnt, op=dist.ReduceOp.SUM)
    tot_ms = float(tt.item())
    roots_all, misses_all, overruns_all, sched_misses_all = (int(x) for x in cnt.tolist())
    value = roots_all / (tot_ms * 1e-3)

    # the other end-of-stream rule at the same rate and waits (the paper's periodic schedule
    # runs to the drain; R-DRAIN switches every node to work-conserving at the last arrival)
    other = None
    try:
        plo = Pipeline(run_cfg.replace(eager_drain=a.drain != "eager"), wl, flags=0, stream=stream)
        plo.bind_device(db_ptr, wl.db_len)
        plo.launch()
        plo.summary()
        o0, o1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        oms, oroots, omiss = 0.0, 0, 0
        for _ in range(a.steps):
            flush.zero_()
            o0.record(stream)
            plo.launch()
            o1.record(stream)
            so = plo.summary()
            oms += o0.elapsed_time(o1)
            oroots += so["roots"]
            omiss += so["miss_events_ns"]
        plo.close()
        other = {"drain": "periodic" if a.drain == "eager" else "eager", "value": oroots / (oms * 1e-3),
                 "ms_per_step": oms / a.steps, "misses": omiss, "max_latency_ns": so["max_latency_ns"]}
    except RuntimeError as ex:
        other = {"failed": str(ex)}

    # logical-clock throughput of the same executor (no real-time pacing)
    lc = logical_cfg(base)
    pll = Pipeline(lc, wl, flags=0, stream=stream)
    pll.bind_device(db_ptr, wl.db_len)
    for _ in range(3):
        pll.launch()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    torch.cuda.synchronize()
    e0.record(stream)
    for _ in range(5):
        pll.launch()
    e1.record(stream)
    torch.cuda.synchronize()
    logical_ips = 5 * pll.stats()["roots"] / (e0.elapsed_time(e1) * 1e-3)
    pll.close()

    # monolithic baseline (§5, Fig. 2): at the enforced rate, and at the fastest
    # rate where both strategies are feasible (the paper's utilisation comparison, L236-L255).
    # Run on streams of the paper's length (50,000 roots each, L230) built the c2 way: a c2
    # stream holds only 7,085 roots, less than one Fig. 2 block at these rates, so its [0, H)
    # window would credit the monolithic processor with at most one partial block.
    ul_len = a.streams * 50_000 + base.stages[0].iparam[0] - 1
    ucfg = cfg.replace(dna=dict(base.dna, db_len=ul_len, n_planted=base.dna["n_planted"] * ul_len // base.dna["db_len"]))
    uwl = G.make_dna(ucfg.seed, **ucfg.dna)
    udb = torch.from_numpy(uwl.db.view("int32")).to(dev)

    def run_policy(policy, tau_x, M=0):
        c = ucfg.replace(interarrival=int(tau_x), policy=policy, block_size=M)
        if policy == 0:
            sol = realtime.solve_at(ucfg, tau_x)
            if sol is None:
                return None
            c = c.replace(wait_time=tuple(sol[0]))
        pp = Pipeline(c, uwl, flags=0, stream=stream)
        pp.bind_device(udb.data_ptr(), uwl.db_len)
        pp.drain()
        sx = pp.stats()
        pp.close()
        return {"tau0_ns": int(tau_x), "active_fraction": sx["active_fraction"],
                "active_fraction_nonempty": sx["active_fraction_nonempty"],
                "hw_busy_fraction": sx["hw_busy_fraction"], "misses": sx["miss_events_ns"],
                "max_latency_ns": sx["max_latency_ns"], **({"M": M} if policy == 2 else {})}

    mono = {"stream_roots": 50_000}
    Mr = realtime.monolithic_at(ucfg, tau)
    mono["at_enforced_rate"] = run_policy(2, tau, Mr[0]) if Mr is not None else {"feasible": False}
    tau_m = tau
    while realtime.monolithic_at(ucfg, tau_m) is None and tau_m < 100 * tau:
        tau_m = int(math.ceil(tau_m * 1.05)) + 1
    for key, tx in (("common_rate", tau_m), ("slow_rate", 4 * tau_m)):
        Mm = realtime.monolithic_at(ucfg, tx)
        if Mm is not None:
            mono[key] = {"tau0_ns": tx, "monolithic": run_policy(2, tx, Mm[0]), "enforced": run_policy(0, tx),
                         "fig2_objective": Mm[1], "fig1_objective": (realtime.solve_at(ucfg, tx) or (0, 0, None))[2]}
    del udb

    # the north_star's threshold / deadline-slack rule (THRESHOLD_SLACK, theta_i from Fig. 1;
    # the slack reserve R_i gets a guard of the largest budget for real-time lateness)
    thr = None
    try:
        cfg_t = cfg.replace(slack_guard=int(max(budgets)))
        tau_t, w_t, th_t, T_t, _ = realtime.find_rate(cfg_t, wl, db_ptr, stream=stream, policy=1)
        plt = Pipeline(cfg_t.replace(interarrival=tau_t, wait_threshold=tuple(th_t), policy=1), wl, flags=0,
                       stream=stream)
        plt.bind_device(db_ptr, wl.db_len)
        plt.launch()
        plt.summary()
        x0, x1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        tms, troots, tmiss = 0.0, 0, 0
        for _ in range(a.steps):
            flush.zero_()
            x0.record(stream)
            plt.launch()
            x1.record(stream)
            sm_t = plt.summary()
            tms += x0.elapsed_time(x1)
            troots += sm_t["roots"]
            tmiss += sm_t["miss_events_ns"]
        stt = plt.stats()
        plt.close()
        thr = {"tau0_ns": tau_t, "theta": list(th_t), "slack_guard_ns": int(max(budgets)),
               "value": troots / (tms * 1e-3), "ms_per_step": tms / a.steps, "misses": tmiss,
               "sustained_items_per_s": a.streams * 1e9 / tau_t, "active_fraction": stt["active_fraction"],
               "max_latency_ns": stt["max_latency_ns"]}
    except RuntimeError as ex:
        thr = {"failed": str(ex)}

    # e2e through the C-ABI with host buffers: the DB stays in pinned host memory and every
    # CTA stages its window from it by TMA (pl_pipeline_bind_host); the step's result is the
    # device-reduced summary (one 56-byte D->H read).  Host wall clock, synchronised.
    e2e = None
    if not a.no_e2e:
        host = torch.from_numpy(wl.db.view("int32")).pin_memory()
        ple = Pipeline(run_cfg, wl, flags=0, stream=stream)
        ple.bind_host(host.data_ptr(), wl.db_len)
        for _ in range(3):
            ple.launch()
            ple.summary()
        s0 = ple.stats()
        torch.cuda.synchronize()
        # pipelined steps (pl_pipeline_step): step k runs on the device while the host reads
        # step k-1's summary; every step's result crosses to the host inside the timed region
        t0 = time.perf_counter()
        e_roots = 0
        e_miss = 0
        for k in range(a.steps + 1):
            sm_ = ple.step() if k < a.steps else ple.step_finish()
            if sm_ is not None:
                e_roots += sm_["roots"]
                e_miss += sm_["miss_events_ns"]
        e_dt = time.perf_counter() - t0
        s1 = ple.stats()
        s2 = ple.stats()                 # the size of one stats read, to exclude it
        ple.close()
        et = torch.tensor([e_dt], dtype=torch.float64, device=dev)
        er = torch.tensor([e_roots, e_miss], dtype=torch.int64, device=dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
            dist.all_reduce(er, op=dist.ReduceOp.SUM)
        e2e_tma = {"value": int(er[0].item()) / float(et.item()), "unit": "items/s",
                   "h2d_bytes_per_step": int(wl.db.nbytes),
                   "d2h_bytes_per_step": (s1["d2h_bytes"] - s0["d2h_bytes"] - (s2["d2h_bytes"] - s1["d2h_bytes"])) // a.steps,
                   "path": "pl_pipeline_bind_host: CTAs pull their DB windows from pinned host memory by TMA "
                           "(cp.async.bulk) every step; pl_pipeline_step: each step's pl_summary is copied to "
                           "pinned host memory and read by the host while the next step runs",
                   "misses": int(er[1].item())}

        # staged: every step's DB is copied host -> device (cudaMemcpyAsync from pinned memory on a
        # copy stream, double-buffered) while the previous step runs, then bound with
        # pl_pipeline_bind_device; results as above (pl_pipeline_step)
        dbufs = [torch.empty_like(db_dev), torch.empty_like(db_dev)]
        cps = torch.cuda.Stream(dev)
        ev_copy = [torch.cuda.Event(), torch.cuda.Event()]
        ev_used = [torch.cuda.Event(), torch.cuda.Event()]
        pls = Pipeline(run_cfg, wl, flags=0, stream=stream)
        pls.bind_device(db_ptr, wl.db_len)
        for _ in range(3):
            pls.launch()
            pls.summary()
        s0 = pls.stats()
        for b in range(2):
            ev_used[b].record(stream)
        torch.cuda.synchronize()
        t0 = time.perf_counter()
        e_roots = e_miss = 0
        h2d = 0
        for k in range(a.steps + 1):
            if k < a.steps:
                b = k & 1
                with torch.cuda.stream(cps):
                    cps.wait_event(ev_used[b])            # the step that last read this buffer is done
                    dbufs[b].copy_(host, non_blocking=True)
                    ev_copy[b].record(cps)
                h2d += host.nbytes
                stream.wait_event(ev_copy[b])
                pls.bind_device(dbufs[b].data_ptr(), wl.db_len)
                sm_ = pls.step()
                ev_used[b].record(stream)
            else:
                sm_ = pls.step_finish()
            if sm_ is not None:
                e_roots += sm_["roots"]
                e_miss += sm_["miss_events_ns"]
        e_dt = time.perf_counter() - t0
        s1 = pls.stats()
        s2 = pls.stats()
        pls.close()
        et = torch.tensor([e_dt], dtype=torch.float64, device=dev)
        er = torch.tensor([e_roots, e_miss], dtype=torch.int64, device=dev)
        if world > 1:
            dist.all_reduce(et, op=dist.ReduceOp.MAX)
            dist.all_reduce(er, op=dist.ReduceOp.SUM)
        e2e = {"value": int(er[0].item()) / float(et.item()), "unit": "items/s",
               "h2d_bytes_per_step": h2d // a.steps,
               "d2h_bytes_per_step": (s1["d2h_bytes"] - s0["d2h_bytes"] - (s2["d2h_bytes"] - s1["d2h_bytes"])) // a.steps,
               "path": "every step: the DB copied host -> device from pinned memory (cudaMemcpyAsync on a copy "
                       "stream, double-buffered, overlapping the previous step) and bound with "
                       "pl_pipeline_bind_device; pl_pipeline_step: each step's pl_summary is copied to pinned "
                       "host memory and read by the host while the next step runs",
               "misses": int(er[1].item()), "tma_from_host": e2e_tma}

    # roofline of the dominant kernel (the executor): algorithmic bytes / launch time
    pk, pk_src = peaks()
    bytes_per_launch = 0.25 * st_last["roots"] / max(1, world) + 24.0 * st["matches"]
    achieved = bytes_per_launch / (tot_ms / a.steps * 1e-3) / 1e9
    cpu = None
    if rank == 0 and not a.no_cpu_baseline:
        rate, cores, dt, r = oracle_rate(logical_cfg(base), wl, min(a.cpu_sample_streams, a.streams))
        cpu = {"value": rate, "unit": "items/s", "cores": cores, "kind": "oracle",
               "sample": f"{min(a.cpu_sample_streams, a.streams)} of {a.streams} c2 streams ({r} roots), "
                         f"logical clock, Table-1 timing, {dt:.1f} s"}
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "items/s", "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": tot_ms / a.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": WORKLOAD, "policy": "FIXED_WAIT", "clock": "globaltimer (1 unit = 1 ns)",
                       "drain": ("eager (R-DRAIN: every node work-conserving once the stream's last root "
                                 "has arrived; PL_EAGER_DRAIN)" if a.drain == "eager" else "periodic (paper rule)"),
                       "deadline_ns": a.deadline_ns, "tau0_ns": tau, "rate_criterion": rate_criterion,
                       "b": list(C.PAPER_B),
                       "budgets_ns": list(budgets), "w_ns": list(w), "gains": [round(g, 5) for g in gains],
                       "streams_per_gpu": a.streams, "l2": "flushed between timed steps (256 MiB memset)",
                       "parallelism": f"{a.streams} streams x {world} GPUs (independent; NCCL stats all-reduce)"},
            "misses": misses_all, "schedule_misses": sched_misses_all, "overruns": overruns_all, "errors": errors,
            "max_lateness_ns": lateness,
            "sustained_items_per_s": world * a.streams * 1e9 / tau,
            "logical_items_per_s": logical_ips,
            "threshold_slack": thr,
            "other_drain": other,
            "utilisation": {"enforced_model": st_last["active_fraction"], "enforced_fig1_T": T,
                            "enforced_hw_busy": st["hw_busy_fraction"], "monolithic": mono},
            "per_firing": {f"node{i}": {"firings": st["firings"][i],
                                        "scheduler_cycles": round(st["phase_cycles"][i][0] / max(1, st["firings"][i])),
                                        "firing_cycles": round(sum(st["phase_cycles"][i][1:5]) / max(1, st["firings"][i])),
                                        "publish_cycles": round(st["phase_cycles"][i][5] / max(1, st["firings"][i])),
                                        "mean_fire_ns": round(st["busy_ns"][i] / max(1, st["firings"][i])),
                                        "max_fire_ns": st["max_fire_ns"][i],
                                        "max_loop_ns": st["max_loop_ns"][i]} for i in range(st["n_stages"])},
            "clocks": clk,
            "e2e": e2e,
            "gpu_launches": a.steps,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": pk, "unit": "GB/s", "frac": achieved / pk,
                         "traffic": ncu_traffic(), "peak_source": pk_src,
                         "algorithmic_bytes_per_launch": bytes_per_launch},
            # the bound that actually sets the rate: Fig. 1 stability (L125/L145) needs
            # P_0 = t_0 + w_0 <= v tau0, so tau0 >= t_0 / v at node 0's calibrated budget
            "rate_bound": {"bound": "node-0 service time (Fig. 1 stability: tau0 >= t_0/v)",
                           "achieved": world * a.streams * 1e9 / tau,
                           "peak": world * a.streams * cfg.vector_width * 1e9 / budgets[0],
                           "unit": "items/s",
                           "frac": (world * a.streams * 1e9 / tau) / (world * a.streams * cfg.vector_width * 1e9 / budgets[0]),
                           "t0_ns": budgets[0], "v": cfg.vector_width},
            "cpu_baseline": cpu,
        }
        print(json.dumps(line), flush=True)
    pl.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
