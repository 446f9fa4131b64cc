#!/usr/bin/env python
"""bench.py — sustained items/s at zero deadline misses of the enforced-waiting executor.

Metric (BASELINE.json): "items/s at 0 deadline misses; SM utilisation vs no-wait baseline".

Workload (default, BASELINE.json configs[3], the largest single-GPU config):
the BLAST-style 4-stage pipeline (seed lookup -> hit enumeration -> ungapped window filter ->
X-drop extension) over a seeded synthetic 100 Mbp DB with heavy-tailed hit amplification (a
1 kbp query with tandem-repeat motif blocks, Pareto(1.5) repeat islands, 6400 planted matches),
one independent stream per CTA on all 148 SMs: 708 K roots per stream, each stream's DB
range slid through a 64 KB smem window by TMA (a1).  Physical %globaltimer clock, 1 unit = 1 ns.
``--workload c2`` runs BASELINE configs[1] (1 Mbp, 148 streams of 7 K roots) instead.

Procedure:
  1. gains g_i from a logical-clock run; service-time budgets t_i = 1.1 x the longest firing
     of a full-vector physical probe + 128 ns, re-measured at the operating point;
  2. the deadline D (c4: 3.5 ms) with a platform-stall allowance of 2.7 ms (reading R-STALL:
     the B200 stops every SM for ~1.6 ms every few seconds, profiles/r02_pause_control.txt, and
     the pipeline needs a few hundred us to catch up): THRESHOLD_SLACK reserves it in every R_i,
     FIXED_WAIT / MONOLITHIC solve Fig. 1 / Fig. 2 at D - 2.7 ms (the schedulable deadline,
     0.8 ms);  b = (1, 3, 9, 6) (L230);
  3. the headline policy is the north_star's THRESHOLD_SLACK rule; tau0 = the smallest
     inter-arrival whose physical run has zero deadline misses (measured), no overflow;
  4. the timed steps run with PL_FIXED_SERVICE (a firing's outputs appear at start + t_i, the
     paper's fixed service time, L69), so every item's measured latency is checked on the
     device against its logical-clock prediction (north_star 5 %; reading R-AGREE).
value = roots processed / device time of the timed launches (CUDA events on the launch stream,
L2 flushed between steps), whole job over all ranks (max-over-ranks time).  FIXED_WAIT (the
paper's rule) and the MONOLITHIC no-internal-wait baseline (§5, Fig. 2) are measured
beside it, and the utilisation of enforced waiting vs monolithic at a common rate.
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
WORKLOADS = {
    "c4": ("c4: BLAST seed-lookup -> hit-enumeration -> ungapped-window -> x-drop, 100 Mbp synthetic DB with "
           "heavy-tailed hit amplification (tandem-repeat query motifs, Pareto(1.5) repeat islands; seed 4 + rank), "
           "1 kbp query, 6400 planted matches, 148 streams x 708 K roots (1 CTA each) per GPU"),
    "c2": ("c2: BLAST seed-lookup -> hit-enumeration -> ungapped-window -> x-drop, 1 Mbp synthetic DB "
           "(seed 2 + rank), 1 kbp query, 64 planted matches, 148 streams (1 CTA each) per GPU"),
}
# c4 schedule parameters of the last GPU bench (profiles/r02_bench_c4_v1.json), for the reference arm,
# which must not load the product library: the oracle simulates the same schedule (1 unit = 1 ns)
REF_C4 = dict(budgets=(8330, 12343, 6113, 12660), tau0=2625, gains=(0.04995, 8.9465, 0.56093))   # profiles/r02_bench_c4_final.json


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=20)
    ap.add_argument("--warmup", type=int, default=5)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--workload", default="c4", choices=["c4", "c2"])
    ap.add_argument("--deadline-ns", type=int, default=None, help="D (default: c4 3.5 ms, c2 350 us)")
    ap.add_argument("--stall-guard-ns", type=int, default=None,
                    help="platform-stall allowance reserved out of D (R-STALL: a ~1.6 ms stall plus the "
                         "catch-up after it; default: c4 2.7 ms, c2 0)")
    ap.add_argument("--streams", type=int, default=148)
    ap.add_argument("--cpu-sample-roots", type=int, default=3000, help="oracle sample: first R roots per stream")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-side", action="store_true", help="skip the FIXED_WAIT / MONOLITHIC side measurements")
    ap.add_argument("--no-stages", action="store_true", help="skip the per-stage K-BENCH kernels (stage_rooflines)")
    ap.add_argument("--budget-margin", type=float, default=1.10,
                    help="t_i = margin x longest measured firing + slack (SURVEY 8(d): x1.1)")
    ap.add_argument("--budget-slack", type=int, default=128)
    ap.add_argument("--refine", type=int, default=None,
                    help="budget refinement rounds at the operating point (default c2: 2; c4: 0 -- on c4 the "
                         "refinement runs at the fastest stall-free rate, far below the injected-stall edge, where "
                         "back-pressure inflates node 2's loop time to twice its firing: profiles/r02_ab/bench_c4_refine0_*.json)")
    ap.add_argument("--confirm", type=int, default=3,
                    help="confirmation runs the operating point must pass (else +10 %% and retry)")
    ap.add_argument("--inject-period-ms", type=float, default=None,
                    help="rate searches inject a platform-length stall every this many ms "
                         "(pl_pipeline_inject_stalls; default: c4 100, c2 off)")
    ap.add_argument("--inject-ms", type=float, default=1.8, help="length of an injected stall (R-STALL: ~1.6 ms)")
    ap.add_argument("--probe-t", type=int, default=None,
                    help="budget probe: every node's budget during the probe (ns; default c4 1000 = all nodes "
                         "overloaded, sharing the SM as in a catch-up, L69's 1/N share; c2 20000)")
    ap.add_argument("--lat-margin", type=float, default=0.85,
                    help="rate search across injected stalls: a trial also needs its largest measured latency "
                         "<= lat_margin x D (near the edge the worst latency is not monotone in tau0)")
    ap.add_argument("--headroom", type=float, default=1.08,
                    help="operating tau0 = headroom x the fastest tau0 miss-free across injected stalls "
                         "(R-STALL: the pipeline must catch up after a ~1.6 ms platform stall within D; the "
                         "injected stalls sample ~20 stream phases per run, a platform stall lands anywhere, "
                         "and 1.5 %% below the edge the catch-up fails by tens of ms: "
                         "profiles/r02_bench_c4_edge_miss.json)")
    a = ap.parse_args()
    if a.deadline_ns is None:
        a.deadline_ns = 3_500_000 if a.workload == "c4" else 350_000
    if a.refine is None:
        a.refine = 0 if a.workload == "c4" else 2
    if a.inject_period_ms is None:
        a.inject_period_ms = 100.0 if a.workload == "c4" else 0.0
    if a.stall_guard_ns is None:
        a.stall_guard_ns = 2_700_000 if a.workload == "c4" else 0
    return a


def base_config(a, rank=0):
    if a.workload == "c4":
        return C.c4(n_streams=a.streams, seed=4 + rank)
    return C.c2(n_streams=a.streams, seed=2 + rank)


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


def ncu_summary(workload):
    """dram bytes and issue figures per launch of the executor from the committed ncu capture."""
    try:
        with open(os.path.join(ROOT, "profiles", f"ncu_summary_{workload}.json")) as f:
            return json.load(f)
    except (OSError, ValueError):
        return {}


def stage_rooflines(base, wl, db_ptr, stream, pk, workload, reps=3):
    """K-BENCH (north_star: "the achieved HBM GB/s of each stage kernel"): every DNA stage over
    this rank's whole DB through pl_stage_batch (S0 over every root, then each stage over the
    previous one's outputs), CUDA events on the launching stream, `reps` launches per stage after
    one warm-up.  Algorithmic bytes: S0 0.25 B per root in + 8 B per output; S1, S2 8 B per input
    + 8 B per output; S3 8 B per input + 24 B per match.  `dram_bytes` is ncu's traffic of the same
    launch from the committed capture (profiles/ncu_kbench_<workload>.json), null if absent."""
    import torch
    from paper_conf_icppw_planob21_b200 import Pipeline
    try:
        with open(os.path.join(ROOT, "profiles", f"ncu_kbench_{workload}.json")) as f:
            ncu = json.load(f)
    except (OSError, ValueError):
        ncu = {}
    k = base.stages[0].iparam[0]
    R = wl.db_len - k + 1
    pl = Pipeline(base.replace(wait_time=(0,) * base.n_stages), wl, flags=0, stream=stream)
    pl.bind_device(db_ptr, wl.db_len)
    cap = R + (R >> 1) + (1 << 20)
    bufs = [torch.empty((cap, 2), dtype=torch.int32, device="cuda") for _ in range(2)]
    names = ["S0 seed lookup", "S1 hit enumeration", "S2 window filter", "S3 X-drop"]
    out, n_in, src = [], R, 0
    for st in range(base.n_stages):
        dst = bufs[st % 2].data_ptr() if st + 1 < base.n_stages else 0
        ocap = cap if st + 1 < base.n_stages else 0
        pl.stage_batch(st, src, n_in, 0, dst, ocap)              # warm-up
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        for _ in range(reps):
            n_out, _ = pl.stage_batch(st, src, n_in, 0, dst, ocap)
        e1.record(stream)
        torch.cuda.synchronize()
        sec = e0.elapsed_time(e1) * 1e-3 / reps
        alg = (0.25 if st == 0 else 8.0) * n_in + (24.0 if st + 1 == base.n_stages else 8.0) * n_out
        rec = {"stage": names[st] if st < 4 else str(st), "inputs": n_in, "outputs": n_out,
               "us": round(sec * 1e6, 1), "items_per_s": n_in / sec, "algorithmic_GBps": alg / sec / 1e9,
               "frac_hbm_algorithmic": alg / sec / 1e9 / pk}
        d = ncu.get(str(st))
        if d:
            rec.update(dram_bytes=d["dram_bytes"], dram_GBps_ncu=d["dram_GBps"], frac_hbm_dram_ncu=d["dram_GBps"] / pk,
                       issue_active_pct=d["issue_active_pct"])
        out.append(rec)
        n_in, src = n_out, dst
    pl.close()
    return {"kernel": "pl_kbench_kernel<KIND> (pl_stage_batch)", "peak_GBps": pk, "reps": reps, "stages": out,
            "ncu_source": ncu.get("source")}


# --------------------------------------------------------------- oracle legs
def oracle_config(a, base):
    """The bench's schedule for the oracle, built without the product library: the headline
    THRESHOLD_SLACK rule with the last measured c4 budgets / rate (REF_C4), thresholds from the
    oracle's own Fig. 1 solver (oracle.run.oracle_schedule), 1 unit = 1 ns."""
    from oracle import run as OR
    if a.workload == "c4":
        cfg = base.replace(service_time=REF_C4["budgets"], interarrival=REF_C4["tau0"], gain=REF_C4["gains"],
                           deadline=a.deadline_ns - a.stall_guard_ns, b=C.PAPER_B, policy=C.THRESHOLD_SLACK)
        cfg = OR.oracle_schedule(cfg, gains=REF_C4["gains"])
        return cfg.replace(deadline=a.deadline_ns, slack_guard=max(REF_C4["budgets"]) + a.stall_guard_ns)
    return OR.oracle_schedule(base.replace(gain=C.TABLE1_G, policy=C.THRESHOLD_SLACK))


def run_reference(a):
    """--impl reference: the oracle (a plain Python DES, as it stands) on the host cores, on the
    same workload and schedule; each step a bounded sample (the first R roots of every stream)."""
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    from oracle import run as OR
    base = base_config(a)
    wl = G.make_dna(base.seed, **base.dna)
    cfg = oracle_config(a, base)
    R = a.cpu_sample_roots
    for _ in range(a.warmup):
        OR.time_oracle(cfg, wl, a.streams, max_roots=max(1, R // 10))
    times, roots, cores = [], 0, 0
    for _ in range(a.steps):
        r = OR.time_oracle(cfg, wl, a.streams, max_roots=R)
        times.append(r["seconds"])
        roots, cores = r["roots"], r["cores"]
    V = roots * a.steps / sum(times)
    line = {"metric": METRIC, "value": V, "unit": "items/s", "n_gpus": a.gpus, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": 1e3 * sum(times) / a.steps, "higher_is_better": True,
            "scaling": "weak", "vs_baseline": None, "dtype": "int64", "data": "synthetic",
            "impl": "reference",
            "config": {"workload": WORKLOADS[a.workload], "policy": "THRESHOLD_SLACK",
                       "clock": "logical (oracle DES, 1 unit = 1 ns)", "deadline_ns": a.deadline_ns,
                       "tau0_ns": cfg.interarrival, "budgets_ns": list(cfg.service_time)},
            "cpu_baseline": {"value": V, "unit": "items/s", "cores": cores, "kind": "oracle",
                             "sample": f"{a.streams} streams x first {R} roots ({roots} roots) per step"},
            "e2e": {"value": V, "unit": "items/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def cpu_baseline(a, base, wl):
    from oracle import run as OR
    cfg = oracle_config(a, base)
    many = OR.time_oracle(cfg, wl, a.streams, max_roots=a.cpu_sample_roots)
    one = OR.time_oracle(cfg, wl, 4, max_roots=a.cpu_sample_roots, procs=1)
    return {"value": many["value"], "unit": "items/s", "cores": many["cores"], "kind": "oracle",
            "sample": f"{a.streams} streams x first {a.cpu_sample_roots} roots ({many['roots']} roots), logical "
                      f"clock, the bench's schedule (1 unit = 1 ns), {many['seconds']:.1f} s",
            "single_core": {"value": one["value"], "roots": one["roots"], "seconds": one["seconds"]},
            "os_cpu_count": os.cpu_count(), "affinity": len(os.sched_getaffinity(0))}


# ------------------------------------------------------------------ our arm
def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
        return
    import torch
    import torch.distributed as dist
    from paper_conf_icppw_planob21_b200 import Pipeline, realtime
    from paper_conf_icppw_planob21_b200._pl import PL_FIXED_SERVICE
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

    def all_max(x):
        if world == 1:
            return x
        t = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        return float(t.item())

    c4 = a.workload == "c4"
    t_setup = time.time()
    base = base_config(a, rank)
    wl = G.make_dna(base.seed, **base.dna)
    db_dev = torch.from_numpy(wl.db.view("int32")).to(dev)
    db_ptr = db_dev.data_ptr()
    stream = torch.cuda.current_stream(dev)
    over = dict(match_capacity=1 << 25, spill_capacity=1 << 19) if c4 else {}
    D, SG = a.deadline_ns, a.stall_guard_ns

    # 1. gains (logical run) and budgets (physical probe, refined at the operating point)
    gains = realtime.measure_gains(base.replace(wait_time=(0,) * 4), wl, db_ptr, stream=stream, over=over)
    # c4: the probe overloads every node (budgets of 1 us at tau0 = 20 ns), so that all four
    # fire back to back and share the SM -- the 1/N processor share at which PAPER.md L69 defines
    # t_i (profiles/r02_c4_probe.txt: 1.3-2.4x the firing times of an isolated node).  A
    # pipeline recovering from a platform stall runs exactly like that.
    budgets, cal = realtime.calibrate_budgets(base, wl, db_ptr, stream=stream, margin=a.budget_margin,
                                              slack_ns=a.budget_slack, probe_tau=20 if c4 else 100, over=over,
                                              probe_t=a.probe_t or (1000 if c4 else 20_000))
    # misses count against D; the schedules are solved at D - SG (R-STALL) and THRESHOLD_SLACK
    # reserves SG in every R_i on top of the largest budget
    cfg0 = base.replace(clock=1, ns_per_unit=1.0, service_time=budgets, gain=gains, deadline=D,
                        b=C.PAPER_B, eager_drain=not c4)
    thr_cfg = lambda b: cfg0.replace(service_time=tuple(b), slack_guard=int(max(b)) + SG)
    if a.refine:
        try:
            budgets, _ = realtime.refine_budgets(thr_cfg(budgets), wl, db_ptr, budgets, margin=a.budget_margin,
                                                 slack_ns=a.budget_slack, rounds=a.refine, stream=stream, log=log,
                                                 over=over, policy=1, max_lateness_ns=None, solve_deadline=D - SG,
                                                 guard_extra=SG, flags=0,   # publish mode: the work's own duration
                                                 lower=not c4)
        except RuntimeError as ex:   # no operating point for the refinement: keep the probe's budgets
            log({"refine_budgets": "skipped", "error": str(ex)})
    if world > 1:   # every rank runs the same schedule: max budgets are conservative
        t = torch.tensor(budgets, dtype=torch.int64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        budgets = tuple(int(x) for x in t.tolist())
    log({"gains": gains, "budgets_ns": budgets, "cal_max_fire_ns": cal["max_fire_ns_runs"],
         "setup_s": round(time.time() - t_setup, 1)})
    cfg = thr_cfg(budgets)

    # 2./3. the fastest miss-free rate of the headline policy (THRESHOLD_SLACK; Fig. 1 thetas)
    inject = (int(a.inject_period_ms * 1e6), int(a.inject_ms * 1e6)) if a.inject_period_ms > 0 else None
    tau, w, th, T, st_ok = realtime.find_rate(cfg, wl, db_ptr, stream=stream, log=log, policy=1, over=over,
                                              max_lateness_ns=None, grow=1.5 if c4 else 1.15, tries=16,
                                              flags=PL_FIXED_SERVICE, solve_deadline=D - SG, max_outliers=0,
                                              inject=inject,
                                              max_latency_ns=int(a.lat_margin * D) if inject else None)
    # the operating point: headroom over the edge the search found on stall-free runs, so that
    # the pipeline catches up after a platform stall within D (R-STALL); confirmed by --confirm
    # runs with zero measured misses whether or not they meet a stall, and zero latency
    # outliers in those that do not; else back off by 10 %
    tau_edge = tau
    tau = int(math.ceil(a.headroom * tau_edge))
    confirm_log = []
    # the confirmation runs meet the timed steps' conditions: L2 flushed before each (a cold L2
    # slows the first firings; on c2's 0.4 ms launches that alone produced misses at the edge)
    flush = torch.empty(256 << 20, dtype=torch.uint8, device=dev)
    for _ in range(8):
        w, th, T = realtime.solve_at(cfg.replace(deadline=D - SG), tau)
        cc = cfg.replace(interarrival=tau, wait_threshold=tuple(th), wait_time=tuple(w), policy=1)
        bad, stalls = 0, 0
        for _ in range(a.confirm):
            pc = Pipeline(cc, wl, flags=PL_FIXED_SERVICE, stream=stream, **over)
            pc.bind_device(db_ptr, wl.db_len)
            flush.zero_()
            pc.launch()
            sc = pc.stats()
            pc.close()
            st_ = realtime.stalled(sc)
            stalls += st_
            bad += sc["miss_events_ns"] + (0 if st_ else sc["latency_outliers"]) + (sc["errors"] != 0)
        confirm_log.append({"tau0_ns": tau, "bad": bad, "stalled_runs": stalls})
        bad = int(all_max(bad))
        if bad == 0:
            break
        tau = int(math.ceil(tau * 1.03))
    log({"confirm": confirm_log})
    tau = int(all_max(tau))
    w, th, T = realtime.solve_at(cfg.replace(deadline=D - SG), tau)
    run_cfg = cfg.replace(interarrival=tau, wait_threshold=tuple(th), wait_time=tuple(w), policy=1)
    pl = Pipeline(run_cfg, wl, flags=PL_FIXED_SERVICE, stream=stream, **over)
    pl.bind_device(db_ptr, wl.db_len)

    for _ in range(a.warmup):
        pl.launch()
    torch.cuda.synchronize()
    if world > 1:
        dist.barrier()
    clocks = ClockSampler(local)
    clocks.start()
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(a.steps)]
    acc = dict(roots=0, misses=0, sched_misses=0, overruns=0, outliers=0, errors=0, lateness=0, relerr=0.0,
               max_lat=0, stall_steps=0, outliers_clean=0, relerr_clean=0.0)
    torch.cuda.synchronize()
    for k in range(a.steps):
        flush.zero_()                                  # L2 flush, outside the timed region
        ev[k][0].record(stream)
        pl.launch()
        ev[k][1].record(stream)
        st = pl.stats()                                # syncs; outside the timed region
        acc["roots"] += st["roots"]
        acc["misses"] += st["miss_events_ns"]          # measured on %globaltimer
        acc["sched_misses"] += st["miss_events"]       # the logical schedule's own
        acc["overruns"] += sum(st["overruns"])
        acc["outliers"] += st["latency_outliers"]
        if realtime.stalled(st):                       # this step met a platform stall (R-STALL)
            acc["stall_steps"] += 1
        else:
            acc["outliers_clean"] += st["latency_outliers"]
            acc["relerr_clean"] = max(acc["relerr_clean"], st["latency_rel_err_max"])
        acc["errors"] |= st["errors"]
        acc["lateness"] = max(acc["lateness"], max(st["max_lateness_ns"]))
        acc["relerr"] = max(acc["relerr"], st["latency_rel_err_max"])
        acc["max_lat"] = max(acc["max_lat"], st["max_latency_ns"])
    torch.cuda.synchronize()
    clk = clocks.stop()
    step_ms = [e0.elapsed_time(e1) for e0, e1 in ev]
    tot_ms = all_max(sum(step_ms))
    if world > 1:
        dist.barrier()
    st_all = allreduce_stats(dict(st, policy=1), device=dev)
    red = {k: acc[k] for k in ("roots", "misses", "sched_misses", "overruns", "outliers", "stall_steps",
                                "outliers_clean")}
    if world > 1:
        t = torch.tensor(list(red.values()), dtype=torch.int64, device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.SUM)
        red = dict(zip(red, (int(x) for x in t.tolist())))
        acc["lateness"] = int(all_max(acc["lateness"]))
        acc["relerr"] = all_max(acc["relerr"])
        acc["max_lat"] = int(all_max(acc["max_lat"]))
        acc["errors"] = st_all["errors"] | acc["errors"]
    value = red["roots"] / (tot_ms * 1e-3)
    # processor utilisation agreement: measured busy time vs the logical schedule's t_i per firing
    model_busy = sum(st["firings"][i] * budgets[i] for i in range(st["n_stages"]))
    util_ratio = sum(st["busy_ns"]) / model_busy if model_busy else None

    # 4. beside it: FIXED_WAIT (the paper's rule) and MONOLITHIC (the no-wait baseline, Fig. 2)
    side = {}

    def run_once(c, flags=PL_FIXED_SERVICE, inj=None):
        pp = Pipeline(c, wl, flags=flags, stream=stream, **over)
        pp.bind_device(db_ptr, wl.db_len)
        if inj:
            pp.inject_stalls(*inj)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        pp.launch()
        e1.record(stream)
        sx = pp.stats()
        pp.close()
        return {"tau0_ns": c.interarrival, "items_per_s": sx["roots"] / (e0.elapsed_time(e1) * 1e-3),
                "misses": sx["miss_events_ns"], "active_fraction": sx["active_fraction"],
                "active_fraction_nonempty": sx["active_fraction_nonempty"],
                "hw_busy_fraction": sx["hw_busy_fraction"], "max_latency_ns": sx["max_latency_ns"],
                "latency_outliers": sx["latency_outliers"], "errors": sx["errors"]}

    if not a.no_side:
        fcfg = cfg0.replace(service_time=budgets)
        try:   # bounded search: c4 FIXED_WAIT runs last seconds each
            tf, wf, thf, Tf, _ = realtime.find_rate(fcfg, wl, db_ptr, stream=stream, over=over, grow=1.5,
                                                    tries=5 if c4 else 12, max_lateness_ns=None,
                                                    flags=PL_FIXED_SERVICE, solve_deadline=D - SG,
                                                    start=tau if c4 else None, inject=inject)
            side["fixed_wait"] = dict(run_once(fcfg.replace(interarrival=tf, wait_time=tuple(wf))),
                                      w_ns=list(wf), fig1_T=Tf)
        except RuntimeError as ex:
            side["fixed_wait"] = {"failed": str(ex)}
        mcfg = fcfg.replace(policy=2)
        msolve = mcfg.replace(deadline=D - SG)
        tm, found = realtime.min_feasible_tau(fcfg.replace(deadline=D - SG)) or 1, None
        for _ in range(20):
            Mm = realtime.monolithic_at(msolve, tm)
            if Mm is not None:
                r = run_once(mcfg.replace(interarrival=tm, block_size=Mm[0]), flags=0, inj=inject)
                if r["misses"] == 0 and r["errors"] == 0:
                    found = dict(r, M=Mm[0], fig2_objective=Mm[1])
                    break
            tm = int(tm * 1.25) + 1
        side["monolithic"] = found or {"failed": "no miss-free tau0 within 20 tries"}
        # the paper's utilisation comparison (L236-L255) at the headline rate
        Mh = realtime.monolithic_at(msolve, tau)
        side["at_headline_rate"] = {
            "tau0_ns": tau,
            "threshold_slack": {"active_fraction": st_all["active_fraction"],
                                "active_fraction_nonempty": st["active_fraction_nonempty"],
                                "hw_busy_fraction": st["hw_busy_fraction"]},
            "monolithic": dict(run_once(mcfg.replace(interarrival=tau, block_size=Mh[0]), flags=0), M=Mh[0])
            if Mh is not None else {"feasible": False}}

    # e2e through the C-ABI with host buffers, live ingest (a1): every step is one persistent run
    # (pl_pipeline_live_start) that consumes the DB while the host pushes it from host memory --
    # slices of every stream through per-stream device rings smaller than the streams, so the
    # pushes are paced by the executor's consumption (back-pressure) and memory stays bounded;
    # latencies count from each root's nominal arrival r tau0, so a late delivery shows up as a
    # miss.  The step's result crosses back inside the timed region: its match records are written
    # by the executor straight into pinned host memory (pl_pipeline_bind_results) and its summary
    # is read after the drain.  Host wall clock.
    e2e = None
    if not a.no_e2e:
        pls = Pipeline(run_cfg, wl, flags=PL_FIXED_SERVICE, stream=stream, **over)
        pls.bind_device(db_ptr, wl.db_len)
        pls.launch()
        n_res = pls.summary()["matches"]
        cap = n_res + (n_res >> 3) + 4096
        res_host = torch.empty(cap * 6, dtype=torch.int32).pin_memory()
        pls.bind_results(res_host.data_ptr(), cap)
        S_ = a.streams
        rng_w = [pls.stream_words(s_) for s_ in range(S_)]
        slice_w = 1024
        ring_w = 1 << 14 if c4 else 0           # c4: 16 K words (256 K bases) per stream < its 44 K words
        torch.cuda.synchronize()
        s0 = pls.stats()
        steps_e = max(1, min(a.steps, 5 if c4 else a.steps))
        t0 = time.perf_counter()
        e_roots = e_miss = e_matches = e_waits = 0
        e_wait_max = 0
        rows = None
        for k in range(steps_e):
            pls.rewind()
            pls.live_start(ring_w)
            pos = [lo for lo, _ in rng_w]
            while True:
                sl = []
                for s_ in range(S_):
                    e_ = min(pos[s_] + slice_w, rng_w[s_][1])
                    sl.append(wl.db[pos[s_]:e_])
                    pos[s_] = e_
                if not any(len(x) for x in sl):
                    break
                pls.push_all(sl)                # blocks while a ring is full
            pls.drain()
            sm_ = pls.summary()
            stx = pls.stats()
            e_roots += sm_["roots"]
            e_miss += sm_["miss_events_ns"]
            e_matches += sm_["matches"]
            e_waits += stx["ingest_waits"]
            e_wait_max = max(e_wait_max, stx["max_ingest_wait_ns"])
            rows = res_host[: 6 * sm_["matches"]]
        e_dt = time.perf_counter() - t0
        s1 = pls.stats()
        rows = rows.view(-1, 6).numpy()
        ref_rows = pls.results_array() if not c4 else None
        pls.close()
        e_dt = all_max(e_dt)
        e2e = {"value": e_roots * max(1, world) / e_dt, "unit": "items/s",
               "h2d_bytes_per_step": (s1["h2d_bytes"] - s0["h2d_bytes"]) // steps_e,
               "d2h_bytes_per_step": (s1["d2h_bytes"] - s0["d2h_bytes"]) // steps_e + 24 * e_matches // steps_e,
               "path": ("live ingest: pl_pipeline_live_start + pl_pipeline_push_all of 1024-word slices per stream "
                        f"into {'16 K-word' if c4 else 'default'} device rings (back-pressured) while the run executes, "
                        "pl_pipeline_drain; matches written to pinned host memory by the executor"),
               "d2h_detail": "pl_stats / pl_summary + 24 B per match record, written to pinned host memory by the executor",
               "steps": steps_e, "misses": e_miss, "matches_per_step": e_matches // steps_e,
               "ingest_waits": e_waits, "max_ingest_wait_ns": e_wait_max,
               "results_checked": bool(len(rows) == e_matches // steps_e and (rows[:, 4] > 0).all()
                                       and (ref_rows is None or len(ref_rows) == len(rows)))}

    # roofline of the dominant kernel (the executor): algorithmic bytes / launch time
    pk, pk_src = peaks()
    ncu = ncu_summary(a.workload)
    launch_s = tot_ms / a.steps * 1e-3
    bytes_per_launch = 0.25 * st["roots"] + 24.0 * st["matches"]
    achieved = bytes_per_launch / launch_s / 1e9
    cpu = None
    if rank == 0 and not a.no_cpu_baseline:
        cpu = cpu_baseline(a, base, wl)
    v, u = run_cfg.vector_width, run_cfg.stages[1].max_out
    if rank == 0:
        line = {
            "metric": METRIC, "value": value, "unit": "items/s", "n_gpus": world, "steps": a.steps,
            "warmup": a.warmup, "ms_per_step": tot_ms / a.steps, "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "int32", "data": "synthetic",
            "config": {"workload": WORKLOADS[a.workload], "policy": "THRESHOLD_SLACK (north_star rule; Fig. 1 thetas)",
                       "clock": "globaltimer (1 unit = 1 ns)", "service": "PL_FIXED_SERVICE (outputs at start + t_i, L69)",
                       "deadline_ns": D, "stall_guard_ns": SG, "tau0_ns": tau, "theta": list(th),
                       "rate_criterion": ((f"{a.headroom} x the fastest tau0 with zero measured misses across "
                                           f"{a.inject_ms} ms stalls injected every {a.inject_period_ms} ms "
                                           f"(pl_pipeline_inject_stalls; R-STALL) ({tau_edge} ns)") if inject else
                                          (f"{a.headroom} x the fastest tau0 with zero measured misses and zero latency "
                                           f"outliers on stall-free runs ({tau_edge} ns)")) +
                                          f"; then {a.confirm} confirmation runs without injection: zero misses, and "
                                          f"zero latency outliers in those without a platform stall (tries: {confirm_log})",
                       "stall_injection_in_rate_search": ({"period_ms": a.inject_period_ms, "len_ms": a.inject_ms,
                                                           "max_latency_frac_of_D": a.lat_margin}
                                                          if inject else None),
                       "tau0_edge_ns": tau_edge, "edge_items_per_s": world * a.streams * 1e9 / tau_edge,
                       "b": list(C.PAPER_B), "budgets_ns": list(budgets), "budget_probe_t_ns": a.probe_t or (1000 if c4 else 20_000),
                       "gains": [round(g, 5) for g in gains],
                       "drain": "eager (R-DRAIN)" if not c4 else "periodic (paper rule)",
                       "streams_per_gpu": a.streams, "roots_per_stream": st["roots"] // a.streams,
                       "arrival_span_ms": st["roots"] / a.streams * tau * 1e-6,
                       "l2": "flushed between timed steps (256 MiB memset)",
                       "parallelism": f"{a.streams} streams x {world} GPUs (independent; NCCL stats all-reduce)"},
            "misses": red["misses"], "schedule_misses": red["sched_misses"], "overruns": red["overruns"],
            "errors": acc["errors"], "max_lateness_ns": acc["lateness"], "max_latency_ns": acc["max_lat"],
            "agreement": {"criterion": "every terminal item: |measured - logical latency| <= 5 % + 64 ns (R-AGREE)",
                          "items": red["roots"],
                          "latency_outliers": red["outliers"], "latency_rel_err_max": acc["relerr"],
                          "steps_with_platform_stall": red["stall_steps"],
                          "latency_outliers_in_steps_without_stall": red["outliers_clean"],
                          "latency_rel_err_max_without_stall": acc["relerr_clean"],
                          "util_measured_over_model": util_ratio},
            "sustained_items_per_s": world * a.streams * 1e9 / tau,
            "per_rank": {"items_per_s": value / world, "streams": a.streams,
                         "workload_seed": f"4 + rank (c5: every rank its own c4 DB)" if c4 else "2 + rank"},
            "window_refills_per_launch": st["window_refills"],
            "utilisation": {"enforced_model": st_all["active_fraction"], "enforced_hw_busy": st["hw_busy_fraction"],
                            "fig1_T": T},
            "side": side,
            "per_node": {f"node{i}": {"firings": st["firings"][i], "mean_fire_ns": round(st["busy_ns"][i] / max(1, st["firings"][i])),
                                      "max_fire_ns": st["max_fire_ns"][i], "max_loop_ns": st["max_loop_ns"][i],
                                      "spilled": st["spilled"][i], "max_queue": st["max_queue"][i],
                                      # scheduler overhead per firing (north_star): leader-lane clock64
                                      # cycles deciding (phase 0) and reserving/publishing (3, 5)
                                      "sched_cycles_per_firing": round(st["phase_cycles"][i][0] / max(1, st["firings"][i])),
                                      "publish_cycles_per_firing": round((st["phase_cycles"][i][3] + st["phase_cycles"][i][5])
                                                                         / max(1, st["firings"][i])),
                                      "stage_scan_cycles_per_firing": round(st["phase_cycles"][i][2] / max(1, st["firings"][i]))}
                         for i in range(st["n_stages"])},
            "clocks": clk,
            "e2e": e2e,
            "gpu_launches": a.steps,
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": pk, "unit": "GB/s", "frac": achieved / pk,
                         "traffic": ncu.get("dram_bytes_per_launch"), "peak_source": pk_src,
                         "algorithmic_bytes_per_launch": bytes_per_launch,
                         "note": "0.25 B per root (2-bit DB) + 24 B per match; the path is not HBM-bound by design"},
            # the executor's issue-slot use from the committed ncu capture of this configuration
            # (profiles/ncu_summary_<workload>.json): the binding resource of a real-time executor
            # is issue slots and latency chains, not bytes; util_same_rate compares enforced waiting
            # with the monolithic baseline at the same (tau0, D)
            "issue": {k: ncu[k] for k in ("issue_active_pct", "warp_inst_per_launch", "warp_inst_per_root",
                                          "sm_throughput_pct", "util_same_rate", "source") if k in ncu},
            # the bound that sets the c4 rate: a repeat island turns every seed into u S2 items (and up
            # to u S3 items), which nodes 2 and 3 serve v per t_i, so tau0 >= u max(t_2, t_3) / v there
            "rate_bound": {"bound": ("island burst at nodes 2-3 (tau0 >= u max(t_2, t_3) / v: a repeat-island seed "
                                     "becomes u S2 items and up to u S3 items)") if c4 else "node-0 service (tau0 >= t_0/v)",
                           "achieved": world * a.streams * 1e9 / tau,
                           "peak": world * a.streams * 1e9 * v / ((u * max(budgets[2], budgets[3])) if c4 else budgets[0]),
                           "unit": "items/s"},
            "cpu_baseline": cpu,
            # per-stage kernels over the same DB, outside the timed region (north_star: HBM GB/s of each
            # stage kernel against the peak)
            "stages": (None if a.no_stages else
                       stage_rooflines(base, wl, db_ptr, stream, pk, a.workload)),
        }
        rb = line["rate_bound"]
        rb["frac"] = rb["achieved"] / rb["peak"]
        print(json.dumps(line), flush=True)
    pl.close()
    if world > 1:
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
