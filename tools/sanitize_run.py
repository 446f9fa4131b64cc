"""Small executor runs for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys

sys.path.insert(0, ".")
from plgen import configs as C
from plgen import dna as G
from paper_conf_icppw_planob21_b200 import Pipeline

# random-gain pipeline, all policies, forced spills
for policy in (C.FIXED_WAIT, C.THRESHOLD_SLACK, C.MONOLITHIC):
    cfg = C.c1(n_streams=2, n_roots=600, wait_time=(64, 90), wait_threshold=(32, 23), policy=policy, block_size=64)
    pl = Pipeline(cfg, None, flags=7, queue_capacity=32 if policy != C.MONOLITHIC else 0)
    pl.push(None, cfg.n_roots)
    pl.drain()
    print(policy, pl.stats()["firings"][:2], flush=True)
    pl.close()
# DNA pipeline, logical and physical, forced spill
cfg = C.c2(n_streams=3, dna=dict(db_len=1 << 14, q_len=1024, n_planted=4), wait_time=(993, 2422, 965, 1628))
wl = G.make_dna(cfg.seed, **cfg.dna)
for clock in (0, 1):
    c = cfg if clock == 0 else cfg.replace(clock=1, service_time=(4000,) * 4, interarrival=100, wait_time=(0,) * 4,
                                           deadline=10**7)
    pl = Pipeline(c, wl, flags=7, queue_capacity=64)
    pl.push(wl.db, wl.db_len)
    pl.drain()
    print("dna clock", clock, pl.stats()["firings"], flush=True)
    pl.close()
# round 2: the sliding window (small ring), live ingest (a ring smaller than the stream), the N4
# cluster executor (DSMEM queues, forced spills), and injected stalls
import numpy as np  # noqa: E402
c = cfg.replace(policy=C.THRESHOLD_SLACK, wait_threshold=(128, 127, 99, 10))
pl = Pipeline(c, wl, flags=7, window_words=256, window_chunk_words=64)
pl.push(wl.db, wl.db_len)
pl.drain()
print("sliding window refills", pl.stats()["window_refills"], flush=True)
pl.close()
pl = Pipeline(c, wl, flags=7, window_words=256, window_chunk_words=64)
pl.live_start(512)
rng = [pl.stream_words(s) for s in range(c.n_streams)]
pos = [lo for lo, _ in rng]
while any(pos[s] < rng[s][1] for s in range(c.n_streams)):
    sl = []
    for s in range(c.n_streams):
        e = min(pos[s] + 61, rng[s][1])
        sl.append(wl.db[pos[s]:e])
        pos[s] = e
    pl.push_all(sl)
pl.drain()
print("live ingest", pl.stats()["firings"], flush=True)
pl.close()
pl = Pipeline(c, wl, flags=7 | 32, queue_capacity=64)
pl.push(wl.db, wl.db_len)
pl.drain()
print("cluster", pl.stats()["firings"], flush=True)
pl.close()
p = c.replace(clock=1, service_time=(4000,) * 4, interarrival=100, deadline=10**7)
pl = Pipeline(p, wl, flags=7 | 8)
pl.push(wl.db, wl.db_len)
pl.inject_stalls(200_000, 50_000)
pl.drain()
print("injected stalls", pl.stats()["max_lateness_ns"], flush=True)
pl.close()
# K-BENCH stage kernels (pl_kbench_kernel<KIND>): every stage of a heavy-tailed DNA workload
# whose extension walks reach both DB ends, and a random-gain chain
import torch  # noqa: E402
cfg = C.c2(n_streams=1, dna=dict(db_len=40_003, q_len=1024, n_planted=12, heavy_tailed=True), wait_time=(0,) * 4)
wl = G.make_dna(cfg.seed, **cfg.dna)
pl = Pipeline(cfg, wl, flags=0)
pl.push(wl.db, wl.db_len)
R = wl.db_len - 6 + 1   # k = 6
bufs = [torch.empty((R * 16, 2), dtype=torch.int32, device="cuda") for _ in range(2)]
n_in, src = R, 0
for st in range(4):
    out = bufs[st % 2].data_ptr() if st < 3 else 0
    n_out, _ = pl.stage_batch(st, src, n_in, 0, out, R * 16 if st < 3 else 0)
    print("kbench stage", st, n_in, "->", n_out, flush=True)
    n_in, src = n_out, out
pl.close()
cfg = C.c1(n_streams=1, n_roots=5000, wait_time=(64, 90))
pl = Pipeline(cfg, None, flags=0)
pl.push(None, cfg.n_roots)
buf = torch.empty((5000 * 4, 2), dtype=torch.int32, device="cuda")
n0, _ = pl.stage_batch(0, 0, 5000, 0, buf.data_ptr(), 5000 * 4)
print("kbench gain model stage 0", n0, flush=True)
pl.close()
