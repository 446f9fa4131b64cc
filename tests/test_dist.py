"""Cross-rank statistics reduction on CPU with gloo, world_size 2.

Streams are independent, so the only collective is an all-reduce of the counters (SUM)
and the maxima (MAX); the active fraction is recomputed from the reduced sums."""
import os
import socket

import pytest
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _stats(rank):
    N = 2
    return {"n_stages": N, "roots": 100 + rank, "firings": [10 + rank, 5], "empty_firings": [1, rank],
            "consumed": [100 + rank, 50], "produced": [50, 100], "active_window": [640 + rank, 480],
            "busy_ns": [1000 * (rank + 1), 0], "spilled": [0, rank], "overruns": [0, 0], "matches": rank,
            "miss_events": 0, "misses": 0, "window": 400 + 4 * rank, "t_end": 500,
            "max_lateness_ns": [rank * 7, 3], "max_fire_ns": [100 - rank, 50 + rank], "max_loop_ns": [9 + rank, 4], "max_latency": 400 + rank,
            "max_latency_ns": 1000 * rank, "wall_ns": 5 + rank, "errors": 1 << rank, "active_fraction": 0.0,
            "miss_events_ns": rank, "max_queue": [3 + rank, 9 - rank]}


def _worker(rank, port, out):
    import torch.distributed as dist
    from paper_conf_icppw_planob21_b200.dist import allreduce_stats
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=2)
    r = allreduce_stats(_stats(rank))
    out[rank] = r
    dist.destroy_process_group()


def test_allreduce_stats_gloo_two_ranks():
    port = _free_port()
    with mp.Manager() as m:
        out = m.dict()
        mp.spawn(_worker, args=(port, out), nprocs=2, join=True)
        a, b = out[0], out[1]
    assert a == b
    assert a["roots"] == 201 and a["firings"] == [21, 10] and a["empty_firings"] == [2, 1]
    assert a["max_lateness_ns"] == [7, 3] and a["max_fire_ns"] == [100, 51] and a["max_loop_ns"] == [10, 4]
    assert a["max_latency"] == 401 and a["wall_ns"] == 6 and a["matches"] == 1
    assert a["window"] == 804
    assert abs(a["active_fraction"] - (641 + 640 + 960) / (2 * 804)) < 1e-12
    assert a["n_ranks"] == 2
    assert a["errors"] == 3                      # each rank's overflow bit survives the reduction
    assert a["miss_events_ns"] == 1 and a["max_queue"] == [4, 9]


def test_single_process_is_identity():
    from paper_conf_icppw_planob21_b200.dist import allreduce_stats
    s = _stats(0)
    assert allreduce_stats(s) is s
