"""Cross-GPU reduction of executor statistics.

Streams are independent pipeline instances (§2.2: one processor per
application instance), so ranks share no data; the only collective is one
all-reduce of the int64 counter vector (SUM) and one of the maxima (MAX), over
NCCL on NVLink/NVSwitch (gloo on CPU for tests).
"""
from __future__ import annotations

SUM_KEYS = ("roots", "firings", "empty_firings", "consumed", "produced", "active_window", "busy_ns",
            "spilled", "overruns", "stalls", "matches", "miss_events", "miss_events_ns", "misses", "window", "t_end",
            "latency_outliers", "window_refills")
MAX_KEYS = ("max_lateness_ns", "max_fire_ns", "max_loop_ns", "max_latency", "max_latency_ns", "wall_ns",
            "max_queue")


def _flatten(st, keys):
    out = []
    for k in keys:
        v = st[k]
        out.extend(int(x) for x in (v if isinstance(v, (list, tuple)) else [v]))
    return out


def _unflatten(st, keys, vals):
    res = dict(st)
    i = 0
    for k in keys:
        v = st[k]
        if isinstance(v, (list, tuple)):
            res[k] = [int(x) for x in vals[i:i + len(v)]]
            i += len(v)
        else:
            res[k] = int(vals[i])
            i += 1
    return res


def allreduce_stats(st: dict, device=None) -> dict:
    """SUM the counters and MAX the maxima of a pl_stats dict over all ranks.
    The active fractions are recomputed from the reduced sums."""
    import torch
    import torch.distributed as dist
    if not (dist.is_available() and dist.is_initialized()) or dist.get_world_size() == 1:
        return st
    sk = [k for k in SUM_KEYS if k in st]
    mk = [k for k in MAX_KEYS if k in st]
    s = torch.tensor(_flatten(st, sk), dtype=torch.int64, device=device)
    # the maxima, then the error flags one bit per slot (a MAX of whole bitmasks would lose bits)
    m = torch.tensor(_flatten(st, mk) + [(int(st.get("errors", 0)) >> b) & 1 for b in range(32)],
                     dtype=torch.int64, device=device)
    dist.all_reduce(s, op=dist.ReduceOp.SUM)
    dist.all_reduce(m, op=dist.ReduceOp.MAX)
    res = _unflatten(st, sk, s.tolist())
    mv = m.tolist()
    res = _unflatten(res, mk, mv[:len(mv) - 32])
    res["errors"] = sum(int(x) << b for b, x in enumerate(mv[len(mv) - 32:]))
    N = st["n_stages"]
    mono = st.get("policy") == 2
    if res["window"]:
        act = sum(res["active_window"][:N])
        res["active_fraction"] = act / (res["window"] * (1 if mono else N))
    res["n_ranks"] = dist.get_world_size()
    return res
