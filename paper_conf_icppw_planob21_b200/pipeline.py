"""Python face of the C-ABI (include/pl.h): the same calls, marshalled with ctypes.

``Pipeline`` mirrors pl_pipeline_* one to one; ``solve_enforced_waits`` /
``solve_monolithic`` mirror pl_solve_*.  A configuration is any object with the
attributes of ``plgen.configs.Config`` (stages, service_time, vector_width, ...).
"""
from __future__ import annotations

import ctypes as C

import numpy as np

from . import _pl
from ._pl import check, lib


def _arr(ctype, xs):
    if xs is None:
        return None
    a = (ctype * len(xs))(*xs)
    return a


def make_config(cfg, flags=0, device=0, n_streams=None, **over):
    """Build a ``pl_config`` (and keep its arrays alive) from a Config-like object."""
    N = len(cfg.stages)
    st = (_pl.pl_stage * N)()
    for i, s in enumerate(cfg.stages):
        st[i].kind = s.kind
        st[i].max_out = s.max_out
        st[i].param = float(s.param)
        for j in range(4):
            st[i].iparam[j] = int(s.iparam[j]) if j < len(s.iparam) else 0
    keep = [st]
    c = _pl.pl_config()
    c.n_stages = N
    c.stages = st
    t = _arr(C.c_int64, [int(x) for x in cfg.service_time]); keep.append(t)
    c.service_time = t
    if getattr(cfg, "gain", None) is not None:
        g = _arr(C.c_double, [float(x) for x in cfg.gain]); keep.append(g)
        c.gain = g
    b = _arr(C.c_uint32, [int(x) for x in cfg.b]); keep.append(b)
    c.b = b
    c.vector_width = cfg.vector_width
    if getattr(cfg, "wait_time", None) is not None:
        w = _arr(C.c_int64, [int(x) for x in cfg.wait_time]); keep.append(w)
        c.wait_time = w
    if getattr(cfg, "wait_threshold", None) is not None:
        th = _arr(C.c_uint32, [int(x) for x in cfg.wait_threshold]); keep.append(th)
        c.wait_threshold = th
    c.deadline = int(cfg.deadline)
    c.interarrival = int(cfg.interarrival)
    c.slack_guard = int(getattr(cfg, "slack_guard", 0))
    c.policy = int(cfg.policy)
    c.clock = int(cfg.clock)
    c.block_size = int(cfg.block_size or 0)
    c.mono_b = int(getattr(cfg, "mono_b", 1) or 1)
    c.mono_S = float(getattr(cfg, "mono_S", 1.0) or 1.0)
    c.n_streams = int(n_streams if n_streams is not None else cfg.n_streams)
    c.n_roots = int(cfg.n_roots or 0)
    c.seed = int(cfg.seed)
    c.device = int(device)
    c.ns_per_unit = float(getattr(cfg, "ns_per_unit", 1.0))
    c.flags = int(flags) | (_pl.PL_EAGER_DRAIN if getattr(cfg, "eager_drain", False) else 0)
    for k, v in over.items():
        setattr(c, k, v)
    return c, keep


class Pipeline:
    """pl_pipeline_* on one handle.  Raises ``PlError`` on every non-OK status."""

    def __init__(self, cfg, workload=None, flags=0, device=0, stream=None, arrivals=None, **over):
        self.cfg = cfg
        self._c, self._keep = make_config(cfg, flags=flags, device=device, **over)
        if arrivals is not None:   # per-root arrival times (pl_config.arrivals; copied at create)
            arr = np.ascontiguousarray(arrivals, dtype=np.int64)
            self._keep.append(arr)
            self._c.arrivals = arr.ctypes.data_as(C.POINTER(C.c_int64))
            self._c.n_arrivals = arr.shape[0]
        wl = None
        if workload is not None:
            q = np.ascontiguousarray(workload.query, dtype=np.uint32)
            self._q = q
            wl = _pl.pl_workload(q.ctypes.data_as(C.POINTER(C.c_uint32)), workload.q_len, workload.db_len)
        h = C.c_void_p()
        check(lib.pl_pipeline_create(C.byref(self._c), C.byref(wl) if wl is not None else None, C.byref(h)),
              "pl_pipeline_create")
        self.h = h
        self.N = len(cfg.stages)
        if stream is not None:
            self.set_stream(stream)

    # -- lifecycle
    def set_stream(self, stream):
        """stream: a torch.cuda.Stream, a raw cudaStream_t int, or None (default stream)."""
        ptr = getattr(stream, "cuda_stream", stream)
        check(lib.pl_pipeline_set_stream(self.h, C.c_void_p(ptr or 0)), "pl_pipeline_set_stream")

    def push(self, items=None, n=None):
        if items is None:
            check(lib.pl_pipeline_push(self.h, None, int(n)), "pl_pipeline_push")
            return
        a = np.ascontiguousarray(items, dtype=np.uint32)
        check(lib.pl_pipeline_push(self.h, a.ctypes.data, int(n)), "pl_pipeline_push")

    def push_ptr(self, host_ptr, n):
        check(lib.pl_pipeline_push(self.h, C.c_void_p(host_ptr), int(n)), "pl_pipeline_push")

    def bind_device(self, dev_ptr, n):
        check(lib.pl_pipeline_bind_device(self.h, C.c_void_p(dev_ptr), int(n)), "pl_pipeline_bind_device")

    def bind_host(self, host_ptr, n):
        """pl_pipeline_bind_host: the DB stays in pinned host memory; CTAs stage it by TMA."""
        check(lib.pl_pipeline_bind_host(self.h, C.c_void_p(host_ptr), int(n)), "pl_pipeline_bind_host")

    def bind_results(self, ptr, cap):
        """pl_pipeline_bind_results: later runs write their match records into `ptr` (device memory
        or pinned+mapped host memory, `cap` records); ptr=None restores the handle's own buffer."""
        check(lib.pl_pipeline_bind_results(self.h, C.c_void_p(ptr or 0), int(cap)), "pl_pipeline_bind_results")

    def queue_peaks(self):
        """pl_pipeline_queue_peaks -> uint32 array [n_streams, N]."""
        n = C.c_uint64()
        check(lib.pl_pipeline_queue_peaks(self.h, None, 0, C.byref(n)), "pl_pipeline_queue_peaks")
        a = np.empty(n.value, dtype=np.uint32)
        check(lib.pl_pipeline_queue_peaks(self.h, a.ctypes.data, n.value, C.byref(n)), "pl_pipeline_queue_peaks")
        return a.reshape(-1, self.N)

    def summary(self) -> dict:
        s = _pl.pl_summary()
        check(lib.pl_pipeline_summary(self.h, C.byref(s)), "pl_pipeline_summary")
        return {k: getattr(s, k) for k, _ in s._fields_}

    # -- live ingest (pl_pipeline_live_start / stream_words / push_stream / push_all)
    def live_start(self, ring_words=0):
        """Launch a persistent run whose DB words arrive by push_stream / push_all while it runs."""
        check(lib.pl_pipeline_live_start(self.h, int(ring_words)), "pl_pipeline_live_start")

    def stream_words(self, s):
        """[word_lo, word_hi) of the packed DB that stream s must be pushed."""
        lo, hi = C.c_uint64(), C.c_uint64()
        check(lib.pl_pipeline_stream_words(self.h, int(s), C.byref(lo), C.byref(hi)), "pl_pipeline_stream_words")
        return lo.value, hi.value

    def push_stream(self, s, words, nonblocking=False):
        """Append the next words (uint32 array) of stream s; raises PlError(PL_EAGAIN) if the
        ring is full and nonblocking."""
        a = np.ascontiguousarray(words, dtype=np.uint32)
        check(lib.pl_pipeline_push_stream(self.h, int(s), a.ctypes.data, a.shape[0], int(bool(nonblocking))),
              "pl_pipeline_push_stream")

    def push_all(self, slices, nonblocking=False):
        """Append slices[s] (uint32 arrays, possibly empty) to every stream s in one call."""
        arrs = [np.ascontiguousarray(x, dtype=np.uint32) for x in slices]
        ptrs = (C.c_void_p * len(arrs))(*[a.ctypes.data if a.size else None for a in arrs])
        ns = (C.c_uint64 * len(arrs))(*[a.shape[0] for a in arrs])
        check(lib.pl_pipeline_push_all(self.h, ptrs, ns, int(bool(nonblocking))), "pl_pipeline_push_all")

    def inject_stalls(self, period_ns, len_ns):
        """pl_pipeline_inject_stalls: every node stops over [T0 + j period, T0 + j period + len)
        of later physical runs (the platform's ~1.6 ms SM stalls, on demand); len_ns=0: off."""
        check(lib.pl_pipeline_inject_stalls(self.h, int(period_ns), int(len_ns)), "pl_pipeline_inject_stalls")

    def launch(self):
        check(lib.pl_pipeline_launch(self.h), "pl_pipeline_launch")

    def step(self):
        """Pipelined run (pl_pipeline_step): launch the next run, return the PREVIOUS step's
        summary (None on the first call) while the new run executes."""
        s, has = _pl.pl_summary(), C.c_int()
        check(lib.pl_pipeline_step(self.h, C.byref(s), C.byref(has)), "pl_pipeline_step")
        return {k: getattr(s, k) for k, _ in s._fields_} if has.value else None

    def step_finish(self):
        """Summary of the last pl_pipeline_step run (None if none is outstanding)."""
        s, has = _pl.pl_summary(), C.c_int()
        check(lib.pl_pipeline_step_finish(self.h, C.byref(s), C.byref(has)), "pl_pipeline_step_finish")
        return {k: getattr(s, k) for k, _ in s._fields_} if has.value else None

    def drain(self):
        check(lib.pl_pipeline_drain(self.h), "pl_pipeline_drain")

    def rewind(self):
        check(lib.pl_pipeline_rewind(self.h), "pl_pipeline_rewind")

    def close(self):
        if getattr(self, "h", None):
            lib.pl_pipeline_destroy(self.h)
            self.h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    # -- outputs
    def stats(self) -> dict:
        s = _pl.pl_stats()
        check(lib.pl_pipeline_stats(self.h, C.byref(s)), "pl_pipeline_stats")
        return s.as_dict()

    def results(self):
        n = C.c_uint64()
        check(lib.pl_pipeline_results(self.h, None, 0, C.byref(n)), "pl_pipeline_results")
        buf = (_pl.pl_match * max(1, n.value))()
        check(lib.pl_pipeline_results(self.h, buf, n.value, C.byref(n)), "pl_pipeline_results")
        return sorted((m.p, m.q, m.db_start, m.q_start, m.len, m.score) for m in buf[:n.value])

    def results_array(self):
        """The match records as an (n, 6) int64 array (p, q, db_start, q_start, len, score),
        rows in lexicographic order (the order of results())."""
        n = C.c_uint64()
        check(lib.pl_pipeline_results(self.h, None, 0, C.byref(n)), "pl_pipeline_results")
        buf = np.empty((max(1, n.value), 6), dtype=np.uint32)
        check(lib.pl_pipeline_results(self.h, buf.ctypes.data, n.value, C.byref(n)), "pl_pipeline_results")
        a = buf[:n.value].astype(np.int64)
        a[:, 5] = buf[:n.value, 5].view(np.int32)
        return a[np.lexsort(a.T[::-1])] if len(a) else a

    def results_raw(self):
        """The match records as an (n, 6) uint32 array in device order (unsorted; score is the
        int32 bit pattern) -- the cheap form for very large result sets."""
        n = C.c_uint64()
        check(lib.pl_pipeline_results(self.h, None, 0, C.byref(n)), "pl_pipeline_results")
        buf = np.empty((max(1, n.value), 6), dtype=np.uint32)
        check(lib.pl_pipeline_results(self.h, buf.ctypes.data, n.value, C.byref(n)), "pl_pipeline_results")
        return buf[:n.value]

    def latency(self):
        n = C.c_uint64()
        check(lib.pl_pipeline_latency(self.h, None, None, 0, C.byref(n)), "pl_pipeline_latency")
        lu = np.empty(n.value, dtype=np.int64)
        ln = np.empty(n.value, dtype=np.int64)
        check(lib.pl_pipeline_latency(self.h, lu.ctypes.data, ln.ctypes.data, n.value, C.byref(n)),
              "pl_pipeline_latency")
        return lu, ln

    def trace(self):
        n = C.c_uint64()
        check(lib.pl_pipeline_trace(self.h, None, 0, C.byref(n)), "pl_pipeline_trace")
        t = np.empty(n.value, dtype=np.uint32)
        check(lib.pl_pipeline_trace(self.h, t.ctypes.data, n.value, C.byref(n)), "pl_pipeline_trace")
        return t

    def firings(self):
        n = C.c_uint64()
        check(lib.pl_pipeline_firings(self.h, None, 0, C.byref(n)), "pl_pipeline_firings")
        buf = (_pl.pl_firing * max(1, n.value))()
        check(lib.pl_pipeline_firings(self.h, buf, n.value, C.byref(n)), "pl_pipeline_firings")
        return [(f.stream, f.node, f.start, f.n, f.first_root, f.last_root) for f in buf[:n.value]]

    def stage_batch(self, stage, in_ptr, n, first_root, out_ptr, cap):
        """pl_stage_batch: one stage over n device entries -> (outputs, longest vector cycles)."""
        n_out = C.c_uint64()
        cyc = C.c_uint64()
        check(lib.pl_stage_batch(self.h, int(stage), C.c_void_p(in_ptr or 0), int(n), int(first_root),
                                 C.c_void_p(out_ptr or 0), int(cap), C.byref(n_out), C.byref(cyc)),
              "pl_stage_batch")
        return n_out.value, cyc.value

    def params(self):
        w = (C.c_int64 * 8)()
        th = (C.c_uint32 * 8)()
        M = C.c_uint32()
        check(lib.pl_pipeline_params(self.h, w, th, C.byref(M)), "pl_pipeline_params")
        return list(w)[:self.N], list(th)[:self.N], M.value


def solve_enforced_waits(cfg):
    """pl_solve_enforced_waits -> (w list, theta list, T_int, T_cont)."""
    c, keep = make_config(cfg)
    N = len(cfg.stages)
    w = (C.c_int64 * N)()
    th = (C.c_uint32 * N)()
    T = C.c_double()
    Tc = C.c_double()
    check(lib.pl_solve_enforced_waits(C.byref(c), w, th, C.byref(T), C.byref(Tc)), "pl_solve_enforced_waits")
    return list(w), list(th), T.value, Tc.value


def solve_monolithic(cfg):
    """pl_solve_monolithic -> (M, objective)."""
    c, keep = make_config(cfg)
    M = C.c_uint32()
    T = C.c_double()
    check(lib.pl_solve_monolithic(C.byref(c), C.byref(M), C.byref(T)), "pl_solve_monolithic")
    return M.value, T.value
