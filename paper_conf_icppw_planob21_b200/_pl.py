"""ctypes binding of include/pl.h — argument marshalling only.

Every step of the hot path runs in libplgpu.so (csrc/).  If the library cannot
be loaded this module raises; there is no CPU fallback.
"""
from __future__ import annotations

import ctypes as C
import os

HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("PLGPU_LIB") or os.path.join(HERE, "libplgpu.so")   # PLGPU_LIB: an experiment build

PL_MAX_STAGES = 8
PL_MAX_U = 16
PL_OK, PL_EINVAL, PL_ENOMEM, PL_EDEVICE, PL_EINFEASIBLE, PL_ESTATE, PL_EAGAIN, PL_EOVERFLOW = 0, -1, -2, -3, -4, -5, -6, -7
PL_REC_LATENCY, PL_REC_TRACE, PL_REC_FIRINGS, PL_FIXED_SERVICE, PL_EAGER_DRAIN = 1, 2, 4, 8, 16
PL_CLUSTER_NODES = 32
STATUS_NAMES = {0: "PL_OK", -1: "PL_EINVAL", -2: "PL_ENOMEM", -3: "PL_EDEVICE", -4: "PL_EINFEASIBLE",
                -5: "PL_ESTATE", -6: "PL_EAGAIN", -7: "PL_EOVERFLOW"}


class pl_stage(C.Structure):
    _fields_ = [("kind", C.c_uint32), ("max_out", C.c_uint32), ("param", C.c_double),
                ("iparam", C.c_int32 * 4)]


class pl_config(C.Structure):
    _fields_ = [("n_stages", C.c_uint32), ("stages", C.POINTER(pl_stage)),
                ("service_time", C.POINTER(C.c_int64)), ("gain", C.POINTER(C.c_double)),
                ("b", C.POINTER(C.c_uint32)), ("vector_width", C.c_uint32),
                ("wait_time", C.POINTER(C.c_int64)), ("wait_threshold", C.POINTER(C.c_uint32)),
                ("deadline", C.c_int64), ("interarrival", C.c_int64), ("slack_guard", C.c_int64),
                ("policy", C.c_uint32), ("clock", C.c_uint32), ("block_size", C.c_uint32),
                ("mono_b", C.c_uint32), ("mono_S", C.c_double), ("n_streams", C.c_uint32),
                ("n_roots", C.c_uint64), ("seed", C.c_uint64), ("device", C.c_int32),
                ("ns_per_unit", C.c_double), ("flags", C.c_uint32), ("queue_capacity", C.c_uint32),
                ("spill_capacity", C.c_uint32), ("firing_log_capacity", C.c_uint32),
                ("match_capacity", C.c_uint64), ("arrivals", C.POINTER(C.c_int64)), ("n_arrivals", C.c_uint64),
                ("window_words", C.c_uint32), ("window_chunk_words", C.c_uint32)]


class pl_workload(C.Structure):
    _fields_ = [("query", C.POINTER(C.c_uint32)), ("q_len", C.c_uint64), ("db_len", C.c_uint64)]


class pl_match(C.Structure):
    _fields_ = [("p", C.c_uint32), ("q", C.c_uint32), ("db_start", C.c_uint32), ("q_start", C.c_uint32),
                ("len", C.c_uint32), ("score", C.c_int32)]


class pl_firing(C.Structure):
    _fields_ = [("start", C.c_int64), ("node", C.c_uint32), ("n", C.c_uint32),
                ("first_root", C.c_uint32), ("last_root", C.c_uint32), ("stream", C.c_uint32),
                ("pad", C.c_uint32)]


class pl_summary(C.Structure):
    _fields_ = [("roots", C.c_uint64), ("matches", C.c_uint64), ("miss_events", C.c_uint64),
                ("miss_events_ns", C.c_uint64), ("max_latency", C.c_int64), ("max_latency_ns", C.c_int64), ("errors", C.c_uint32),
                ("launches", C.c_uint32), ("latency_outliers", C.c_uint64)]


_A8 = C.c_uint64 * PL_MAX_STAGES
_I8 = C.c_int64 * PL_MAX_STAGES


class pl_stats(C.Structure):
    _fields_ = [("n_stages", C.c_uint32), ("n_streams", C.c_uint32), ("roots", C.c_uint64),
                ("firings", _A8), ("empty_firings", _A8), ("consumed", _A8), ("produced", _A8),
                ("active_window", _I8), ("busy_ns", _I8), ("spilled", _A8), ("overruns", _A8), ("stalls", _A8),
                ("max_queue", C.c_uint32 * PL_MAX_STAGES),
                ("max_lateness_ns", _I8), ("sched_cycles", _A8), ("max_fire_ns", _I8), ("max_loop_ns", _I8),
                ("phase_cycles", (C.c_uint64 * 6) * PL_MAX_STAGES), ("matches", C.c_uint64),
                ("miss_events", C.c_uint64), ("miss_events_ns", C.c_uint64), ("misses", C.c_uint64),
                ("max_latency", C.c_int64),
                ("max_latency_ns", C.c_int64), ("window", C.c_int64), ("t_end", C.c_int64),
                ("active_fraction", C.c_double), ("active_fraction_nonempty", C.c_double),
                ("active_fraction_drain", C.c_double),
                ("hw_busy_fraction", C.c_double), ("wall_ns", C.c_int64), ("errors", C.c_uint32),
                ("launches", C.c_uint32), ("h2d_bytes", C.c_uint64), ("d2h_bytes", C.c_uint64),
                ("window_refills", C.c_uint64), ("latency_outliers", C.c_uint64),
                ("latency_rel_err_max", C.c_double), ("ingest_waits", C.c_uint64),
                ("max_ingest_wait_ns", C.c_int64)]

    def as_dict(self):
        N = self.n_stages
        out = {}
        for name, _ in self._fields_:
            val = getattr(self, name)
            if name == "phase_cycles":
                out[name] = [list(val[i]) for i in range(N)]
            else:
                out[name] = list(val)[:N] if hasattr(val, "__len__") else val
        return out


def _load():
    if not os.path.exists(LIB_PATH):
        raise ImportError(f"{LIB_PATH} not built — run `python paper_conf_icppw_planob21_b200/build.py` "
                          "(there is no CPU fallback)")
    lib = C.CDLL(LIB_PATH)
    P = C.c_void_p
    sig = {
        "pl_pipeline_create": (C.c_int32, [C.POINTER(pl_config), C.POINTER(pl_workload), C.POINTER(P)]),
        "pl_pipeline_set_stream": (C.c_int32, [P, P]),
        "pl_pipeline_push": (C.c_int32, [P, P, C.c_uint64]),
        "pl_pipeline_bind_device": (C.c_int32, [P, P, C.c_uint64]),
        "pl_pipeline_bind_host": (C.c_int32, [P, P, C.c_uint64]),
        "pl_pipeline_summary": (C.c_int32, [P, C.POINTER(pl_summary)]),
        "pl_pipeline_step": (C.c_int32, [P, C.POINTER(pl_summary), C.POINTER(C.c_int)]),
        "pl_pipeline_step_finish": (C.c_int32, [P, C.POINTER(pl_summary), C.POINTER(C.c_int)]),
        "pl_pipeline_queue_peaks": (C.c_int32, [P, P, C.c_uint64, C.POINTER(C.c_uint64)]),
        "pl_pipeline_bind_results": (C.c_int32, [P, P, C.c_uint64]),
        "pl_pipeline_launch": (C.c_int32, [P]),
        "pl_pipeline_inject_stalls": (C.c_int32, [P, C.c_int64, C.c_int64]),
        "pl_pipeline_live_start": (C.c_int32, [P, C.c_uint32]),
        "pl_pipeline_stream_words": (C.c_int32, [P, C.c_uint32, C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
        "pl_pipeline_push_stream": (C.c_int32, [P, C.c_uint32, P, C.c_uint64, C.c_int]),
        "pl_pipeline_push_all": (C.c_int32, [P, P, P, C.c_int]),
        "pl_pipeline_drain": (C.c_int32, [P]),
        "pl_pipeline_rewind": (C.c_int32, [P]),
        "pl_pipeline_stats": (C.c_int32, [P, C.POINTER(pl_stats)]),
        "pl_pipeline_results": (C.c_int32, [P, P, C.c_uint64, C.POINTER(C.c_uint64)]),
        "pl_pipeline_latency": (C.c_int32, [P, P, P, C.c_uint64, C.POINTER(C.c_uint64)]),
        "pl_pipeline_trace": (C.c_int32, [P, P, C.c_uint64, C.POINTER(C.c_uint64)]),
        "pl_pipeline_firings": (C.c_int32, [P, P, C.c_uint64, C.POINTER(C.c_uint64)]),
        "pl_pipeline_params": (C.c_int32, [P, P, P, P]),
        "pl_pipeline_destroy": (None, [P]),
        "pl_last_error": (C.c_char_p, []),
        "pl_version": (C.c_char_p, []),
        "pl_solve_enforced_waits": (C.c_int32, [C.POINTER(pl_config), P, P, P, P]),
        "pl_solve_monolithic": (C.c_int32, [C.POINTER(pl_config), P, P]),
        "pl_stage_batch": (C.c_int32, [P, C.c_uint32, P, C.c_uint64, C.c_uint64, P, C.c_uint64,
                                       C.POINTER(C.c_uint64), C.POINTER(C.c_uint64)]),
    }
    for name, (res, args) in sig.items():
        fn = getattr(lib, name, None)
        if fn is None and os.environ.get("PLGPU_LIB"):   # an older experiment build (tools/): skip
            continue
        if fn is None:
            raise ImportError(f"{LIB_PATH} lacks {name}: rebuild it")
        fn.restype = res
        fn.argtypes = args
    return lib


lib = _load()
EXPORTED = ("pl_pipeline_create", "pl_pipeline_set_stream", "pl_pipeline_push", "pl_pipeline_bind_device",
            "pl_pipeline_launch", "pl_pipeline_drain", "pl_pipeline_rewind", "pl_pipeline_stats",
            "pl_pipeline_results", "pl_pipeline_latency", "pl_pipeline_trace", "pl_pipeline_firings",
            "pl_pipeline_params", "pl_pipeline_destroy", "pl_last_error", "pl_solve_enforced_waits",
            "pl_solve_monolithic", "pl_version", "pl_stage_batch", "pl_pipeline_bind_host",
            "pl_pipeline_summary", "pl_pipeline_queue_peaks",
            "pl_pipeline_step", "pl_pipeline_step_finish", "pl_pipeline_bind_results",
            "pl_pipeline_inject_stalls", "pl_pipeline_live_start", "pl_pipeline_stream_words",
            "pl_pipeline_push_stream", "pl_pipeline_push_all")


class PlError(RuntimeError):
    def __init__(self, status, where):
        self.status = status
        msg = lib.pl_last_error().decode(errors="replace")
        super().__init__(f"{where}: {STATUS_NAMES.get(status, status)}: {msg}")


def check(status, where):
    if status != PL_OK:
        raise PlError(status, where)
