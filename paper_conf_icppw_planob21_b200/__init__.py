"""paper_conf_icppw_planob21_b200 — B200-native enforced-waiting streaming-pipeline executor.

Plano & Buhler, "Enabling Real-Time Irregular Data-Flow Pipelines on SIMD Devices"
(SRMPDS '21).  The hot path lives in the C-ABI library ``libplgpu.so``
(csrc/: persistent sm_100a kernels + host runtime + solvers, include/pl.h); this
package is its thin Python binding plus the torch.distributed counter reduction
used for multi-GPU runs.  Importing it fails loudly if the library is missing.
"""
from ._pl import PlError, lib, LIB_PATH  # noqa: F401
from .pipeline import Pipeline, make_config, solve_enforced_waits, solve_monolithic  # noqa: F401
