"""Named configurations (BASELINE.json ``configs``) as plain data.

These are *inputs* — pipeline parameters and workload recipes — consumed by
both the CUDA path (marshalled into ``pl_config``, include/pl.h) and the
oracle.  No arithmetic of the method lives here.

Units: one logical time unit ("cycle" in PAPER.md L208/L212).  In the physical
(%globaltimer) clock mode one unit is ``ns_per_unit`` nanoseconds.
"""
from __future__ import annotations

import dataclasses
from typing import List, Optional

# stage kinds (include/pl.h enum pl_stage_kind)
BERNOULLI, FIXED_GAIN, POISSON_CAPPED, SEED_LOOKUP, HIT_ENUM, UNGAPPED_WINDOW, UNGAPPED_XDROP, KEEP_EVERY = range(8)
# policies (enum pl_policy)
FIXED_WAIT, THRESHOLD_SLACK, MONOLITHIC = range(3)
# clocks (enum pl_clock)
CLOCK_LOGICAL, CLOCK_GLOBALTIMER = range(2)

DNA_KINDS = (SEED_LOOKUP, HIT_ENUM, UNGAPPED_WINDOW, UNGAPPED_XDROP)

# PAPER.md Table 1 (L218–L225), v = 128, u = 16 (L208); b from L230.
TABLE1_T = (287, 955, 402, 2753)
TABLE1_G = (0.379, 1.920, 0.0332)
TABLE1_V = 128
TABLE1_U = 16
PAPER_B = (1, 3, 9, 6)


@dataclasses.dataclass
class Stage:
    kind: int
    param: float = 0.0          # g (Bernoulli), c (fixed gain), lambda (Poisson), modulus (KEEP_EVERY)
    max_out: int = 1            # u: cap on outputs per input
    iparam: tuple = (0, 0, 0, 0)  # DNA: (k, W, T2, 0) window / (k, X, T3, 0) x-drop / (k, u, 0, 0)


@dataclasses.dataclass
class Config:
    name: str
    stages: List[Stage]
    service_time: tuple          # t_i
    vector_width: int            # v
    deadline: int                # D
    interarrival: int            # tau0
    b: tuple                     # b_i (queue multipliers, L133)
    gain: Optional[tuple] = None  # g_i for the solver (N-1 values)
    wait_time: Optional[tuple] = None       # w_i
    wait_threshold: Optional[tuple] = None  # theta_i
    policy: int = FIXED_WAIT
    clock: int = CLOCK_LOGICAL
    block_size: int = 0          # M (monolithic)
    mono_b: int = 1
    mono_S: float = 1.0
    n_streams: int = 1
    n_roots: int = 0             # gain model: roots per stream; DNA: derived from db_len
    seed: int = 0
    ns_per_unit: float = 1.0
    slack_guard: int = 0         # THRESHOLD_SLACK: extra reserve added to R_i (physical lateness guard)
    eager_drain: bool = False    # R-DRAIN: work-conserving firing once the stream's last root has arrived
    # DNA workload recipe (plgen.dna.make_dna kwargs); None for gain-model pipelines
    dna: Optional[dict] = None

    @property
    def n_stages(self) -> int:
        return len(self.stages)

    def replace(self, **kw) -> "Config":
        return dataclasses.replace(self, **kw)


def dna_stages(k: int = 6, u: int = TABLE1_U, W: int = 8, T2: Optional[int] = None,
               X: int = 20, T3: int = 30) -> List[Stage]:
    """k=6, W=8, T2=k+3, X=20, T3=30, u=16, +1/-3."""
    if T2 is None:
        T2 = k + 3
    return [Stage(SEED_LOOKUP, 0.0, 1, (k, 0, 0, 0)),
            Stage(HIT_ENUM, 0.0, u, (k, u, 0, 0)),
            Stage(UNGAPPED_WINDOW, 0.0, 1, (k, W, T2, 0)),
            Stage(UNGAPPED_XDROP, 0.0, 1, (k, X, T3, 0))]


def c1(**kw) -> Config:
    """BASELINE.json configs[0]: 2-stage, Bernoulli 0.5 then fixed gain 2, 1e5 items, v=32.
    Builder timing: t=(64,96), tau0=4, b=(1,2), D=500."""
    cfg = Config(name="c1", stages=[Stage(BERNOULLI, 0.5, 1), Stage(FIXED_GAIN, 2.0, 2)],
                 service_time=(64, 96), vector_width=32, deadline=500, interarrival=4,
                 b=(1, 2), gain=(0.5,), n_roots=100_000, seed=1)
    return cfg.replace(**kw)


def c1r(**kw) -> Config:
    """Regular variant of c1: S0 keeps every 2nd root."""
    cfg = c1(name="c1r", stages=[Stage(KEEP_EVERY, 2.0, 1), Stage(FIXED_GAIN, 2.0, 2)])
    return cfg.replace(**kw)


def gain_model_blast(**kw) -> Config:
    """The paper-faithful random-gain BLAST model (Table 1):
    nodes 0,2,3 Bernoulli(g_i), node 1 min(Poisson(1.92), 16).  g_3 is N/A in
    the paper (L225); node 3 is the sink and passes its input through."""
    st = [Stage(BERNOULLI, TABLE1_G[0], 1), Stage(POISSON_CAPPED, TABLE1_G[1], TABLE1_U),
          Stage(BERNOULLI, TABLE1_G[2], 1), Stage(BERNOULLI, 1.0, 1)]
    cfg = Config(name="gm", stages=st, service_time=TABLE1_T, vector_width=TABLE1_V,
                 deadline=50_000, interarrival=10, b=PAPER_B, gain=TABLE1_G,
                 n_roots=50_000, seed=0)
    return cfg.replace(**kw)


def c2(**kw) -> Config:
    """BASELINE.json configs[1]: BLAST-style 4-stage pipeline, 1 Mbp DB, 1 kbp query,
    64 planted matches, 1 B200.  Logical timing = Table 1, v=128, b=(1,3,9,6)."""
    cfg = Config(name="c2", stages=dna_stages(), service_time=TABLE1_T, vector_width=TABLE1_V,
                 deadline=50_000, interarrival=10, b=PAPER_B, gain=None, seed=2,
                 dna=dict(db_len=1 << 20, q_len=1024, n_planted=64))
    return cfg.replace(**kw)


def c4(**kw) -> Config:
    """BASELINE.json configs[3]: 100 Mbp DB with heavy-tailed hit amplification,
    one stream per CTA across all SMs."""
    cfg = c2(name="c4", n_streams=148, seed=4,
             dna=dict(db_len=100 << 20, q_len=1024, n_planted=6400, heavy_tailed=True))
    return cfg.replace(**kw)


def sweep_grid():
    """c3 grid: tau0 x D."""
    taus = (3, 5, 10, 20, 50, 100)
    Ds = (20_000, 25_000, 50_000, 100_000, 200_000, 350_000)
    return [(t, d) for t in taus for d in Ds]
