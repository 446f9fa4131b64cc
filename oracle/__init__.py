"""ORACLE — test infrastructure only.

A plain, slow, obviously-correct CPU implementation of what the hot path
computes, written from PAPER.md (Plano & Buhler, SRMPDS '21) and the readings
listed in DESIGN.md.  Only ``tests/``, ``__graft_entry__.smoke()`` and
``bench.py``'s ``cpu_baseline`` / ``--impl reference`` legs may import it.  It
shares no code with the CUDA path (``paper_conf_icppw_planob21_b200``); the
only common module is ``plgen`` (seeded input generators, no method arithmetic).

Modules:
  stages  — per-item stage semantics (BLAST [1] via PAPER.md L204)
  des     — discrete-event simulation of the execution model (§2,
            §4, §5 L157/L184)
  solver  — the optimisation problems of Fig. 1 (L139–L151) and Fig. 2 (L165–L180)
            by their definitions (integer brute force, exhaustive M) plus scipy
            SLSQP for the continuous Fig. 1 optimum
  run     — CLI / timing harness of the DES over a bounded sample of a configuration's
            streams (`python -m oracle.run --config c4 ...`), used by bench.py's cpu_baseline
            and --impl reference legs

Parity status per function is listed in DESIGN.md "Oracle pins".  Functions
without an independent pin say "parity unpinned" in their docstring.
"""
