"""Synthetic DNA workloads (seeded), 2-bit packed.

Layout (both sides read it):
  base j of a sequence sits at bits 2*(j mod 16) of little-endian uint32 word
  j // 16, with A=0, C=1, G=2, T=3 (SURVEY.md §8(c) C-S "Encoding").

Recipes:
  * c2 / c3: DB of ``db_len`` iid uniform bases, query of ``q_len`` iid
    uniform bases, ``n_planted`` planted segments: each a random query
    substring of length U[min_len, max_len] with ``subst`` iid substitutions
    (each substituted base replaced by a different base, uniformly), written at
    non-overlapping uniformly drawn DB offsets.
  * c4 / c5: ``heavy_tailed=True`` additionally puts ``n_motif_blocks`` tandem
    repeat blocks of random 6-mer motifs (``motif_copies`` copies each) into
    the query, and repeat islands drawn from those motifs into the DB with
    Pareto(alpha) lengths clipped to [island_min, island_max], one island per
    ``island_every`` bases on average.  Hits inside islands amplify to the cap u.

Nothing here implements the method: this is the paper's workload *shape*
(§6.1: human genome vs a microbial query) made synthetic.
"""
from __future__ import annotations

import dataclasses
import numpy as np


@dataclasses.dataclass
class DnaWorkload:
    db: np.ndarray          # uint32 packed words, len = ceil(db_len/16)
    db_len: int
    query: np.ndarray       # uint32 packed words
    q_len: int
    planted: list           # [(db_off, q_off, length)]
    seed: int

    def db_bases(self) -> np.ndarray:
        return unpack(self.db, self.db_len)

    def query_bases(self) -> np.ndarray:
        return unpack(self.query, self.q_len)


def pack(bases: np.ndarray) -> np.ndarray:
    """Pack a uint8 array of 2-bit codes into little-endian uint32 words."""
    b = np.asarray(bases, dtype=np.uint32)
    n = b.shape[0]
    nw = (n + 15) // 16
    pad = np.zeros(nw * 16, dtype=np.uint32)
    pad[:n] = b
    pad = pad.reshape(nw, 16)
    shifts = (2 * np.arange(16, dtype=np.uint32))[None, :]
    return np.bitwise_or.reduce(pad << shifts, axis=1).astype(np.uint32)


def unpack(words: np.ndarray, n: int) -> np.ndarray:
    w = np.asarray(words, dtype=np.uint32)
    shifts = (2 * np.arange(16, dtype=np.uint32))[None, :]
    return ((w[:, None] >> shifts) & 3).reshape(-1)[:n].astype(np.uint8)


def _substitute(rng, seg: np.ndarray, rate: float) -> np.ndarray:
    seg = seg.copy()
    m = rng.random(seg.shape[0]) < rate
    k = int(m.sum())
    if k:
        seg[m] = (seg[m] + rng.integers(1, 4, size=k)) % 4
    return seg


def make_dna(seed: int, db_len: int = 1 << 20, q_len: int = 1024, n_planted: int = 64,
             min_len: int = 64, max_len: int = 256, subst: float = 0.05,
             heavy_tailed: bool = False, n_motif_blocks: int = 8, motif_copies: int = 20,
             island_every: int = 1 << 16, pareto_alpha: float = 1.5,
             island_min: int = 200, island_max: int = 20000) -> DnaWorkload:
    rng = np.random.default_rng(np.random.PCG64(seed))
    db = rng.integers(0, 4, size=db_len, dtype=np.uint8)
    query = rng.integers(0, 4, size=q_len, dtype=np.uint8)
    motifs = []
    if heavy_tailed:
        # tandem-repeat blocks in the query, evenly spread with random spacers
        blk = 6 * motif_copies
        free = q_len - n_motif_blocks * blk
        assert free >= 0, "query too short for the motif blocks"
        gaps = rng.multinomial(free, [1.0 / (n_motif_blocks + 1)] * (n_motif_blocks + 1))
        pos = int(gaps[0])
        for b in range(n_motif_blocks):
            motif = rng.integers(0, 4, size=6, dtype=np.uint8)
            motifs.append(motif)
            query[pos:pos + blk] = np.tile(motif, motif_copies)
            pos += blk + int(gaps[b + 1])
    # planted segments at non-overlapping DB offsets (rejection on overlap)
    planted = []
    occupied = []
    tries = 0
    while len(planted) < n_planted and tries < 100 * max(1, n_planted):
        tries += 1
        length = int(rng.integers(min_len, max_len + 1))
        if length > q_len or length > db_len:
            continue
        q_off = int(rng.integers(0, q_len - length + 1))
        d_off = int(rng.integers(0, db_len - length + 1))
        if any(not (d_off + length <= a or b <= d_off) for a, b in occupied):
            continue
        occupied.append((d_off, d_off + length))
        db[d_off:d_off + length] = _substitute(rng, query[q_off:q_off + length], subst)
        planted.append((d_off, q_off, length))
    if heavy_tailed and motifs:
        n_isl = max(1, db_len // island_every)
        for _ in range(n_isl):
            # Pareto(alpha) with scale island_min, clipped to island_max
            length = int(min(island_max, island_min * (1.0 + rng.pareto(pareto_alpha))))
            length = min(length, db_len)
            off = int(rng.integers(0, db_len - length + 1))
            motif = motifs[int(rng.integers(0, len(motifs)))]
            reps = (length + 5) // 6
            db[off:off + length] = np.tile(motif, reps)[:length]
    planted.sort()
    return DnaWorkload(db=pack(db), db_len=db_len, query=pack(query), q_len=q_len,
                       planted=planted, seed=seed)


def stream_bounds(n_roots: int, n_streams: int) -> list:
    """Contiguous root ranges, stream s = [s*R//S, (s+1)*R//S)."""
    return [((s * n_roots) // n_streams, ((s + 1) * n_roots) // n_streams) for s in range(n_streams)]
