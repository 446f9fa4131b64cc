"""Per-item stage semantics, written out plainly (ORACLE — test infrastructure).

PAPER.md gives only gains and service times for the BLAST pipeline (§6.1
L204–L225).  The per-item semantics below are the builder's reading of classic
BLAST [1] (ref [1] L269) recorded in SURVEY.md §8(c) C-S and
DESIGN.md "Readings" R-S0..R-S3; the random-gain stages follow PAPER.md L210.

An entry is a tuple ``(root, lin, q)``:
  root — global root id (DNA: the DB position p of the seed; gain model: the item index)
  lin  — lineage (DNA: hit index j from S1; gain model: mixed-radix child path)
  q    — DNA query position of the hit (None before S1 / in the gain model)

Each stage function maps one entry to the list of its children, in child order.
"""
from __future__ import annotations

MASK64 = (1 << 64) - 1

# ---------------------------------------------------------------- sequences


def base(words, j: int) -> int:
    """Base j of a 2-bit packed sequence: bits 2*(j mod 16) of word j//16."""
    return (int(words[j >> 4]) >> (2 * (j & 15))) & 3


def unpack_list(words, n: int) -> list:
    return [base(words, j) for j in range(n)]


def unpack_bytes(words, n: int) -> bytes:
    """The same codes as unpack_list, one byte per base (bytes index like a list of ints);
    decoded with numpy shifts so that a 100 Mbp DB unpacks in about a second.  Pinned against
    base() by tests/test_oracle_stages.py::test_unpack_bytes_matches_base."""
    import numpy as np
    w = np.asarray(words, dtype=np.uint32)
    shifts = (2 * np.arange(16, dtype=np.uint32))[None, :]
    return ((w[:, None] >> shifts) & 3).astype(np.uint8).reshape(-1)[:n].tobytes()


def key(seq: list, p: int, k: int) -> int:
    """key(s, p) = sum_{j<k} s[p+j] * 4^(k-1-j)  (first base most significant; C-S)."""
    v = 0
    for j in range(k):
        v = v * 4 + seq[p + j]
    return v


def query_index(query: list, k: int) -> dict:
    """All query positions q in [0, Lq-k] grouped by key, ascending (C-S S1)."""
    idx = {}
    for q in range(len(query) - k + 1):
        idx.setdefault(key(query, q, k), []).append(q)
    return idx


class DnaContext:
    """The DB and query as plain lists of base codes plus the query index."""

    def __init__(self, db_words, db_len, q_words, q_len, k):
        self.db = unpack_bytes(db_words, db_len)
        self.query = unpack_list(q_words, q_len)
        self.k = k
        self.index = query_index(self.query, k)

    @property
    def n_roots(self) -> int:
        return len(self.db) - self.k + 1


def sigma(a: int, b: int) -> int:
    """+1 match / -3 mismatch (DESIGN.md R-S2)."""
    return 1 if a == b else -3


def s0_seed_lookup(ctx: DnaContext, e):
    """S0: keep p iff the k-mer db[p..p+k) occurs in the query (R-S0)."""
    root, lin, q = e
    return [e] if key(ctx.db, root, ctx.k) in ctx.index else []


def s1_hit_enum(ctx: DnaContext, e, u: int):
    """S1: p -> (p, q_j, j) for the first min(c, u) query occurrences, ascending q (R-S1)."""
    root, lin, q = e
    occ = ctx.index.get(key(ctx.db, root, ctx.k), [])
    return [(root, j, occ[j]) for j in range(min(len(occ), u))]


def _best_right(ctx, p, q, limit, X=None):
    """Walk d = 1, 2, ... to the right of the seed (db[p+k-1+d] vs query[q+k-1+d]).

    limit: max d (W) or None; X: x-drop or None.  Returns (best, d_best) where
    best = max(0, max_d R(d)) and d_best the smallest d attaining it (0 if best is 0).
    """
    k = ctx.k
    score = best = 0
    dbest = 0
    d = 1
    while True:
        if limit is not None and d > limit:
            break
        i, j = p + k - 1 + d, q + k - 1 + d
        if i >= len(ctx.db) or j >= len(ctx.query):
            break
        score += sigma(ctx.db[i], ctx.query[j])
        if score > best:
            best, dbest = score, d
        if X is not None and score <= best - X:
            break
        d += 1
    return best, dbest


def _best_left(ctx, p, q, limit, X=None):
    """Mirror of _best_right: db[p-d] vs query[q-d]."""
    score = best = 0
    dbest = 0
    d = 1
    while True:
        if limit is not None and d > limit:
            break
        i, j = p - d, q - d
        if i < 0 or j < 0:
            break
        score += sigma(ctx.db[i], ctx.query[j])
        if score > best:
            best, dbest = score, d
        if X is not None and score <= best - X:
            break
        d += 1
    return best, dbest


def s2_window(ctx: DnaContext, e, W: int, T2: int):
    """S2: keep (p, q) iff k + best_left(W) + best_right(W) >= T2 (R-S2)."""
    root, lin, q = e
    bl, _ = _best_left(ctx, root, q, W)
    br, _ = _best_right(ctx, root, q, W)
    return [e] if ctx.k + bl + br >= T2 else []


def s3_xdrop(ctx: DnaContext, e, X: int, T3: int):
    """S3: ungapped X-drop extension both ways; emit an HSP record if score >= T3 (R-S3).

    Returns [(p, q, db_start, q_start, length, score)] or [].
    """
    root, lin, q = e
    bl, dl = _best_left(ctx, root, q, None, X)
    br, dr = _best_right(ctx, root, q, None, X)
    score = ctx.k + bl + br
    if score < T3:
        return []
    return [(root, q, root - dl, q - dl, ctx.k + dl + dr, score)]


# ---------------------------------------------------------- random-gain model

SM_GAMMA = 0x9E3779B97F4A7C15
SM_M1 = 0xBF58476D1CE4E5B9
SM_M2 = 0x94D049BB133111EB


def splitmix64(x: int) -> int:
    """SplitMix64 finaliser (Steele, Lea & Flood 2014), the counter-based generator (R-RNG)."""
    z = (x + SM_GAMMA) & MASK64
    z = ((z ^ (z >> 30)) * SM_M1) & MASK64
    z = ((z ^ (z >> 27)) * SM_M2) & MASK64
    return z ^ (z >> 31)


def gain_hash(seed: int, stage: int, root: int, lin: int) -> int:
    """h = splitmix64(seed ^ stage*GAMMA ^ root*M1 ^ lin)  (mod 2^64; R-RNG)."""
    x = seed ^ ((stage * SM_GAMMA) & MASK64) ^ ((root * SM_M1) & MASK64) ^ lin
    return splitmix64(x & MASK64)


def g_bernoulli(seed, stage, e, thr: int):
    """One output with probability g (h < floor(g 2^64)), else none."""
    root, lin, q = e
    return [e] if gain_hash(seed, stage, root, lin) < thr else []


def g_fixed(e, c: int):
    """Exactly c outputs, lineage lin*c + j (deterministic gain; c1's second stage)."""
    root, lin, q = e
    return [(root, lin * c + j, None) for j in range(c)]


def g_poisson_capped(seed, stage, e, thr: list, u: int):
    """min(Poisson(lambda), u) outputs by inversion: count = #{k<u : h >= thr_k} (L210, A15).
    Children get lineage lin*u + j."""
    root, lin, q = e
    h = gain_hash(seed, stage, root, lin)
    cnt = sum(1 for k in range(u) if h >= thr[k])
    return [(root, lin * u + j, None) for j in range(cnt)]


def g_keep_every(e, m: int):
    """Deterministic filter: keep iff root mod m == 0 (regular pipeline c1r, pin P3)."""
    root, lin, q = e
    return [e] if root % m == 0 else []
