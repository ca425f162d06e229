"""Seeded synthetic workload generator (shared by the oracle and the CUDA path).

Holds NONE of the method's arithmetic: no scoring, no DP, no packing.  It only
produces sequence sets in the paper's indexed format (PAPER.md P20 §IV.B: "the total
number of sequences, the size of the biggest sequence and the offset that marks the
beginning of each sequence") plus the scoring inputs (a substitution matrix is an
input to the method, like the sequences).

Randomness is a counter-based splitmix64, evaluated vectorised with numpy uint64
arithmetic, so every draw is a pure function of (seed, stream, counter).

Recipe:
  * alphabet: the 20 standard amino acids (P12 §II: "20 amino acids") drawn with
    UniProtKB/Swiss-Prot composition (external constants, reading R14);
  * DB lengths: log-normal body with the configured mean/median, clipped to
    [10, 35,213], plus a 0.2 % heavy tail log-uniform in [3,000, 35,213]; the body
    location is solved so the overall mean hits the target (reading R14);
  * queries: 40 with "equally distributed sizes, ranging from 100 amino acids to
    approximately 5,000" (P20 §V), L_k = round(100 + k (L_max-100)/39) with L_max from
    Table II (P20) (reading R15), "chosen ... from each genomic database" (P20):
    written over 40 seeded DB slots (reading R16);
  * each query gets 5 planted homologs at 90/70/50/40/30 % identity with 2 % indels.
"""
from __future__ import annotations

import math
from dataclasses import dataclass, field

import numpy as np

AMINO = "ARNDCQEGHILKMFPSTWYV"
# UniProtKB/Swiss-Prot amino-acid composition in percent (external).
COMPOSITION = {
    "A": 8.25, "R": 5.53, "N": 4.06, "D": 5.46, "C": 1.38, "Q": 3.93, "E": 6.72,
    "G": 7.07, "H": 2.27, "I": 5.91, "L": 9.65, "K": 5.80, "M": 2.41, "F": 3.86,
    "P": 4.74, "S": 6.64, "T": 5.35, "W": 1.10, "Y": 2.92, "V": 6.86,
}
MAX_DB_LEN = 35213
MIN_DB_LEN = 10

_M64 = np.uint64(0xFFFFFFFFFFFFFFFF)
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_C1 = np.uint64(0xBF58476D1CE4E5B9)
_C2 = np.uint64(0x94D049BB133111EB)


def splitmix64(seed: int, counter) -> np.ndarray:
    """splitmix64 output for state seed + (counter+1)*golden (vectorised, wraps mod 2^64)."""
    c = np.asarray(counter, dtype=np.uint64)
    with np.errstate(over="ignore"):
        z = np.uint64(seed & 0xFFFFFFFFFFFFFFFF) + (c + np.uint64(1)) * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _C1
        z = (z ^ (z >> np.uint64(27))) * _C2
        z = z ^ (z >> np.uint64(31))
    return z


def stream_seed(seed: int, tag: str) -> int:
    """Derive an independent stream seed from (seed, tag)."""
    h = 1469598103934665603
    for ch in tag.encode():
        h = ((h ^ ch) * 1099511628211) & 0xFFFFFFFFFFFFFFFF
    return int(splitmix64(seed ^ h, 0))


def uniform01(seed: int, counter) -> np.ndarray:
    """53-bit uniform in (0, 1)."""
    u = splitmix64(seed, counter) >> np.uint64(11)
    return (u.astype(np.float64) + 0.5) * (1.0 / 9007199254740992.0)


def randint(seed: int, counter, hi: int) -> np.ndarray:
    """Uniform integers in [0, hi) (multiply-shift on the top 32 bits)."""
    u = (splitmix64(seed, counter) >> np.uint64(32)).astype(np.uint64)
    with np.errstate(over="ignore"):
        return ((u * np.uint64(hi)) >> np.uint64(32)).astype(np.int64)


@dataclass
class SeqSet:
    """The paper's indexed format (P20 §IV.B): count, max length, offsets; ASCII residues."""
    residues: np.ndarray  # uint8 ASCII, concatenated
    offsets: np.ndarray   # int64, n+1 entries, offsets[0] = 0
    names: list = field(default_factory=list)

    @property
    def n(self) -> int:
        return len(self.offsets) - 1

    @property
    def lengths(self) -> np.ndarray:
        return np.diff(self.offsets)

    @property
    def max_len(self) -> int:
        return int(self.lengths.max()) if self.n else 0

    @property
    def total(self) -> int:
        return int(self.offsets[-1])

    def seq(self, i: int) -> bytes:
        return self.residues[self.offsets[i]:self.offsets[i + 1]].tobytes()

    def subset(self, idx) -> "SeqSet":
        return SeqSet.from_list([self.seq(int(i)) for i in idx])

    @staticmethod
    def from_list(seqs) -> "SeqSet":
        bs = [s.encode() if isinstance(s, str) else bytes(s) for s in seqs]
        lens = np.array([len(b) for b in bs], dtype=np.int64)
        off = np.zeros(len(bs) + 1, dtype=np.int64)
        np.cumsum(lens, out=off[1:])
        res = np.frombuffer(b"".join(bs), dtype=np.uint8).copy() if bs else np.zeros(0, np.uint8)
        return SeqSet(res, off)


def _composition_cdf32() -> np.ndarray:
    p = np.array([COMPOSITION[a] for a in AMINO], dtype=np.float64)
    p = p / p.sum()
    return np.round(np.cumsum(p)[:-1] * 4294967296.0).astype(np.uint64)


_AMINO_BYTES = np.frombuffer(AMINO.encode(), dtype=np.uint8)


def residues(seed: int, start: int, count: int, freqs: dict | None = None) -> np.ndarray:
    """count residues (ASCII uint8) drawn i.i.d. from the composition, counters start.."""
    if freqs is None:
        cdf = _composition_cdf32()
        letters = _AMINO_BYTES
    else:
        keys = sorted(freqs)
        p = np.array([freqs[k] for k in keys], np.float64)
        p /= p.sum()
        cdf = np.round(np.cumsum(p)[:-1] * 4294967296.0).astype(np.uint64)
        letters = np.frombuffer("".join(keys).encode(), np.uint8)
    out = np.empty(count, dtype=np.uint8)
    chunk = 1 << 24
    for s in range(0, count, chunk):
        e = min(count, s + chunk)
        u = splitmix64(seed, np.arange(start + s, start + e, dtype=np.uint64)) >> np.uint64(32)
        out[s:e] = letters[np.searchsorted(cdf, u, side="right")]
    return out


def _lognormal_lengths(seed: int, n: int, mean: float, median: float, tail_frac: float,
                       lo: int = MIN_DB_LEN, hi: int = MAX_DB_LEN) -> np.ndarray:
    from scipy.special import ndtri

    sigma = math.sqrt(max(1e-9, 2.0 * math.log(mean / median)))
    n_tail = int(round(n * tail_frac))
    k = np.arange(n, dtype=np.uint64)
    z = ndtri(uniform01(stream_seed(seed, "len-body"), k))
    ut = uniform01(stream_seed(seed, "len-tail"), k)
    tail_len = np.exp(math.log(3000.0) + ut * (math.log(hi) - math.log(3000.0)))
    is_tail = np.zeros(n, bool)
    if n_tail:
        pick = np.argsort(splitmix64(stream_seed(seed, "tail-pick"), k), kind="stable")[:n_tail]
        is_tail[pick] = True

    def draw(mu):
        body = np.exp(mu + sigma * z)
        v = np.where(is_tail, tail_len, body)
        return np.clip(np.rint(v), lo, hi).astype(np.int64)

    # solve the body location so the overall mean (tail included) hits the target
    a, b = math.log(median) - 3.0, math.log(median) + 1.0
    for _ in range(60):
        mid = 0.5 * (a + b)
        if draw(mid).mean() < mean:
            a = mid
        else:
            b = mid
    return draw(0.5 * (a + b))


def query_lengths(n_queries: int, l_max: int, l_min: int = 100) -> list[int]:
    """Reading R15: L_k = round(100 + k (L_max - 100)/(n-1)), k = 0..n-1."""
    if n_queries == 1:
        return [l_min]
    return [int(math.floor(l_min + k * (l_max - l_min) / (n_queries - 1) + 0.5))
            for k in range(n_queries)]


def mutate(seed: int, src: bytes, identity: float, indel: float = 0.02) -> bytes:
    """A homolog of src: each position kept with prob. identity, else substituted;
    with prob. indel an insertion or deletion of one residue."""
    n = len(src)
    k = np.arange(4 * n + 8, dtype=np.uint64)
    u = uniform01(seed, k)
    subs = residues(stream_seed(seed, "subs"), 0, 2 * n + 4)
    out = bytearray()
    si = 0
    for i in range(n):
        r = u[4 * i]
        if r < indel / 2:              # deletion
            continue
        if r < indel:                  # insertion before this residue
            out.append(subs[si]); si += 1
        if u[4 * i + 1] < identity:
            out.append(src[i])
        else:
            out.append(subs[si]); si += 1
    return bytes(out)


@dataclass
class Workload:
    name: str
    queries: SeqSet
    db: SeqSet
    meta: dict


# name: (n_queries, L_max, n_db, mean, median, tail, n_homologs)
CONFIGS = {
    "C1": dict(n_queries=1, l_max=100, n_db=2000, mean=350.0, median=285.0, tail=0.0,
               homologs=True, seed=1001,
               doc="1 query of 100 aa vs 2,000 SwissProt-shaped sequences (mean ~350)"),
    "C2": dict(n_queries=40, l_max=4996, n_db=25160, mean=550.0, median=430.0, tail=0.002,
               homologs=True, seed=1002,
               doc="40 queries 100-4,996 aa vs Ensembl-Dog-shaped db (25,160 seqs)"),
    "C3": dict(n_queries=40, l_max=4981, n_db=34705, mean=550.0, median=430.0, tail=0.002,
               homologs=True, seed=1003,
               doc="40 queries 100-4,981 aa vs RefSeq-Human-shaped db (34,705 seqs)"),
    "C4": dict(n_queries=40, l_max=4998, n_db=537505, mean=355.0, median=285.0, tail=0.002,
               homologs=True, seed=1004,
               doc="40 queries 100-4,998 aa vs SwissProt-shaped db (537,505 seqs)"),
    "C5": dict(n_queries=8, l_max=5000, n_db=2048, mean=None, median=None, tail=0.0,
               homologs=False, seed=1005,
               doc="8 x 5,000-aa queries vs 2,048 sequences of 10k-35k aa (long-sequence stress)"),
    # NEXT-4 shapes (Table II): Ensembl Rat and RefSeq Mouse
    "RAT": dict(n_queries=40, l_max=4992, n_db=32971, mean=550.0, median=430.0, tail=0.002,
                homologs=True, seed=1006, doc="40 queries vs Ensembl-Rat-shaped db (32,971 seqs)"),
    "MOUSE": dict(n_queries=40, l_max=5000, n_db=29437, mean=550.0, median=430.0, tail=0.002,
                  homologs=True, seed=1007, doc="40 queries vs RefSeq-Mouse-shaped db (29,437)"),
}


def make_workload(name: str, n_db: int | None = None, n_queries: int | None = None,
                  l_max: int | None = None, seed: int | None = None) -> Workload:
    """Build a config (optionally scaled down: fewer DB sequences / queries)."""
    cfg = dict(CONFIGS[name])
    if n_db is not None:
        cfg["n_db"] = n_db
    if n_queries is not None:
        cfg["n_queries"] = n_queries
    if l_max is not None:
        cfg["l_max"] = l_max
    if seed is not None:
        cfg["seed"] = seed
    seed = cfg["seed"]
    nd, nq = cfg["n_db"], cfg["n_queries"]

    if name == "C5":
        lens = 10000 + randint(stream_seed(seed, "c5-len"), np.arange(nd, dtype=np.uint64), 25001)
        qlens = [cfg["l_max"]] * nq
    else:
        lens = _lognormal_lengths(seed, nd, cfg["mean"], cfg["median"], cfg["tail"])
        qlens = query_lengths(nq, cfg["l_max"])

    # database residues
    off = np.zeros(nd + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    res = residues(stream_seed(seed, "db-res"), 0, int(off[-1]))
    seqs_override = {}

    # queries ("chosen ... from each genomic database", P20): generated, then
    # written over seeded DB slots (reading R16)
    qs = []
    qoff = 0
    for k, L in enumerate(qlens):
        if name == "C5" and k == nq - 1:
            # planted overflow query: W/C-rich (mean diagonal >= 6.6, self-score > 32767)
            q = residues(stream_seed(seed, "q-overflow"), 0, L, {"W": 0.5, "C": 0.3, "Y": 0.2})
        else:
            q = residues(stream_seed(seed, "queries"), qoff, L)
        qoff += L
        qs.append(q.tobytes())
    slot_order = np.argsort(splitmix64(stream_seed(seed, "slots"), np.arange(nd, dtype=np.uint64)),
                            kind="stable")
    used = 0
    planted = []
    if name == "C5":
        # embed each query inside a long DB sequence (keeps lengths in [10k, 35k])
        for k, q in enumerate(qs):
            if used >= nd:
                break
            slot = int(slot_order[used]); used += 1
            L = int(lens[slot])
            flank = residues(stream_seed(seed, f"flank{k}"), 0, max(0, L - len(q)))
            cut = len(flank) // 2
            seqs_override[slot] = flank[:cut].tobytes() + q + flank[cut:].tobytes()
            planted.append(dict(query=k, slot=slot, kind="self"))
    else:
        for k, q in enumerate(qs):
            if used >= nd:
                break
            slot = int(slot_order[used]); used += 1
            seqs_override[slot] = q
            planted.append(dict(query=k, slot=slot, kind="self"))
        if cfg["homologs"]:
            for k, q in enumerate(qs):
                for h, ident in enumerate((0.9, 0.7, 0.5, 0.4, 0.3)):
                    if used >= nd:
                        break
                    slot = int(slot_order[used]); used += 1
                    seqs_override[slot] = mutate(stream_seed(seed, f"hom{k}.{h}"), q, ident)
                    planted.append(dict(query=k, slot=slot, kind=f"homolog{int(ident*100)}"))

    if seqs_override:
        lens2 = lens.copy()
        for s, b in seqs_override.items():
            lens2[s] = len(b)
        off2 = np.zeros(nd + 1, np.int64)
        np.cumsum(lens2, out=off2[1:])
        res2 = np.empty(int(off2[-1]), np.uint8)
        # copy the untouched runs of sequences between overridden slots in bulk
        prev = 0
        for s in sorted(seqs_override) + [nd]:
            if s > prev:
                res2[off2[prev]:off2[s]] = res[off[prev]:off[s]]
            prev = s + 1
        for s, b in seqs_override.items():
            res2[off2[s]:off2[s + 1]] = np.frombuffer(b, np.uint8)
        off, res = off2, res2

    db = SeqSet(res, off)
    queries = SeqSet.from_list(qs)
    meta = dict(config=name, seed=seed, n_db=nd, n_queries=nq, query_lengths=qlens,
                db_residues=int(off[-1]), planted=planted, doc=cfg["doc"],
                cells=int(sum(qlens)) * int(off[-1]))
    return Workload(name, queries, db, meta)


def random_matrix(seed: int, lo: int = -8, hi: int = 12) -> np.ndarray:
    """A random symmetric 24x24 int8 substitution matrix (input for parity tests)."""
    k = np.arange(24 * 24, dtype=np.uint64)
    m = (lo + randint(seed, k, hi - lo + 1)).reshape(24, 24)
    m = np.triu(m) + np.triu(m, 1).T
    return m.astype(np.int8)


def random_seqset(seed: int, n: int, min_len: int, max_len: int, alphabet: str = AMINO) -> SeqSet:
    """n sequences, lengths uniform in [min_len, max_len], residues uniform over alphabet."""
    k = np.arange(n, dtype=np.uint64)
    lens = min_len + randint(stream_seed(seed, "rl"), k, max_len - min_len + 1)
    off = np.zeros(n + 1, np.int64)
    np.cumsum(lens, out=off[1:])
    letters = np.frombuffer(alphabet.encode(), np.uint8)
    idx = randint(stream_seed(seed, "rr"), np.arange(int(off[-1]), dtype=np.uint64), len(alphabet))
    return SeqSet(letters[idx], off)
