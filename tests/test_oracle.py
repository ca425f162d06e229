"""Pins for the oracle (oracle/): things other than the oracle itself fix these values.

Each test names what pins it: a value printed in the paper (PAPER.md P12/P14), a
hand-worked alignment, exhaustive enumeration (oracle/bruteforce.c, no shared code
with the DP), a closed form, a textbook routine (Kadane), or an invariant of the
definition.  Chosen so that a dropped term, a wrong sign or
index, or a transposed operand in sw_oracle.c fails at least one of them.
"""
import os

import numpy as np
import pytest

import oracle
import seqgen

GOLD = os.path.join(os.path.dirname(__file__), "golden")
AA = seqgen.AMINO


def _golden(name):
    kv, rows = {}, []
    for line in open(os.path.join(GOLD, name)):
        line = line.strip()
        if not line or line.startswith("#"):
            continue
        k, _, v = line.partition(" ")
        if k == "H":
            rows.append([int(x) for x in v.split()])
        else:
            kv[k] = v
    return kv, rows


def _dna_matrix(ma, mi):
    m = np.full((24, 24), mi, np.int8)
    np.fill_diagonal(m, ma)
    return m


def _rand_seq(rng, n, alphabet=AA):
    return "".join(alphabet[i] for i in rng.integers(0, len(alphabet), n))


# ---------------------------------------------------------------- BLOSUM62 transcription
def test_blosum62_checksums():
    kv, _ = _golden("blosum62_checksums.txt")
    B = oracle.blosum62().astype(int)
    S20 = B[:20, :20]
    assert (B == B.T).all()
    diag = {tok[0]: int(tok[1:]) for tok in kv["diagonal"].split()}
    for a, v in diag.items():
        assert B[oracle.code(a), oracle.code(a)] == v
    assert S20.sum() == int(kv["sum20x20"])
    assert S20.min() == int(kv["min20x20"]) and S20.max() == int(kv["max20x20"])
    assert B[oracle.code("X"), oracle.code("X")] == int(kv["XX"])
    assert B[oracle.code("*"), oracle.code("*")] == int(kv["**"])
    # the '*' row is -4 everywhere except */* (NCBI convention)
    assert (B[23, :23] == -4).all()


def test_alphabet_codes():
    for k, ch in enumerate(oracle.ALPHABET):
        assert oracle.code(ch) == k
        assert oracle.code(ch.lower()) == k
    for bad in "JOU1-. ":
        assert oracle.code(bad) == -1
    with pytest.raises(ValueError):
        oracle.pair_score("AJA", "AAA")


# ---------------------------------------------------------------- paper-printed values
def test_fig2_local_score_and_matrix():
    """P12/P14 Fig. 2: SW similarity matrix of GAAGCTA x GCTGACCT, score 3."""
    kv, rows = _golden("fig2_linear_sw.txt")
    M = _dna_matrix(int(kv["match"]), int(kv["mismatch"]))
    go, ge = int(kv["gap_open"]), int(kv["gap_extend"])
    s, H, E, F = oracle.dump(kv["s"], kv["t"], M, go, ge)
    assert s == int(kv["score"]) == 3
    assert (H[0] == 0).all() and (H[:, 0] == 0).all()  # "first row and column ... zeroes"
    assert H[1:].tolist() == rows
    assert oracle.pair_score(kv["s"], kv["t"], M, go, ge) == 3


def test_fig1_alignment_score():
    """P12 Fig. 1: the printed global alignment scores 4; a local alignment is >= any."""
    kv, _ = _golden("fig1_global_alignment.txt")
    M = _dna_matrix(int(kv["match"]), int(kv["mismatch"]))
    go, ge = int(kv["gap_open"]), int(kv["gap_extend"])
    assert oracle.alignment_score(kv["row_s"], kv["row_t"], M, go, ge) == 4
    s, t = kv["row_s"].replace("-", ""), kv["row_t"].replace("-", "")
    sw = oracle.pair_score(s, t, M, go, ge)
    assert sw >= 4 and sw == int(kv["sw_score"])
    assert oracle.bruteforce(s[:8], t[:8], M, go, ge) == oracle.pair_score(s[:8], t[:8], M, go, ge)


def test_affine_hand_pins():
    for line in open(os.path.join(GOLD, "affine_pins.txt")):
        if line.startswith("#") or not line.strip():
            continue
        q, d, go, ge, want = line.split()
        assert oracle.pair_score(q, d, None, int(go), int(ge)) == int(want), line
        assert oracle.bruteforce(q, d, None, int(go), int(ge)) == int(want), line


def test_alignment_scorer_affine():
    # W-W over WAW: 11 + 11 - (10 + 2)
    assert oracle.alignment_score("W-W", "WAW") == 10
    assert oracle.alignment_score("W--W", "WAAW") == 22 - 14
    # adjacent gaps in opposite rows are two separate gap runs
    assert oracle.alignment_score("W-AW", "WA-W") == 22 - 24


# ---------------------------------------------------------------- exhaustive enumeration
@pytest.mark.parametrize("go,ge", [(10, 2), (0, 1), (1, 1), (0, 0), (3, 0), (5, 3)])
def test_bruteforce_blosum(go, ge):
    rng = np.random.default_rng(100 + go * 7 + ge)
    for _ in range(60):
        q = _rand_seq(rng, int(rng.integers(0, 7)))
        d = _rand_seq(rng, int(rng.integers(0, 7)))
        assert oracle.pair_score(q, d, None, go, ge) == oracle.bruteforce(q, d, None, go, ge), (q, d)


def test_bruteforce_random_matrix_asymmetric():
    """Asymmetric matrix: catches a transposed S[q][d] vs S[d][q] lookup."""
    rng = np.random.default_rng(7)
    for trial in range(80):
        M = rng.integers(-6, 9, size=(24, 24)).astype(np.int8)
        go, ge = int(rng.integers(0, 6)), int(rng.integers(0, 4))
        q = _rand_seq(rng, int(rng.integers(1, 7)), "ACDEFG")
        d = _rand_seq(rng, int(rng.integers(1, 7)), "ACDEFG")
        assert oracle.pair_score(q, d, M, go, ge) == oracle.bruteforce(q, d, M, go, ge)


def test_bruteforce_low_complexity():
    """Repeats and long gaps: exercises E/F chains (gap extension) heavily."""
    rng = np.random.default_rng(11)
    for _ in range(60):
        q = _rand_seq(rng, int(rng.integers(3, 8)), "WA")
        d = _rand_seq(rng, int(rng.integers(3, 8)), "WAC")
        for go, ge in ((10, 2), (2, 1), (0, 3)):
            assert oracle.pair_score(q, d, None, go, ge) == oracle.bruteforce(q, d, None, go, ge)


# ---------------------------------------------------------------- closed forms / invariants
def test_I1_nonnegative_and_empty():
    assert oracle.pair_score("", "ACD") == 0
    assert oracle.pair_score("ACD", "") == 0
    assert oracle.pair_score("", "") == 0
    assert oracle.pair_score("WWW", "PPP") == 0  # all mismatches negative -> empty alignment


def test_I2_symmetry():
    rng = np.random.default_rng(2)
    for _ in range(40):
        q, d = _rand_seq(rng, int(rng.integers(1, 60))), _rand_seq(rng, int(rng.integers(1, 60)))
        assert oracle.pair_score(q, d) == oracle.pair_score(d, q)


def test_I3_self_score_closed_form():
    """score(q,q) = sum_i S[q_i][q_i] for BLOSUM62 over the 20 standard aa."""
    B = oracle.blosum62().astype(int)
    # precondition: S(a,b) <= (S(a,a)+S(b,b))/2 for all standard pairs
    for a in range(20):
        for b in range(20):
            assert 2 * B[a, b] <= B[a, a] + B[b, b]
    rng = np.random.default_rng(3)
    for L in (1, 5, 50, 400, 1500):
        q = _rand_seq(rng, L)
        want = sum(B[oracle.code(c), oracle.code(c)] for c in q)
        assert oracle.pair_score(q, q) == want


def test_I4_monotone_in_gaps_and_substring():
    rng = np.random.default_rng(4)
    for _ in range(25):
        q, d = _rand_seq(rng, 80), _rand_seq(rng, 120)
        d = d[:30] + q[10:50] + d[30:]  # a planted match with room for gaps
        prev = None
        for go in (0, 2, 5, 10, 20):
            s = oracle.pair_score(q, d, None, go, 2)
            assert prev is None or s <= prev
            prev = s
        prev = None
        for ge in (0, 1, 2, 4, 8):
            s = oracle.pair_score(q, d, None, 10, ge)
            assert prev is None or s <= prev
            prev = s
        a, b = sorted(rng.integers(0, len(d), 2))
        assert oracle.pair_score(q, d[a:b]) <= oracle.pair_score(q, d)


def _kadane_ungapped(q, d, M):
    """Textbook: max over diagonals of the maximum-subarray sum (>= 0)."""
    best = 0
    cq = [oracle.code(c) for c in q]
    cd = [oracle.code(c) for c in d]
    for off in range(-len(q) + 1, len(d)):
        run = 0
        for i in range(len(q)):
            j = i + off
            if 0 <= j < len(d):
                run = max(0, run + int(M[cq[i], cd[j]]))
                best = max(best, run)
    return best


def test_I6_large_open_is_ungapped_kadane():
    B = oracle.blosum62()
    rng = np.random.default_rng(6)
    for _ in range(30):
        q, d = _rand_seq(rng, int(rng.integers(1, 40))), _rand_seq(rng, int(rng.integers(1, 40)))
        go = 11 * min(len(q), len(d)) + 1
        assert oracle.pair_score(q, d, None, go, 1) == _kadane_ungapped(q, d, B)


def test_I7_single_residue_query():
    B = oracle.blosum62()
    rng = np.random.default_rng(8)
    for _ in range(30):
        q = _rand_seq(rng, 1)
        d = _rand_seq(rng, int(rng.integers(1, 50)))
        want = max(0, max(int(B[oracle.code(q), oracle.code(c)]) for c in d))
        assert oracle.pair_score(q, d) == want


def test_I8_concatenation_and_padding():
    rng = np.random.default_rng(9)
    for _ in range(25):
        q = _rand_seq(rng, 60)
        d1, d2 = _rand_seq(rng, 70), _rand_seq(rng, 50)
        s = oracle.pair_score(q, d1 + d2)
        assert s >= max(oracle.pair_score(q, d1), oracle.pair_score(q, d2))
        # (b) appending residues that score <= 0 against every query residue ('*' is -4)
        assert oracle.pair_score(q, d1 + "*" * 17) == oracle.pair_score(q, d1)
        assert oracle.pair_score(q + "*" * 9, d1) == oracle.pair_score(q, d1)


def test_I9_border_init_irrelevant():
    """Reading R5: any E/F border init in [-2^29, 0] gives the same score."""
    rng = np.random.default_rng(10)
    for _ in range(30):
        q, d = _rand_seq(rng, int(rng.integers(1, 70))), _rand_seq(rng, int(rng.integers(1, 70)))
        for go, ge in ((10, 2), (0, 1), (3, 0)):
            ref = oracle.pair_score(q, d, None, go, ge)
            for init in (0, -1, -(go + ge), -1000, oracle.NEG_INF):
                assert oracle.pair_score(q, d, None, go, ge, border_init=init) == ref


def test_dump_consistent_with_definition_edges():
    s, H, E, F = oracle.dump("HEAGAWGHEE", "PAWHEAE")
    assert s == H.max() == oracle.pair_score("HEAGAWGHEE", "PAWHEAE")
    assert (H >= 0).all()
    # every H cell is one of its four candidates (0, diagonal, E, F)
    B = oracle.blosum62()
    q, d = "HEAGAWGHEE", "PAWHEAE"
    for i in range(1, len(q) + 1):
        for j in range(1, len(d) + 1):
            cands = {0, H[i - 1, j - 1] + B[oracle.code(q[i - 1]), oracle.code(d[j - 1])],
                     E[i, j], F[i, j]}
            assert H[i, j] in cands and H[i, j] == max(cands)


# ---------------------------------------------------------------- search / pairs / top-k
def test_search_equals_pairwise_and_thread_invariant():
    qs = seqgen.random_seqset(21, 5, 1, 90)
    db = seqgen.random_seqset(22, 40, 0, 150)
    s1 = oracle.search(qs, db, n_threads=1)
    s4 = oracle.search(qs, db, n_threads=4)
    assert (s1 == s4).all()
    for qi in range(qs.n):
        for di in range(0, db.n, 7):
            assert s1[qi, di] == oracle.pair_score(qs.seq(qi), db.seq(di))
    qi = np.array([0, 4, 2], np.int32)
    di = np.array([3, 39, 0], np.int32)
    assert (oracle.pairs(qs, db, qi, di) == s1[qi, di]).all()


def test_topk_definition():
    scores = np.array([[5, 9, 9, 1, 0], [0, 0, 0, 0, 0]], np.int32)
    s, i = oracle.topk(scores, 3)
    assert s.tolist() == [[9, 9, 5], [0, 0, 0]]
    assert i.tolist() == [[1, 2, 0], [0, 1, 2]]
    s, i = oracle.topk(scores, 7)
    assert i[0].tolist() == [1, 2, 0, 3, 4, -1, -1] and s[0, 5:].tolist() == [0, 0]


def test_golden_digests_are_the_oracles():
    """tests/golden/oracle_digests.json (used by the full-matrix GPU parity test) holds the
    oracle's own digests: recompute the small config here and check the file's format."""
    import hashlib
    import json
    import os
    path = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "oracle_digests.json")
    with open(path) as f:
        g = json.load(f)
    w = seqgen.make_workload("C1")
    sc = oracle.search(w.queries, w.db)
    assert g["C1"]["sha256_scores"] == hashlib.sha256(np.ascontiguousarray(sc, dtype="<i4").tobytes()).hexdigest()
    s, i = oracle.topk(sc, 10)
    assert g["C1"]["top10_scores"] == s.tolist() and g["C1"]["top10_index"] == i.tolist()
    for cfg, e in g.items():
        assert len(e["sha256_scores"]) == 64 and e["n_queries"] > 0 and e["n_db"] > 0
        assert len(e["top10_index"]) == e["n_queries"]
