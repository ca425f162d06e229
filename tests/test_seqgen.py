"""The seeded input generator: determinism, shapes and the recipe of DESIGN.md §4."""
import numpy as np
import pytest

import seqgen


def test_splitmix64_known_values():
    # reference values of splitmix64 with state 0 (Vigna's reference implementation):
    # first outputs are 0xe220a8397b1dcdaf, 0x6e789e6aa1b965f4, 0x06c45d188009454f
    out = seqgen.splitmix64(0, np.arange(3, dtype=np.uint64))
    assert [int(x) for x in out] == [0xE220A8397B1DCDAF, 0x6E789E6AA1B965F4, 0x06C45D188009454F]


def test_deterministic_and_counter_based():
    a = seqgen.residues(5, 0, 1000)
    b = seqgen.residues(5, 0, 1000)
    c = seqgen.residues(5, 500, 500)
    assert (a == b).all() and (a[500:] == c).all()


def test_composition():
    r = seqgen.residues(77, 0, 2_000_000)
    freq = {chr(k): v for k, v in zip(*np.unique(r, return_counts=True))}
    tot = sum(seqgen.COMPOSITION.values())
    for aa, pct in seqgen.COMPOSITION.items():
        assert abs(freq[aa] / len(r) - pct / tot) < 0.002


def test_query_lengths_reading_R15():
    L = seqgen.query_lengths(40, 4998)
    assert L[0] == 100 and L[-1] == 4998 and len(L) == 40
    assert all(b > a for a, b in zip(L, L[1:]))


def test_c1_c2_shapes():
    w = seqgen.make_workload("C1")
    assert w.queries.n == 1 and w.queries.lengths[0] == 100 and w.db.n == 2000
    assert 300 < w.db.total / w.db.n < 420
    w2 = seqgen.make_workload("C2", n_db=3000)
    assert w2.db.n == 3000 and w2.queries.n == 40
    assert w2.db.lengths.min() >= 10 and w2.db.lengths.max() <= seqgen.MAX_DB_LEN
    # queries drawn into the DB (reading R16) and homologs planted
    selfs = [p for p in w2.meta["planted"] if p["kind"] == "self"]
    assert len(selfs) == 40
    for p in selfs:
        assert w2.db.seq(p["slot"]) == w2.queries.seq(p["query"])
    w3 = seqgen.make_workload("C2", n_db=3000)
    assert (w3.db.residues == w2.db.residues).all() and (w3.db.offsets == w2.db.offsets).all()


def test_c5_shape():
    w = seqgen.make_workload("C5", n_db=64)
    assert w.db.lengths.min() >= 10000 and w.db.lengths.max() <= 35000
    assert (w.queries.lengths == 5000).all()
    for p in w.meta["planted"]:
        assert w.queries.seq(p["query"]) in w.db.seq(p["slot"])


def test_seqset_indexed_format():
    s = seqgen.SeqSet.from_list(["AC", "", "WWW"])
    assert s.n == 3 and s.offsets.tolist() == [0, 2, 2, 5] and s.max_len == 3
    assert s.seq(2) == b"WWW" and s.seq(1) == b""


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C5", "RAT", "MOUSE", "C5@256", "C4"])
def test_generated_inputs_match_committed_digests(cfg):
    """The seeded inputs behind tests/golden/oracle_digests.json are byte-identical on this
    host (the generator's length draws use libm; a different rounding fails here, loudly)."""
    import hashlib
    import json
    import os
    import numpy as np
    g = json.load(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "input_digests.json")))[cfg]

    def dig(s):
        h = hashlib.sha256()
        h.update(np.ascontiguousarray(s.offsets, dtype="<i8").tobytes())
        h.update(np.ascontiguousarray(s.residues, dtype=np.uint8).tobytes())
        return h.hexdigest()
    name, _, n_db = cfg.partition("@")
    w = seqgen.make_workload(name, n_db=int(n_db) if n_db else None)
    assert (w.queries.n, w.db.n) == (g["n_queries"], g["n_db"])
    assert dig(w.queries) == g["queries"] and dig(w.db) == g["db"]
