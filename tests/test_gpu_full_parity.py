"""Every pair of every full-size config, bit-exact: libsw's complete score matrix is hashed
and compared with the SHA-256 of the oracle's matrix for the same seeded inputs
(tests/golden/oracle_digests.json, written by tools/make_golden_digests.py, which calls only
oracle/).  BASELINE.json north_star: "bit-exact scores versus the oracle on all five
configs".  Runs in the launch configuration bench.py times (PSS + WA, 4 streams, top-10).
"""
import hashlib
import json
import os

import numpy as np
import pytest

import seqgen
from paper_conf_ipps_mendoncam13_b200 import Database

pytestmark = pytest.mark.gpu

GOLDEN = os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "oracle_digests.json")


def _golden():
    with open(GOLDEN) as f:
        return json.load(f)


@pytest.mark.parametrize("cfg", ["C1", "C2", "C3", "C4", "C5", "RAT", "MOUSE", "C5@256"])
def test_full_matrix_digest(cfg):
    """(C5@256: C5's database cut to 256 sequences, one GPU's share at 8 GPUs -- the K3
    cluster-split path.)"""
    g = _golden()
    if cfg not in g:
        pytest.skip(f"no oracle digest for {cfg} yet")
    e = g[cfg]
    name, _, n_db = cfg.partition("@")
    w = seqgen.make_workload(name, n_db=int(n_db) if n_db else None)
    assert (w.queries.n, w.db.n) == (e["n_queries"], e["n_db"])
    D = Database(w.db, devices=[0])
    try:
        r = D.search(w.queries, top_k=10)
    finally:
        D.close()
    sc = np.ascontiguousarray(r.scores, dtype="<i4")
    assert int(sc.max()) == e["max_score"]
    assert int((sc > 32767).sum()) == e["n_above_int16"]
    assert hashlib.sha256(sc.tobytes()).hexdigest() == e["sha256_scores"]
    assert (np.asarray(r.hit_scores) == np.asarray(e["top10_scores"])).all()
    assert (np.asarray(r.hit_index) == np.asarray(e["top10_index"])).all()
