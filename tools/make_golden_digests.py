"""Write tests/golden/oracle_digests.json: for each full-size config, the SHA-256 of the
ORACLE's complete score matrix (int32 little-endian, [n_queries][n_db], original orders)
and its top-10 hits.  Calls only oracle/ and seqgen/ (the seeded generator): no value in
the file comes from the CUDA path.  The GPU test (tests/test_gpu_full_parity.py) hashes
libsw's matrix for the same seeded inputs and compares, i.e. every pair of every config is
checked bit-exactly (BASELINE.json north_star: "bit-exact scores versus the oracle on all
five configs").

  python tools/make_golden_digests.py [C1 C2 C3 C5 C4 ...]   (C4 takes ~1 h on 8 cores)
  A name "CFG@N" is config CFG with its database cut to N sequences (e.g. C5@256: one GPU's
  share of C5 at 8 GPUs).
"""
import hashlib
import json
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import seqgen  # noqa: E402

OUT = os.environ.get("GOLDEN_OUT") or os.path.join(ROOT, "tests", "golden", "oracle_digests.json")


def digest(scores: np.ndarray) -> str:
    return hashlib.sha256(np.ascontiguousarray(scores, dtype="<i4").tobytes()).hexdigest()


def main(cfgs):
    data = {}
    if os.path.exists(OUT):
        with open(OUT) as f:
            data = json.load(f)
    for cfg in cfgs:
        name, _, n_db = cfg.partition("@")
        w = seqgen.make_workload(name, n_db=int(n_db) if n_db else None)
        t = time.perf_counter()
        sc = oracle.search(w.queries, w.db)
        dt = time.perf_counter() - t
        s, i = oracle.topk(sc, 10)
        data[cfg] = {
            "sha256_scores": digest(sc),
            "n_queries": int(w.queries.n), "n_db": int(w.db.n),
            "cells": int(w.meta["cells"]), "max_score": int(sc.max()),
            "n_above_int16": int((sc > 32767).sum()),
            "top10_scores": s.tolist(), "top10_index": i.tolist(),
            "oracle_seconds": round(dt, 1), "oracle_threads": os.cpu_count(),
            "matrix": "BLOSUM62", "gap_open": 10, "gap_extend": 2,
            "writer": "tools/make_golden_digests.py (oracle.search on seqgen.make_workload(cfg[, n_db]))",
        }
        with open(OUT + ".tmp", "w") as f:
            json.dump(data, f, indent=1)
        os.replace(OUT + ".tmp", OUT)
        print(f"{cfg}: {dt:.0f} s, max {sc.max()}, sha256 {data[cfg]['sha256_scores'][:16]}", flush=True)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C1", "C2", "C3", "C5", "C4"])
