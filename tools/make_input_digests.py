"""Write tests/golden/input_digests.json: SHA-256 of every config's seeded inputs (queries and
database: offsets + residues) as seqgen generates them.  The generator draws lengths with
floating-point libm calls (ndtri / exp / rint); tests/test_seqgen.py regenerates the configs and
compares, so a host whose libm rounds differently fails loudly instead of silently changing the
inputs behind tests/golden/oracle_digests.json.
  python tools/make_input_digests.py [C1 C2 ...]"""
import hashlib
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import seqgen  # noqa: E402

OUT = os.path.join(ROOT, "tests", "golden", "input_digests.json")


def seqset_digest(s):
    h = hashlib.sha256()
    h.update(np.ascontiguousarray(s.offsets, dtype="<i8").tobytes())
    h.update(np.ascontiguousarray(s.residues, dtype=np.uint8).tobytes())
    return h.hexdigest()


def main(cfgs):
    data = json.load(open(OUT)) if os.path.exists(OUT) else {}
    for cfg in cfgs:
        name, _, n_db = cfg.partition("@")
        w = seqgen.make_workload(name, n_db=int(n_db) if n_db else None)
        data[cfg] = {"queries": seqset_digest(w.queries), "db": seqset_digest(w.db),
                     "n_queries": int(w.queries.n), "n_db": int(w.db.n), "db_residues": int(w.db.total)}
        print(cfg, data[cfg]["db"][:16], flush=True)
    json.dump(data, open(OUT, "w"), indent=1)


if __name__ == "__main__":
    main(sys.argv[1:] or ["C1", "C2", "C3", "C4", "C5", "RAT", "MOUSE", "C5@256"])
