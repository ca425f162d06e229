import sys; sys.path.insert(0,'.')
import numpy as np, oracle, seqgen
from paper_conf_ipps_mendoncam13_b200 import Database
w = seqgen.make_workload("C5", n_db=24)
ref = oracle.search(w.queries, w.db)
D = Database(w.db)
for streams in (4, 1):
    r = D.search(w.queries, top_k=5, streams=streams)
    bad = np.argwhere(r.scores != ref)
    print("streams", streams, "bad", len(bad), "ovf", r.stats["n_overflow_pairs"], [(int(q), int(d), int(r.scores[q,d]), int(ref[q,d])) for q, d in bad[:10]])
print("planted", w.meta["planted"])
