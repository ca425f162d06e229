"""Precision routing (alpha + beta > 16384): every pair re-scored by the int32 kernel (K2).
Device time of one search of C2's queries against the first N database sequences.
  python tools/k2_routing_timing.py [--n-db 2000]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--n-db", type=int, default=2000)
args = ap.parse_args()
w = seqgen.make_workload("C2")
db = seqgen.SeqSet.from_list([w.db.seq(i) for i in range(args.n_db)])
D = Database(db, devices=[0])
best = None
for _ in range(3):
    r = D.search(w.queries, top_k=5, gap_open=20000, gap_extend=3)
    best = r.stats if best is None or r.stats["seconds_device"] < best["seconds_device"] else best
D.close()
import paper_conf_ipps_mendoncam13_b200 as _p; print(_p.__file__)
print(f"routing C2 x {args.n_db} seqs: {best['seconds_device'] * 1e3:.1f} ms, {best['gcups']:.1f} GCUPS, "
      f"{best['n_overflow_pairs']} pairs re-run")
