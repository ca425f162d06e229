"""K2 (int32 re-run) timing on one big pair: a 5,000-aa query vs a 35,000-residue sequence
(C5's planted overflow shape).  alpha + beta > 16384 routes every pair to K2; the time is
the K2 launch's own (stats kernel_seconds_k2).  SW_K2_BIG=<huge>: the single-CTA path.
  python tools/k2_timing.py [--m 5000] [--n 35000] [--reps 5]"""
import argparse
import os
import sys

# every pair is routed to K2 here, and a routed search runs big pairs one block each
# (throughput); time the split path that a saturated big pair takes in a normal search
os.environ.setdefault("SW_K2_BIG", str(1 << 24))

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--m", type=int, default=5000)
ap.add_argument("--n", type=int, default=35000)
ap.add_argument("--reps", type=int, default=5)
args = ap.parse_args()
qs = seqgen.SeqSet.from_list([seqgen.residues(1, 0, args.m).tobytes()])
db = seqgen.SeqSet.from_list([seqgen.residues(2, 0, args.n).tobytes()])
D = Database(db, devices=[0])
ts = []
for _ in range(args.reps + 1):
    r = D.search(qs, top_k=1, gap_open=20000, gap_extend=3)
    ts.append(r.stats["kernel_seconds_k2"])
D.close()
t = min(ts[1:])
print(f"K2 {args.m} x {args.n}: {t * 1e3:.2f} ms ({args.m * args.n / t / 1e9:.1f} GCUPS), "
      f"SW_K2_BIG={os.environ.get('SW_K2_BIG', 'default')}, score {int(r.scores[0, 0])}")
