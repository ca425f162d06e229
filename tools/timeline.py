"""Device timeline of one search (unit replicas per stream, device ms since the worker's
start event) -- where a step's time goes.
  python tools/timeline.py --config C5 [--n-db 256] [--streams 4] [--reps 2]"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--n-db", type=int, default=None)
ap.add_argument("--streams", type=int, default=4)
ap.add_argument("--reps", type=int, default=2)
ap.add_argument("--unit-cells", type=int, default=0)
ap.add_argument("--summary", action="store_true", help="print only the summary line")
args = ap.parse_args()
w = seqgen.make_workload(args.config, n_db=args.n_db)
D = Database(w.db, devices=[0])
best = None
for _ in range(args.reps + 1):
    st = D.search(w.queries, top_k=10, outputs_on_device=True, streams=args.streams,
                  target_unit_cells=args.unit_cells).stats
    if best is None or st["seconds_device"] < best["seconds_device"]:
        best = st
print(f"{args.config} n_db={w.db.n}: {best['gcups']:.1f} GCUPS, device {1e3 * best['seconds_device']:.2f} ms, "
      f"units {best['n_units']}, overflow pairs {best['n_overflow_pairs']}, launches {best['kernel_launches']}")
for e in ([] if args.summary else sorted(best["unit_log"], key=lambda e: (e["stream"], e["dev_t0"]))):
    print(f"  stream {e['stream']} unit {e['unit']:4d} kind {'K1' if e['kind'] == 0 else 'K3'} pack {e['pair']:3d} "
          f"[{e.get('b0')},{e.get('b1')}) C={e.get('cluster')} "
          f"dev {e['dev_t0']:8.2f} -> {e['dev_t1']:8.2f} ms ({e['device_ms']:7.2f}) cells {e['cells']:.3e} "
          f"-> {e['cells'] / max(e['device_ms'], 1e-6) / 1e6:7.1f} GCUPS")
D.close()
