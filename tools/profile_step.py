"""One (or more) sw_search steps on a config, for ncu launch lists / captures.
  python tools/profile_step.py --config C4 [--steps 1] [--n-db N]"""
import argparse
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--steps", type=int, default=1)
ap.add_argument("--n-db", type=int, default=None)
ap.add_argument("--n-queries", type=int, default=None)
ap.add_argument("--streams", type=int, default=3)
ap.add_argument("--long-threshold", type=int, default=0)
ap.add_argument("--unit-cells", type=int, default=0)
ap.add_argument("--dump-log", default=None)
ap.add_argument("--print-k1", type=int, default=0, help="print the first N K1 units (launch order)")
args = ap.parse_args()
w = seqgen.make_workload(args.config, n_db=args.n_db, n_queries=args.n_queries)
D = Database(w.db)
for s in range(args.steps):
    t = time.perf_counter()
    r = D.search(w.queries, top_k=10, outputs_on_device=True, streams=args.streams,
                 long_threshold=args.long_threshold, target_unit_cells=args.unit_cells)
    st = r.stats
    print(f"step {s}: {st['gcups']:.1f} GCUPS dev {st['seconds_device']:.3f}s wall {time.perf_counter()-t:.3f}s "
          f"k1 {st['kernel_seconds_k1']:.3f}s/{st['cells_k1']:.3e} k3 {st['kernel_seconds_k3']:.3f}s/{st['cells_k3']:.3e} "
          f"units {st['n_units']} launches {st['kernel_launches']}", flush=True)
    if args.print_k1:
        k1 = sorted((e for e in st["unit_log"] if e["kind"] == 0), key=lambda e: e["t_start"])
        for e in k1[:args.print_k1]:
            print(f"k1 unit {e['unit']} cells {e['cells']} pair {e['pair']}")
    if args.dump_log:
        import json
        json.dump(st["unit_log"], open(args.dump_log, "w"))
