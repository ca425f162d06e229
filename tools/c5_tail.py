"""C5 (long-sequence, intra-task K3 path) timeline: GCUPS and where the step's tail goes.

  python tools/c5_tail.py [--unit-cells N ...]

For each setting: device seconds, GCUPS, units, the moment the last unit starts, and the
per-unit durations (a K3 unit lasts as long as its longest warp task = one whole
(query pack, long sequence) pair)."""
import argparse
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C5")
ap.add_argument("--unit-cells", type=int, nargs="*", default=[0])
ap.add_argument("--streams", type=int, nargs="*", default=[4])
ap.add_argument("--reps", type=int, default=3)
ap.add_argument("--n-db", type=int, default=None)
args = ap.parse_args()

w = seqgen.make_workload(args.config, n_db=args.n_db) if args.n_db else seqgen.make_workload(args.config)
D = Database(w.db, devices=[0])
cells = int(w.meta["cells"])
for uc in args.unit_cells:
    for ns in args.streams:
        best = None
        for _ in range(args.reps + 1):
            r = D.search(w.queries, top_k=10, outputs_on_device=True, streams=ns, target_unit_cells=uc)
            st = r.stats
            if best is None or st["seconds_device"] < best["seconds_device"]:
                best = st
        log = best["unit_log"]
        t0 = min(e["t_start"] for e in log)
        last_start = max(e["t_start"] for e in log) - t0
        end = max(e["t_end"] for e in log) - t0
        durs = sorted(((e["t_end"] - e["t_start"]) * 1e3, e["kind"], e["cells"]) for e in log)
        print(json.dumps({"unit_cells": uc, "streams": ns, "sec": best["seconds_device"],
                          "gcups": cells / best["seconds_device"] / 1e9, "units": len(log),
                          "last_start_ms": 1e3 * last_start, "end_ms": 1e3 * end,
                          "k3_kernel_s": best["kernel_seconds_k3"], "k2_kernel_s": best["kernel_seconds_k2"],
                          "last_unit_end_dev_ms": max(e["dev_t1"] for e in log), "k1_kernel_s": best["kernel_seconds_k1"],
                          "longest_units_ms": [round(d, 1) for d, _, _ in durs[-6:]],
                          "shortest_units_ms": [round(d, 1) for d, _, _ in durs[:3]]}), flush=True)
D.close()
