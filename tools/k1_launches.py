"""Per-launch K1 rates of a single-stream search (each launch alone on the GPU): groups,
cells, device ms and GCUPS per unit, sorted by launch order; summary by unit size class.
  python tools/k1_launches.py [--config C4] [--out FILE]"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--out", default=None)
args = ap.parse_args()
w = seqgen.make_workload(args.config)
D = Database(w.db)
D.search(w.queries, top_k=10, outputs_on_device=True, streams=1)
r = D.search(w.queries, top_k=10, outputs_on_device=True, streams=1)
log = sorted(r.stats["unit_log"], key=lambda e: e["dev_t0"])
k1 = [e for e in log if e["kind"] == 0]
tot_c = sum(e["cells"] for e in k1)
tot_t = sum(e["device_ms"] for e in k1) * 1e-3
print(f"K1: {len(k1)} launches, {tot_c:.3e} cells, {tot_t:.3f} s -> {tot_c / tot_t / 1e9:.1f} GCUPS alone")
rates = sorted((e["cells"] / (e["device_ms"] * 1e6), e["cells"], e["device_ms"], e["unit"]) for e in k1)
for q in (0, 0.1, 0.25, 0.5, 0.75, 0.9, 1.0):
    x = rates[min(len(rates) - 1, int(q * len(rates)))]
    print(f"  p{int(q * 100):3d}: {x[0]:8.1f} GCUPS  cells {x[1]:.3e}  {x[2]:.2f} ms  unit {x[3]}")
small = [x for x in rates if x[1] < 0.5 * tot_c / len(k1)]
print(f"  units below half the mean size: {len(small)}, their cells {sum(x[1] for x in small) / tot_c:.3%}, "
      f"time {sum(x[2] for x in small) * 1e-3 / tot_t:.3%}")
if args.out:
    json.dump(dict(k1=[dict(unit=e["unit"], cells=e["cells"], ms=e["device_ms"], pair=e["pair"]) for e in k1]),
              open(args.out, "w"))
D.close()
