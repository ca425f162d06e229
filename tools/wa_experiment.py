"""The paper's workload-adjustment experiment (Fig. 6, P22 §V.B) and non-dedicated run
(Figs. 7/8, P24 §V.C) on one B200: P slave workers share the GPU (separate streams and
replicas of the database); one of them can emulate a slower PE (6x, Fig. 5's ratio),
from the start or from a point mid-run (local load).  For each policy (SS, PSS) and WA
on/off it reports makespan (device), GCUPS, tail (makespan - median worker finish),
duplicated cells, WA grants and master interactions; scores are checked identical across
all runs.

  python tools/wa_experiment.py [--config C2] [--workers 4] [--reps 2] [--out FILE]
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C2")
    ap.add_argument("--workers", type=int, default=4)
    ap.add_argument("--reps", type=int, default=2)
    ap.add_argument("--slowdown", type=int, default=6)
    ap.add_argument("--out", default=None)
    ap.add_argument("--unit-cells", type=int, default=0,
                    help="target_unit_cells (0 = auto; 2**62 = the paper's very coarse tasks, one per pack)")
    args = ap.parse_args()
    w = seqgen.make_workload(args.config)
    D = Database(w.db, devices=[0] * args.workers)
    straggler = 1 << (args.workers - 1)
    base = D.search(w.queries, top_k=10, streams=2)   # warm-up + reference scores
    ref = base.scores.copy()
    t_ref = base.stats["seconds_device"]
    scenarios = [("homogeneous", 0, 0), ("straggler", straggler, 0),
                 ("local_load_midrun", straggler, int(1000 * 0.3 * t_ref))]
    rows = []
    for name, mask, after in scenarios:
        for policy in ("pss", "ss"):
            for wa in (True, False):
                best = None
                for _ in range(args.reps):
                    r = D.search(w.queries, top_k=10, streams=2, policy=policy, workload_adjust=wa,
                                 straggler_mask=mask, straggler_slowdown=args.slowdown,
                                 straggler_after_ms=after, target_unit_cells=args.unit_cells)
                    assert (r.scores == ref).all(), "scores differ across schedules"
                    st = r.stats
                    if best is None or st["seconds_device"] < best["seconds_device"]:
                        best = st
                log = best["unit_log"]
                per_worker = {}
                for e in log:
                    d = per_worker.setdefault(e["worker"], {"units": 0, "committed": 0, "cells": 0,
                                                            "last_end": 0.0})
                    d["units"] += 1
                    d["committed"] += e["committed"]
                    d["cells"] += e["cells"]
                    d["last_end"] = max(d["last_end"], e["t_end"])
                row = dict(scenario=name, policy=policy, wa=wa, makespan_s=best["seconds_device"],
                           gcups=best["gcups"], tail_s=best["tail_seconds"],
                           duplicated_cells=best["duplicated_cells"], wa_grants=best["n_wa_grants"],
                           requests=best["n_requests"], units=best["n_units"], per_worker=per_worker,
                           timeline=[(e["worker"], round(e["t_start"], 4), round(e["t_end"], 4),
                                      e["cells"], e["committed"]) for e in log])
                rows.append(row)
                print(f"{name:18s} {policy:3s} WA={'on ' if wa else 'off'} makespan {row['makespan_s']:.3f}s "
                      f"{row['gcups']:8.1f} GCUPS tail {row['tail_s']:.3f}s dup {row['duplicated_cells']:.2e} "
                      f"wa {row['wa_grants']} req {row['requests']}", flush=True)
    # WA gain per scenario/policy (the paper's Fig. 6 quantity)
    summary = {}
    for name, _, _ in scenarios:
        for policy in ("pss", "ss"):
            on = next(r for r in rows if r["scenario"] == name and r["policy"] == policy and r["wa"])
            off = next(r for r in rows if r["scenario"] == name and r["policy"] == policy and not r["wa"])
            summary[f"{name}/{policy}"] = dict(gcups_gain_pct=100.0 * (on["gcups"] / off["gcups"] - 1.0),
                                               makespan_on=on["makespan_s"], makespan_off=off["makespan_s"],
                                               tail_on=on["tail_s"], tail_off=off["tail_s"])
            print(f"WA gain {name}/{policy}: {summary[f'{name}/{policy}']['gcups_gain_pct']:+.1f} % GCUPS")
    out = dict(config=args.config, workers=args.workers, slowdown=args.slowdown, unit_cells=args.unit_cells,
               note="P workers share one B200 (separate streams/replicas); the straggler holds each "
                    "completion back by (slowdown-1) x the unit's device time",
               summary=summary, runs=rows)
    if args.out:
        with open(args.out, "w") as f:
            json.dump(out, f, indent=1)
    D.close()


if __name__ == "__main__":
    main()
