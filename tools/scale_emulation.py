"""Strong-scaling emulation on one B200 (no multi-GPU node available): N workers share the
GPU, each on its own green-context SM partition (sw_opts.worker_sms = n_SM // 8 by default,
rounded down to a multiple of 8: 16 SMs), i.e. N emulated GPUs of 16 SMs whose kernels cannot
leave their SMs (they share the L2 and HBM).  For N = 1, 2, 4, 8 it reports device-timed GCUPS of the whole
search (PSS + WA, the in-process data plane: committed segments and hit lists copied to the
first worker and merged), the efficiency GCUPS(N) / (N x GCUPS(1)), units per worker,
request messages and the bytes the merge moved.  Scores are checked against the oracle's digest.
  python tools/scale_emulation.py [--config C4] [--sms 18] [--streams 2] [--out FILE]"""
import argparse
import hashlib
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402

ap = argparse.ArgumentParser()
ap.add_argument("--config", default="C4")
ap.add_argument("--sms", type=int, default=0, help="SMs per emulated GPU (0 = n_SM // 8)")
ap.add_argument("--streams", type=int, default=2)
ap.add_argument("--ns", default="1,2,4,8")
ap.add_argument("--reps", type=int, default=1)
ap.add_argument("--out", default=None)
args = ap.parse_args()
import torch  # noqa: E402
n_sm = torch.cuda.get_device_properties(0).multi_processor_count
sms = args.sms or n_sm // 8
w = seqgen.make_workload(args.config)
gold = json.load(open(os.path.join(ROOT, "tests", "golden", "oracle_digests.json"))).get(args.config)
rows = []
for n in [int(x) for x in args.ns.split(",")]:
    D = Database(w.db, devices=[0] * n)
    D.search(w.queries, top_k=10, streams=args.streams, worker_sms=sms, want_scores=False)   # warm-up
    best = None
    for _ in range(args.reps):
        r = D.search(w.queries, top_k=10, streams=args.streams, worker_sms=sms)
        if best is None or r.stats["seconds_device"] < best[1]["seconds_device"]:
            best = (r, r.stats)
    r, st = best
    ok = None
    if gold:
        ok = hashlib.sha256(np.ascontiguousarray(r.scores, dtype="<i4").tobytes()).hexdigest() == gold["sha256_scores"]
    per = {}
    for e in st["unit_log"]:
        per.setdefault(e["worker"], 0)
        per[e["worker"]] += e["committed"]
    row = dict(n=n, sms_per_worker=sms, gcups=st["gcups"], seconds=st["seconds_device"], units=st["n_units"],
               committed_per_worker=per, tail_s=st["tail_seconds"], wa_grants=st["n_wa_grants"],
               cancelled=st["n_cancelled"], request_messages=st["n_requests"], peer_bytes=st["peer_bytes"],
               digest_ok=ok, partition_mode=st["partition_mode"], partition_sms=st["partition_sms"])
    rows.append(row)
    print(json.dumps(row), flush=True)
    D.close()
g1 = rows[0]["gcups"]
for row in rows:
    row["efficiency"] = row["gcups"] / (row["n"] * g1) if rows[0]["n"] == 1 else None
    eff = f"{row['efficiency']:.3f}" if row["efficiency"] is not None else "n/a"
    print(f"N={row['n']}: {row['gcups']:.1f} GCUPS, efficiency {eff}, tail {row['tail_s']:.3f} s, "
          f"merge moved {row['peer_bytes'] / 1e6:.1f} MB, digest {row['digest_ok']}", flush=True)
if args.out:
    json.dump(dict(config=args.config, sms_per_worker=sms, streams=args.streams, n_sm=n_sm,
                   note="N workers on one B200, each on its own green-context partition of partition_sms SMs "
                        "(partition_mode 2; 1 = CTA caps): N emulated GPUs",
                   rows=rows), open(args.out, "w"), indent=1)
