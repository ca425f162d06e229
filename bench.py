#!/usr/bin/env python
"""bench.py — GCUPS of the Smith-Waterman/Gotoh database search (BASELINE.json metric)
on the SwissProt-shaped 40-query workload (C4 = BASELINE configs[3]) over N B200s.

  python bench.py [--gpus N] [--steps K] [--warmup W] [--config C4] [--impl ours|reference]
  (N > 1: launched by torchrun, one process per GPU; the PSS/WA master runs in rank 0)

A step = one sw_search of all queries against the whole database: query profiles (K4),
inter-task DP (K1), intra-task DP for long sequences (K3), int32 re-run (K2), cross-rank
merge (NCCL) and top-k (K5).  The packed database is resident in HBM (sw_db_create, timed
separately); `value` is device-timed (CUDA events inside libsw, max over ranks); `e2e` is
the same search through the C-ABI with host buffers (queries in, scores + hits out to
pinned host memory) timed by the host clock around the call.
"""
from __future__ import annotations

import argparse
import hashlib
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")   # before torch creates a context

import numpy as np  # noqa: E402

import seqgen  # noqa: E402

PAPER_CONTEXT = ("paper: 7,190 s on 1 SSE core (Core i7 3.4 GHz) vs 112 s on 4x GTX580 + 4 SSE cores "
                 "for 40 queries vs SwissProt (PAPER.md P12); derived ~2.7 and ~174 GCUPS")
DPX_RATE = 64.0   # measured lane-ops/clk/SM of VIMNMX3.S16x2 / VIADDMNMX.S16x2 (tools/dpx_peak)
DPX_PER_CELL = 2.0  # K1/K3 inner loop: 4 three-input DPX per s16x2 lane word = 2 per cell
DPX_FORMULATION = 2.25  # + the running maximum (0.5 VIMNMX3 per word): the kernel's own ALU ops/cell
MICROBENCH_CELLS_PER_CLK = 24.5  # the same cell update in a register-only loop (tools/dp_variants.cu,
                                 # profiles/r01_dp_variants.txt): no barriers, borders or profile staging


def env_rank():
    return (int(os.environ.get("RANK", "0")), int(os.environ.get("WORLD_SIZE", "1")),
            int(os.environ.get("LOCAL_RANK", "0")))


class ClockSampler:
    """nvidia-smi clocks and throttle reasons sampled during the timed region."""
    FIELDS = ["clocks.sm", "clocks.max.sm", "clocks_event_reasons.hw_slowdown",
              "clocks_event_reasons.hw_thermal_slowdown", "clocks_event_reasons.sw_thermal_slowdown",
              "clocks_event_reasons.sw_power_cap"]

    def __init__(self, gpu: int):
        self.gpu, self.rows, self.proc = gpu, [], None

    def start(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), "--query-gpu=" + ",".join(self.FIELDS),
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.thread = threading.Thread(target=self._read, daemon=True)
            self.thread.start()
        except FileNotFoundError:
            self.proc = None

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) == len(self.FIELDS):
                self.rows.append(parts)

    def stop(self):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except Exception:
                self.proc.kill()
        sm = [float(r[0]) for r in self.rows if r[0].replace(".", "").isdigit()]
        mx = [float(r[1]) for r in self.rows if r[1].replace(".", "").isdigit()]
        reasons = set()
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        for r in self.rows:
            for k, nm in enumerate(names):
                if r[2 + k].lower().startswith("active"):
                    reasons.add(nm)
        return {"sm_mhz": statistics.median(sm) if sm else None,
                "sm_max_mhz": max(mx) if mx else None, "reasons": sorted(reasons),
                "samples": len(self.rows)}


def oracle_rate(w, seconds_target=15.0, seed=99, max_threads=None):
    """Time the oracle (as it stands) on a bounded random sample of the workload's pairs,
    on all host cores.  Returns (GCUPS, cores, description)."""
    import oracle
    cores = max_threads or os.cpu_count() or 1
    rng = np.random.default_rng(seed)
    qlen = w.queries.lengths

    def run(n_db):
        di = rng.integers(0, w.db.n, n_db)
        qi = np.repeat(np.arange(w.queries.n, dtype=np.int32), n_db)
        dd = np.tile(di, w.queries.n).astype(np.int32)
        cells = int((qlen[qi] * w.db.lengths[dd]).sum())
        t = time.perf_counter()
        oracle.pairs(w.queries, w.db, qi, dd, n_threads=cores)
        return cells, time.perf_counter() - t

    cells, dt = run(20)                       # calibration
    rate = cells / max(dt, 1e-6)
    avg_cells_per_db = cells / 20
    n_db = int(max(20, min(w.db.n, seconds_target * rate / max(avg_cells_per_db, 1))))
    cells, dt = run(n_db)
    desc = (f"all {w.queries.n} queries x {n_db} random DB sequences of {w.name} "
            f"({cells:.3e} cells, {dt:.1f} s, OpenMP dynamic over pairs)")
    return cells / dt / 1e9, cores, desc, cells, dt


def cpu_model():
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    return line.split(":", 1)[1].strip()
    except OSError:
        pass
    return None


def reference_arm(args):
    rank, world, _ = env_rank()
    if rank != 0:
        return 0
    w = seqgen.make_workload(args.config)
    per_step = []
    cores = os.cpu_count()
    desc = ""
    for k in range(args.warmup + args.steps):
        g, cores, desc, cells, dt = oracle_rate(w, seconds_target=args.ref_seconds, seed=1000 + k)
        if k >= args.warmup:
            per_step.append((cells, dt))
    cells = sum(c for c, _ in per_step)
    sec = sum(t for _, t in per_step)
    value = cells / sec / 1e9
    line = {"metric": "GCUPS", "value": value, "unit": "GCUPS", "n_gpus": args.gpus,
            "steps": args.steps, "warmup": args.warmup, "ms_per_step": 1e3 * sec / args.steps,
            "higher_is_better": True, "scaling": "strong", "vs_baseline": None, "dtype": "int32",
            "data": "synthetic", "impl": "reference",
            "config": {"workload": args.config, "doc": w.meta["doc"],
                       "note": "oracle (plain C Gotoh, OpenMP over pairs) on host cores; each step a "
                               "bounded random sample of the workload's pairs"},
            "cpu_baseline": {"value": value, "unit": "GCUPS", "cores": cores, "kind": "oracle",
                             "sample": desc, "cpu_model": cpu_model()},
            "e2e": {"value": value, "unit": "GCUPS", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0},
            "context": PAPER_CONTEXT}
    print(json.dumps(line), flush=True)
    return 0


def load_traffic():
    """DRAM bytes per cell of the K1 launch captured with ncu --set full (profiles/)."""
    p = os.path.join(ROOT, "profiles", "ncu_k1_summary.json")
    try:
        with open(p) as f:
            d = json.load(f)
        if d.get("cells"):
            return d["dram_bytes_per_launch"] / d["cells"], d
        return None, d
    except Exception:
        return None, None


def emulated_scaling(args, w, kw, local, flush_l2):
    """N emulated GPUs on one B200 (no multi-GPU node in this pool): N workers, each on its own
    green-context SM partition (sw_opts.worker_sms), the same workload; one device-timed search
    per N (libsw's CUDA events); the scores of every N must equal N = 1's."""
    import torch
    from paper_conf_ipps_mendoncam13_b200 import Database
    nsm_all = torch.cuda.get_device_properties(local).multi_processor_count
    sms = nsm_all // 8
    rows, ref_digest = [], None
    for n in [int(x) for x in args.emulated_scaling.split(",") if x]:
        De = Database(w.db, devices=[local] * n)
        flush_l2()
        r = De.search(w.queries, top_k=args.top_k, worker_sms=sms, **kw)
        dg = hashlib.sha256(np.ascontiguousarray(r.scores, dtype="<i4").tobytes()).hexdigest()
        ref_digest = ref_digest or dg
        rows.append({"n": n, "gcups": r.stats["gcups"], "seconds": r.stats["seconds_device"],
                     "partition_mode": r.stats["partition_mode"], "partition_sms": r.stats["partition_sms"],
                     "tail_s": r.stats["tail_seconds"], "peer_bytes": r.stats["peer_bytes"],
                     "scores_equal_n1": dg == ref_digest})
        De.close()
    g1 = next((x["gcups"] for x in rows if x["n"] == 1), None)
    for x in rows:
        x["efficiency"] = x["gcups"] / (x["n"] * g1) if g1 else None
    emulated = {"rows": rows, "kind": "strong scaling, N emulated GPUs on one B200",
                "note": "each worker on a disjoint green-context SM partition (partition_mode 2; its kernels "
                        "cannot leave its partition_sms SMs; L2/HBM shared); PSS + WA, in-process data "
                        "plane; efficiency = GCUPS(N) / (N x GCUPS(1))"}
    return emulated


def emulated_wa(args, w, kw, local, flush_l2):
    """BASELINE config 4's "8xB200 with workload adjustment on vs off" on one B200: args.emulated_wa
    workers on disjoint green-context SM partitions; the last one is a non-dedicated GPU (a
    co-running load kernel holds all but ceil(SMs / 6) of its SMs, the paper's superpi run,
    P24 §V.C).  PSS, the default units; device-timed makespan, tail (last completion - median
    worker's last completion), duplicated cells; scores identical in every run."""
    import torch
    from paper_conf_ipps_mendoncam13_b200 import Database
    n = args.emulated_wa
    sms = torch.cuda.get_device_properties(local).multi_processor_count // n
    D = Database(w.db, devices=[local] * n)
    base = {k: v for k, v in kw.items() if k not in ("workload_adjust", "straggler_mask")}
    rows, ref = [], None
    try:
        D.search(w.queries, top_k=args.top_k, worker_sms=sms, **base)   # warm-up
        for scen, mask in (("homogeneous", 0), ("loaded_gpu", 1 << (n - 1))):
            for wa in (False, True):
                flush_l2()
                r = D.search(w.queries, top_k=args.top_k, worker_sms=sms, workload_adjust=wa, straggler_mask=mask,
                             straggler_slowdown=6, straggler_mode="noise", **base)
                dg = hashlib.sha256(np.ascontiguousarray(r.scores, dtype="<i4").tobytes()).hexdigest()
                ref = ref or dg
                st = r.stats
                rows.append({"scenario": scen, "wa": wa, "gcups": st["gcups"], "makespan_s": st["seconds_device"],
                             "tail_s": st["tail_seconds"], "duplicated_cells": st["duplicated_cells"],
                             "wa_grants": st["n_wa_grants"], "cancelled": st["n_cancelled"],
                             "partition_mode": st["partition_mode"], "partition_sms": st["partition_sms"],
                             "scores_equal": dg == ref})
    finally:
        D.close()
    gain = {}
    for scen in ("homogeneous", "loaded_gpu"):
        off = next(x for x in rows if x["scenario"] == scen and not x["wa"])
        on = next(x for x in rows if x["scenario"] == scen and x["wa"])
        gain[scen] = {"gcups_gain_pct": 100.0 * (on["gcups"] / off["gcups"] - 1.0),
                      "tail_off_s": off["tail_s"], "tail_on_s": on["tail_s"]}
    return {"gpus": n, "rows": rows, "wa_gain": gain,
            "note": "N emulated GPUs (green-context SM partitions) on one B200; 'loaded_gpu': a local-load kernel "
                    "holds all but ceil(SMs/6) SMs of the last GPU from the start; PSS, default units"}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C4")
    ap.add_argument("--n-db", type=int, default=None, help="scale the DB down (debug only)")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--e2e-steps", type=int, default=2)
    ap.add_argument("--cpu-seconds", type=float, default=15.0)
    ap.add_argument("--ref-seconds", type=float, default=12.0)
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--emulated-wa", type=int, default=8,
                    help="N=1 runs only: WA on vs off on this many emulated GPUs (green SM partitions), "
                         "homogeneous and with a co-running load kernel on the last one; 0 = skip")
    ap.add_argument("--emulated-scaling", default="1,2,4,8",
                    help="N=1 runs only: N emulated GPUs on disjoint green-context SM partitions of "
                         "n_SM // 8 SMs (rounded to 8) for each listed N, one device-timed search each; "
                         "'' = skip")
    ap.add_argument("--policy", default="pss")
    ap.add_argument("--no-wa", action="store_true")
    ap.add_argument("--straggler-mask", type=int, default=0)
    ap.add_argument("--streams", type=int, default=4)
    ap.add_argument("--unit-cells", type=int, default=0)
    ap.add_argument("--top-k", type=int, default=10)
    ap.add_argument("--trace", default=None,
                    help="write the last timed step's unit log as a Chrome trace (JSON) to this path")
    ap.add_argument("--long-threshold", type=int, default=0,
                    help="DB length routed to the intra-task kernel K3 (0 = libsw's auto)")
    args = ap.parse_args()
    if args.impl == "reference":
        return reference_arm(args)

    import torch
    from paper_conf_ipps_mendoncam13_b200 import Database
    from paper_conf_ipps_mendoncam13_b200 import dist as swdist

    rank, world, local = env_rank()
    # SW_BENCH_ONE_GPU=1: every rank on cuda:0 with a gloo merge (validates the multi-process
    # path on a one-GPU box; NCCL refuses two ranks on one device)
    one_gpu = os.environ.get("SW_BENCH_ONE_GPU") == "1"
    if one_gpu:
        local = 0
    torch.cuda.set_device(local)
    if world > 1:
        import torch.distributed as tdist
        if one_gpu:
            tdist.init_process_group("gloo")
        else:
            tdist.init_process_group("nccl", device_id=torch.device("cuda", local))

    t = time.perf_counter()
    w = seqgen.make_workload(args.config, n_db=args.n_db)
    gen_s = time.perf_counter() - t
    t = time.perf_counter()
    D = Database(w.db, devices=[local])
    db_create_s = time.perf_counter() - t
    cells = int(w.meta["cells"])
    kw = dict(policy=args.policy, workload_adjust=not args.no_wa, streams=args.streams,
              target_unit_cells=args.unit_cells, straggler_mask=args.straggler_mask,
              long_threshold=args.long_threshold)

    def step():
        if world > 1:
            tdist.barrier()
            torch.cuda.synchronize()
            _, _, _, st = swdist.search(D, w.queries, rank, world, top_k=args.top_k, **kw)
            # libsw device time (common start after every slave registered) + the merge and
            # top-k on torch's stream (CUDA events)
            return st["seconds_device"] + st["merge_seconds"], st
        r = D.search(w.queries, top_k=args.top_k, outputs_on_device=True, **kw)
        return r.stats["seconds_device"], r.stats

    # L2 (126 MB): the C4 packed DB (196 MB) exceeds it; smaller databases are flushed
    # before every timed step by writing a 512 MB buffer (outside libsw's timed span)
    db_bytes = int(w.db.total)
    flush = None if db_bytes > 126_000_000 else torch.empty(512 << 20, dtype=torch.uint8, device="cuda")

    def flush_l2():
        if flush is not None:
            flush.fill_(1)
            torch.cuda.synchronize()

    for _ in range(args.warmup):
        step()
    if world > 1:
        tdist.barrier()
    torch.cuda.synchronize()
    sampler = ClockSampler(local)
    sampler.start()
    time.sleep(0.3)
    dev_s, launches, wall0 = 0.0, 0, time.perf_counter()
    stats = []
    for _ in range(args.steps):
        flush_l2()
        sec, st = step()
        dev_s += sec
        launches += st["kernel_launches"]
        stats.append(st)
    wall = time.perf_counter() - wall0
    clocks = sampler.stop()
    if args.trace and rank == 0:
        from paper_conf_ipps_mendoncam13_b200 import chrome_trace
        with open(args.trace, "w") as f:
            json.dump(chrome_trace(stats[-1].get("unit_log", []), name=f"{args.config} step"), f)
    if world > 1:
        tt = torch.tensor([dev_s], device="cuda", dtype=torch.float64)
        tdist.all_reduce(tt, op=tdist.ReduceOp.MAX)
        dev_s = float(tt.item())
    value = cells * args.steps / dev_s / 1e9
    ms = 1e3 * dev_s / args.steps

    # ---- e2e: host buffers through the C-ABI (queries H2D, scores + hits D2H, pinned).
    # N > 1: every rank reads back its own committed slice (disjoint), rank 0 the merged hits
    e2e = None
    nq, nd = w.queries.n, w.db.n
    h2d = int(w.queries.total + 8 * (nq + 1) + 576)
    d2h = int(4 * nq * nd + 8 * nq * args.top_k)
    if args.e2e_steps > 0:
        pin_s = torch.empty((nq, nd), dtype=torch.int32, pin_memory=True)
        pin_h = torch.empty((nq, args.top_k, 2), dtype=torch.int32, pin_memory=True)
        tsum = 0.0
        for k in range(args.e2e_steps + 1):
            if world > 1:
                tdist.barrier()
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            if world > 1:
                sc, hs, hi, _ = swdist.search(D, w.queries, rank, world, top_k=args.top_k, **kw)
                pin_s.copy_(sc, non_blocking=True)
                if rank == 0:
                    pin_h[..., 0].copy_(hs, non_blocking=True)
                    pin_h[..., 1].copy_(hi, non_blocking=True)
                torch.cuda.synchronize()
            else:
                D.search(w.queries, top_k=args.top_k, out_scores=pin_s, out_hits=pin_h, **kw)
            dt = time.perf_counter() - t0
            if k > 0:
                tsum += dt
        if world > 1:
            tt = torch.tensor([tsum], device="cuda", dtype=torch.float64)
            tdist.all_reduce(tt, op=tdist.ReduceOp.MAX)
            tsum = float(tt.item())
        e2e = {"value": cells * args.e2e_steps / tsum / 1e9, "unit": "GCUPS",
               "h2d_bytes_per_step": h2d, "d2h_bytes_per_step": d2h,
               "note": ("sw_search with host queries and pinned host outputs (scores + hits), host "
                        "clock around the call; packed DB resident (created once, db_create_s)"
                        + ("; per rank: its committed score slice + (rank 0) the merged hits, max over "
                           "ranks" if world > 1 else ""))}

    # ---- roofline of the dominant kernel (K1, integer/DPX pipe bound), rank 0 at every N:
    # one local search with a single stream, so every inter-task (K1) launch runs by itself;
    # achieved = K1 cells per launch / average K1 launch duration (CUDA events around each
    # launch on its stream, inside libsw)
    last = stats[-1]
    sm_mhz = clocks["sm_mhz"] or 1965.0
    nsm = torch.cuda.get_device_properties(local).multi_processor_count
    peak = nsm * sm_mhz * 1e6 * DPX_RATE / DPX_PER_CELL / 1e9
    peak_max = nsm * 1965e6 * DPX_RATE / DPX_PER_CELL / 1e9
    peak_form = nsm * sm_mhz * 1e6 * DPX_RATE / DPX_FORMULATION / 1e9
    per_gpu = value / world
    roofline = cpu = None
    if rank == 0:
        flush_l2()
        alone = D.search(w.queries, top_k=args.top_k, outputs_on_device=True, streams=1,
                         **{k: v for k, v in kw.items() if k != "streams"}).stats
        k1_launches = sum(1 for e in alone.get("unit_log", []) if e["kind"] == 0)
        k1_alone = (alone["cells_k1"] / alone["kernel_seconds_k1"] / 1e9) if alone["kernel_seconds_k1"] > 0 else None
        k3_alone = (alone["cells_k3"] / alone["kernel_seconds_k3"] / 1e9) if alone["kernel_seconds_k3"] > 0 else None
        bytes_per_cell, ncu = load_traffic()
        cells_per_launch = alone["cells_k1"] / k1_launches if k1_launches else None
        traffic = (bytes_per_cell * cells_per_launch) if (bytes_per_cell and cells_per_launch) else None
        # the dominant kernel: K1 unless long sequences carry most cells (C5: K3)
        k3_dominant = alone["cells_k3"] > alone["cells_k1"]
        dom = k3_alone if k3_dominant else k1_alone
        if k3_dominant:
            traffic = None   # the committed ncu capture is of K1
        roofline = {"bound": "alu", "achieved": dom, "peak": peak, "unit": "GCUPS",
                    "frac": (dom / peak) if dom else None, "traffic": traffic,
                    "kernel": ("k3_kernel (intra-task DP, the dominant kernel for this workload)" if k3_dominant else
                               "k1_kernel (inter-task DP, the dominant kernel)") +
                              ": cells per launch / average launch duration, each launch alone on the GPU (1 stream)",
                    "k1_alone_gcups": k1_alone,
                    "k1_launches": k1_launches, "k1_cells_per_launch": cells_per_launch,
                    "k1_avg_launch_ms": (1e3 * alone["kernel_seconds_k1"] / k1_launches) if k1_launches else None,
                    "k3_alone_gcups": k3_alone,
                    "k3_alone_note": ("K3 units of this workload each run alone (1 stream): an occupancy figure "
                                      "when its long sequences are few (C4: a unit fills well under the 592 resident "
                                      "K3 slots); in the step K3 units overlap K1 units. Where K3 carries the work "
                                      "(C5) the step runs at ~6.06 TCUPS (DESIGN.md section 9)"),
                    "step_gcups_per_gpu": per_gpu, "step_frac": per_gpu / peak,
                    "peak_at_max_clock": peak_max,
                    "formulation_peak": peak_form,
                    "k1_frac_of_formulation": (k1_alone / peak_form) if k1_alone else None,
                    "microbench_ceiling": nsm * sm_mhz * 1e6 * MICROBENCH_CELLS_PER_CLK / 1e9,
                    "k1_frac_of_microbench": (k1_alone / (nsm * sm_mhz * 1e6 * MICROBENCH_CELLS_PER_CLK / 1e9))
                                             if k1_alone else None,
                    "step_frac_of_microbench": per_gpu / (nsm * sm_mhz * 1e6 * MICROBENCH_CELLS_PER_CLK / 1e9),
                    "step_frac_of_formulation": per_gpu / peak_form,
                    "derivation": f"{nsm} SMs x {sm_mhz:.0f} MHz (median under load) x {DPX_RATE:.0f} "
                                  f"DPX lane-ops/clk/SM (measured, tools/dpx_peak.cu) / "
                                  f"{DPX_PER_CELL:.0f} three-input DPX per cell (4 per s16x2 lane word); "
                                  f"formulation_peak uses the kernel's own {DPX_FORMULATION} ALU-pipe ops per "
                                  f"cell (4 DPX + 0.5 VIMNMX3 for the running maximum per s16x2 word)",
                    "traffic_note": "dram__bytes_read+write per K1 launch: bytes per cell of the ncu --set full "
                                    "capture (profiles/ncu_k1_summary.json) x the average cells per K1 launch",
                    "k1_cells_share": last["cells_k1"] / max(1, last["cells_k1"] + last["cells_k3"])}
        if not args.no_cpu_baseline:
            g, cores, desc, _, _ = oracle_rate(w, seconds_target=args.cpu_seconds)
            g1, _, desc1, _, _ = oracle_rate(w, seconds_target=3.0, seed=7, max_threads=1)
            cpu = {"value": g, "unit": "GCUPS", "cores": cores, "kind": "oracle", "sample": desc,
                   "single_core": {"value": g1, "sample": desc1}, "cpu_model": cpu_model()}

    # ---- emulated multi-GPU strong scaling (no multi-GPU node in this pool): N workers on
    # one B200, each on its own green-context SM partition (sw_opts.worker_sms), the same
    # workload; one device-timed search per N (libsw's CUDA events), scores of every N equal
    emulated = None
    if world == 1 and args.emulated_scaling:
        try:
            emulated = emulated_scaling(args, w, kw, local, flush_l2)
        except Exception as e:   # an experiment: never lose the bench line for it
            emulated = {"error": f"{type(e).__name__}: {e}"}

    wa_exp = None
    if world == 1 and args.emulated_wa > 1:
        try:
            wa_exp = emulated_wa(args, w, kw, local, flush_l2)
        except Exception as e:   # an experiment: never lose the bench line for it
            wa_exp = {"error": f"{type(e).__name__}: {e}"}

    if rank == 0:
        line = {"metric": "GCUPS", "value": value, "unit": "GCUPS", "n_gpus": world,
                "steps": args.steps, "warmup": args.warmup, "ms_per_step": ms,
                "higher_is_better": True, "scaling": "strong", "vs_baseline": None,
                "dtype": "s16x2 (int32 re-run)", "data": "synthetic",
                "config": {"workload": args.config, "doc": w.meta["doc"], "n_db": nd,
                           "n_queries": nq, "db_residues": int(w.db.total),
                           "cells_per_step": cells, "policy": args.policy,
                           "workload_adjust": not args.no_wa, "streams_per_gpu": args.streams,
                           "top_k": args.top_k,
                           "l2": (f"inputs larger than L2 (packed DB {db_bytes / 1e6:.0f} MB > 126 MB); no flush"
                                  if flush is None else
                                  f"packed DB {db_bytes / 1e6:.0f} MB < L2: 512 MB buffer written before each step"),
                           "units_per_step": last["n_units"],
                           "overflow_pairs": last["n_overflow_pairs"],
                           "wa_grants": last["n_wa_grants"],
                           "wa_cancelled": last["n_cancelled"],
                           "request_messages": last["n_requests"],
                           "data_plane": ({"hits_allgather_bytes_per_rank": last.get("gather_bytes", 0),
                                           "scores": "rank-local committed slices (no collective)"}
                                          if world > 1 else {"peer_bytes": last["peer_bytes"]}),
                           "db_create_s": db_create_s, "generate_s": gen_s,
                           "wall_s_timed": wall, "parallelism": f"dp{world} (PSS/WA units)"},
                "gpu_launches": launches, "clocks": clocks, "e2e": e2e, "roofline": roofline,
                "cpu_baseline": cpu, "emulated_scaling": emulated, "emulated_wa": wa_exp,
                "context": PAPER_CONTEXT}
        print(json.dumps(line), flush=True)
    if world > 1:
        tdist.barrier()
        tdist.destroy_process_group()
    D.close()
    return 0


if __name__ == "__main__":
    sys.exit(main())
