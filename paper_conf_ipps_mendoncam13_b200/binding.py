"""Thin ctypes binding of libsw (include/sw.h, include/sw_sched.h).

Argument marshalling only: every step of the search runs in libsw's kernels and host
runtime.  There is no CPU fallback; if libsw.so cannot be loaded this module raises.
PyTorch is used (optionally) only for device buffers when outputs stay on the GPU.
"""
from __future__ import annotations

import ctypes
import json
import os
from dataclasses import dataclass

import numpy as np

from . import _build

# several workers' streams on one GPU exceed CUDA's default 8 hardware work queues and would
# falsely serialize; must be set before the process creates its CUDA context
os.environ.setdefault("CUDA_DEVICE_MAX_CONNECTIONS", "32")

_lib = None

SW_OK, SW_EINVAL, SW_ERESIDUE, SW_ENOMEM, SW_ECUDA, SW_ENET, SW_EBUSY = 0, -1, -2, -3, -4, -5, -6
SW_POLICY_SS, SW_POLICY_PSS = 0, 1
SW_TASK_READY, SW_TASK_EXECUTING, SW_TASK_FINISHED = 0, 1, 2
SW_STRAGGLER_HOLD, SW_STRAGGLER_SM_CAP, SW_STRAGGLER_NOISE = 0, 1, 2
_STRAGGLER_MODES = {"hold": SW_STRAGGLER_HOLD, "sm_cap": SW_STRAGGLER_SM_CAP, "noise": SW_STRAGGLER_NOISE}
SW_MAX_TOP_K, SW_MAX_QUERY_LEN = 64, 65535


class SwError(RuntimeError):
    def __init__(self, code, msg):
        super().__init__(f"libsw error {code}: {msg}")
        self.code = code


class sw_seqset(ctypes.Structure):
    _fields_ = [("n", ctypes.c_int32), ("offsets", ctypes.POINTER(ctypes.c_int64)),
                ("residues", ctypes.c_void_p), ("max_len", ctypes.c_int32)]


class sw_opts(ctypes.Structure):
    _fields_ = [("policy", ctypes.c_int32), ("workload_adjust", ctypes.c_int32),
                ("omega", ctypes.c_int32), ("streams_per_device", ctypes.c_int32),
                ("target_unit_cells", ctypes.c_int64), ("long_threshold", ctypes.c_int32),
                ("outputs_on_device", ctypes.c_int32), ("straggler_mask", ctypes.c_uint64),
                ("straggler_slowdown", ctypes.c_int32), ("dist_rank", ctypes.c_int32),
                ("dist_world", ctypes.c_int32), ("dist_port", ctypes.c_int32),
                ("dist_host", ctypes.c_char_p), ("straggler_after_ms", ctypes.c_int32),
                ("straggler_mode", ctypes.c_int32), ("worker_sms", ctypes.c_int32),
                ("reserved", ctypes.c_int32 * 5)]


class sw_alignment(ctypes.Structure):
    _fields_ = [("score", ctypes.c_int32), ("q_begin", ctypes.c_int32), ("q_end", ctypes.c_int32),
                ("d_begin", ctypes.c_int32), ("d_end", ctypes.c_int32), ("n_ops", ctypes.c_int32),
                ("ops_offset", ctypes.c_int64)]


class sw_stats(ctypes.Structure):
    _fields_ = [("cells", ctypes.c_int64), ("seconds_device", ctypes.c_double),
                ("seconds_wall", ctypes.c_double), ("gcups", ctypes.c_double),
                ("duplicated_cells", ctypes.c_int64), ("n_units", ctypes.c_int32),
                ("n_overflow_pairs", ctypes.c_int32), ("n_wa_grants", ctypes.c_int32),
                ("n_requests", ctypes.c_int32), ("kernel_launches", ctypes.c_int32),
                ("n_devices", ctypes.c_int32), ("kernel_seconds_k1", ctypes.c_double),
                ("kernel_seconds_k3", ctypes.c_double), ("cells_k1", ctypes.c_int64),
                ("cells_k3", ctypes.c_int64), ("tail_seconds", ctypes.c_double),
                ("unit_log_json", ctypes.c_char_p), ("n_grant_messages", ctypes.c_int32),
                ("n_cancelled", ctypes.c_int32), ("seconds_last_unit", ctypes.c_double),
                ("peer_bytes", ctypes.c_int64), ("sched_log_json", ctypes.c_char_p),
                ("kernel_seconds_k2", ctypes.c_double), ("n_k2_launches", ctypes.c_int32),
                ("partition_mode", ctypes.c_int32), ("partition_sms", ctypes.c_int32)]


# every symbol include/*.h declares (tests check the library exports all of them)
EXPORTS = ["sw_opts_default", "sw_db_create", "sw_db_destroy", "sw_db_residues", "sw_db_size",
           "sw_db_devices", "sw_search", "sw_topk_device", "sw_merge_hits", "sw_last_error", "sw_version",
           "sw_sched_create", "sw_sched_destroy", "sw_sched_report", "sw_sched_request",
           "sw_sched_request_wait", "sw_sched_complete", "sw_sched_abandon", "sw_sched_fail_worker",
           "sw_sched_start", "sw_sched_is_finished", "sw_sched_state",
           "sw_sched_committed_by", "sw_sched_replicas", "sw_sched_phi", "sw_sched_rate",
           "sw_sched_counter", "sw_sched_log_json", "sw_master_start", "sw_master_stop",
           "sw_slave_connect", "sw_slave_request", "sw_slave_request_wait", "sw_slave_report",
           "sw_slave_complete", "sw_slave_abandon", "sw_slave_start", "sw_slave_is_finished",
           "sw_slave_done", "sw_slave_counter", "sw_align"]


def lib():
    """Load libsw.so (building it in-tree first if it is missing or stale)."""
    global _lib
    if _lib is not None:
        return _lib
    checked = os.environ.get("SW_CHECKED") == "1"   # the bounds-asserting build (tests)
    path = _build.LIB_CHECKED if checked else _build.LIB
    try:
        if _build._stale(checked):
            _build.build(checked=checked)
    except Exception as e:  # nvcc missing etc.: only fatal if there is no library at all
        if not os.path.exists(path):
            raise ImportError(f"libsw.so is missing and could not be built: {e}") from e
    if not os.path.exists(path):
        raise ImportError(f"libsw.so not found at {path}")
    L = ctypes.CDLL(path)
    P = ctypes.POINTER
    L.sw_opts_default.argtypes = [P(sw_opts)]
    L.sw_db_create.argtypes = [P(sw_seqset), P(ctypes.c_int), ctypes.c_int, P(ctypes.c_void_p)]
    L.sw_db_create.restype = ctypes.c_int
    L.sw_db_destroy.argtypes = [ctypes.c_void_p]
    L.sw_db_residues.argtypes = [ctypes.c_void_p]
    L.sw_db_residues.restype = ctypes.c_int64
    L.sw_db_size.argtypes = [ctypes.c_void_p]
    L.sw_db_size.restype = ctypes.c_int32
    L.sw_db_devices.argtypes = [ctypes.c_void_p]
    L.sw_db_devices.restype = ctypes.c_int32
    L.sw_search.argtypes = [P(sw_seqset), ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                            ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p, ctypes.c_void_p,
                            P(sw_opts), P(sw_stats)]
    L.sw_search.restype = ctypes.c_int
    L.sw_topk_device.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                 ctypes.c_int32, ctypes.c_void_p]
    L.sw_topk_device.restype = ctypes.c_int
    L.sw_merge_hits.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32,
                                ctypes.c_int32, ctypes.c_int32, ctypes.c_void_p]
    L.sw_merge_hits.restype = ctypes.c_int
    L.sw_last_error.restype = ctypes.c_char_p
    L.sw_version.restype = ctypes.c_char_p
    L.sw_sched_create.argtypes = [ctypes.c_int32, ctypes.c_int32, P(ctypes.c_int64), ctypes.c_int32,
                                  ctypes.c_int32, ctypes.c_int32]
    L.sw_sched_create.restype = ctypes.c_void_p
    L.sw_sched_destroy.argtypes = [ctypes.c_void_p]
    L.sw_sched_report.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_double, ctypes.c_double,
                                  ctypes.c_double]
    L.sw_sched_request.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_double,
                                   P(ctypes.c_int32), ctypes.c_int32]
    L.sw_sched_request.restype = ctypes.c_int32
    L.sw_sched_request_wait.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_double,
                                        P(ctypes.c_int32), ctypes.c_int32, ctypes.c_double]
    L.sw_sched_request_wait.restype = ctypes.c_int32
    L.sw_sched_fail_worker.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_double]
    L.sw_sched_complete.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double]
    L.sw_sched_complete.restype = ctypes.c_int32
    L.sw_sched_abandon.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double]
    L.sw_sched_start.argtypes = [ctypes.c_void_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double]
    L.sw_sched_start.restype = ctypes.c_int32
    for name in ("sw_sched_is_finished", "sw_sched_state", "sw_sched_committed_by",
                 "sw_sched_replicas"):
        getattr(L, name).argtypes = [ctypes.c_void_p, ctypes.c_int32]
        getattr(L, name).restype = ctypes.c_int32
    L.sw_sched_phi.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_sched_phi.restype = ctypes.c_int32
    L.sw_sched_rate.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_sched_rate.restype = ctypes.c_double
    L.sw_sched_counter.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_sched_counter.restype = ctypes.c_int64
    L.sw_sched_log_json.argtypes = [ctypes.c_void_p]
    L.sw_sched_log_json.restype = ctypes.c_char_p
    L.sw_master_start.argtypes = [ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, P(ctypes.c_int64),
                                  ctypes.c_int32, ctypes.c_int32, ctypes.c_int32, ctypes.c_uint64]
    L.sw_master_start.restype = ctypes.c_void_p
    L.sw_master_stop.argtypes = [ctypes.c_void_p]
    L.sw_slave_connect.argtypes = [ctypes.c_char_p, ctypes.c_int32, ctypes.c_int32, ctypes.c_double,
                                   ctypes.c_uint64]
    L.sw_slave_connect.restype = ctypes.c_void_p
    L.sw_slave_request.argtypes = [ctypes.c_void_p, P(ctypes.c_int32), ctypes.c_int32]
    L.sw_slave_request.restype = ctypes.c_int32
    L.sw_slave_request_wait.argtypes = [ctypes.c_void_p, P(ctypes.c_int32), ctypes.c_int32, ctypes.c_double]
    L.sw_slave_request_wait.restype = ctypes.c_int32
    L.sw_slave_counter.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_slave_counter.restype = ctypes.c_int64
    L.sw_slave_report.argtypes = [ctypes.c_void_p, ctypes.c_double, ctypes.c_double]
    L.sw_slave_complete.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_slave_complete.restype = ctypes.c_int32
    L.sw_slave_abandon.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_slave_start.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_slave_start.restype = ctypes.c_int32
    L.sw_slave_is_finished.argtypes = [ctypes.c_void_p, ctypes.c_int32]
    L.sw_slave_is_finished.restype = ctypes.c_int32
    L.sw_slave_done.argtypes = [ctypes.c_void_p]
    L.sw_align.argtypes = [P(sw_seqset), ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int32,
                           ctypes.c_int32, P(ctypes.c_int32), P(ctypes.c_int32), ctypes.c_int32,
                           P(sw_alignment), ctypes.c_char_p, ctypes.c_int64]
    L.sw_align.restype = ctypes.c_int
    _lib = L
    return L


def _check(rc):
    if rc != SW_OK:
        raise SwError(rc, lib().sw_last_error().decode(errors="replace"))


def _seqset(s, keep):
    off = np.ascontiguousarray(s.offsets, dtype=np.int64)
    res = np.ascontiguousarray(s.residues, dtype=np.uint8)
    keep += [off, res]
    return sw_seqset(int(s.n), off.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                     res.ctypes.data if res.size else None, 0)


@dataclass
class SearchResult:
    scores: object          # [nq, ndb] int32 (numpy, or torch on device), or None
    hit_scores: object      # [nq, k]
    hit_index: object       # [nq, k] (-1 = empty)
    stats: dict


def grant_timeline(sched_log):
    """The master's grants (sched_log of a search) with times relative to the first event:
    [{"t_rel", "worker", "unit", "phi", "rate", "wa"}] -- the per-interaction marks of the
    paper's Figs. 7/8 (package weight Φ and mean rate v̄ of the requesting PE)."""
    if not sched_log:
        return []
    t0 = min(e["t"] for e in sched_log)
    return [dict(t_rel=e["t"] - t0, worker=e["worker"], unit=e["unit"], phi=e.get("phi", 0),
                 rate=e.get("rate", 0.0), wa=e["ev"] == "W", ev=e["ev"])
            for e in sched_log if e["ev"] in ("G", "W")]


def chrome_trace(unit_log, name="sw_search", sched_log=None) -> dict:
    """The per-unit event log of a search (stats["unit_log"]) as a Chrome-trace / Perfetto
    JSON object (SURVEY §5 tracing): one process per worker (GPU), one thread per stream, a
    complete event per unit replica (host clock from launch to observed completion; args:
    cells, device_ms, committed, pack) and an instant event at each grant on a "master"
    thread -- the analogue of the paper's per-interaction marks (P24 Figs. 7/8)."""
    ev = []
    sched_log = grant_timeline(sched_log) if sched_log and "t_rel" not in sched_log[0] else sched_log
    workers = sorted({e["worker"] for e in unit_log})
    for w in workers:
        ev.append({"ph": "M", "name": "process_name", "pid": w, "args": {"name": f"{name}: worker {w}"}})
        ev.append({"ph": "M", "name": "thread_name", "pid": w, "tid": -1, "args": {"name": "master grants"}})
    for e in unit_log:
        kind = "K1 inter-task" if e["kind"] == 0 else "K3 intra-task"
        tag = " cancelled" if e.get("cancelled") else (" lost" if not e["committed"] else "")
        ev.append({"ph": "X", "name": f"unit {e['unit']} ({kind}){tag}", "cat": "unit",
                   "pid": e["worker"], "tid": e.get("stream", 0),
                   "ts": 1e6 * e["t_start"], "dur": max(0.0, 1e6 * (e["t_end"] - e["t_start"])),
                   "args": {"cells": e["cells"], "cells_done": e.get("cells_done", e["cells"]),
                            "pack": e["pair"], "committed": e["committed"],
                            "cancelled": e.get("cancelled", 0), "slowed": e.get("slowed", 0),
                            "device_ms": e.get("device_ms"), "dev_t0_ms": e.get("dev_t0"),
                            "dev_t1_ms": e.get("dev_t1")}})
        ev.append({"ph": "i", "name": f"grant unit {e['unit']}", "cat": "grant", "s": "t",
                   "pid": e["worker"], "tid": -1, "ts": 1e6 * e["t_grant"]})
    for g in sched_log or []:
        if g.get("ev") in ("G", "W"):   # Φ and v̄ of the requesting worker at each grant
            ev.append({"ph": "C", "name": "PSS package weight phi", "pid": g["worker"],
                       "ts": 1e6 * g["t_rel"], "args": {"phi": g.get("phi", 0)}})
            ev.append({"ph": "C", "name": "rate v (GCUPS)", "pid": g["worker"],
                       "ts": 1e6 * g["t_rel"], "args": {"v": 1e-9 * g.get("rate", 0.0)}})
    return {"traceEvents": ev, "displayTimeUnit": "ms"}


def _stats_dict(st: sw_stats) -> dict:
    d = {k: getattr(st, k) for k, _ in sw_stats._fields_ if k not in ("unit_log_json", "sched_log_json")}
    d["unit_log"] = json.loads(st.unit_log_json.decode()) if st.unit_log_json else []
    d["sched_log"] = json.loads(st.sched_log_json.decode()) if st.sched_log_json else []
    return d


class Database:
    """A packed database replicated on one or more GPUs (sw_db_create)."""

    def __init__(self, db, devices=None):
        keep = []
        ss = _seqset(db, keep)
        h = ctypes.c_void_p()
        if devices:
            arr = (ctypes.c_int * len(devices))(*devices)
            _check(lib().sw_db_create(ctypes.byref(ss), arr, len(devices), ctypes.byref(h)))
        else:
            _check(lib().sw_db_create(ctypes.byref(ss), None, 0, ctypes.byref(h)))
        self._h = h
        self.n = db.n
        self.lengths = np.diff(np.asarray(db.offsets)).astype(np.int64)
        self.devices = list(devices) if devices else [0]

    def close(self):
        if getattr(self, "_h", None):
            lib().sw_db_destroy(self._h)
            self._h = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    @property
    def residues(self) -> int:
        return int(lib().sw_db_residues(self._h))

    def search(self, queries, matrix=None, gap_open=10, gap_extend=2, top_k=10, want_scores=True,
               policy="pss", workload_adjust=True, omega=4, streams=4, target_unit_cells=0,
               long_threshold=0, outputs_on_device=False, straggler_mask=0, straggler_slowdown=6,
               straggler_after_ms=0, straggler_mode="sm_cap", worker_sms=0, dist=None, out_scores=None,
               out_hits=None) -> SearchResult:
        """sw_search.  Host outputs are numpy arrays (pinned buffers may be passed via
        out_scores / out_hits); with outputs_on_device the outputs are torch CUDA tensors.
        straggler_mode: "sm_cap" (GPU-side, default), "noise" (GPU-side local load) or
        "hold" (host-side) -- see SW_STRAGGLER_* in include/sw.h."""
        keep = []
        qs = _seqset(queries, keep)
        nq, nd = int(queries.n), int(self.n)
        o = sw_opts()
        lib().sw_opts_default(ctypes.byref(o))
        o.policy = SW_POLICY_SS if policy == "ss" else SW_POLICY_PSS
        o.workload_adjust = int(bool(workload_adjust))
        o.omega = omega
        o.streams_per_device = streams
        o.target_unit_cells = target_unit_cells
        o.long_threshold = long_threshold
        o.outputs_on_device = int(bool(outputs_on_device))
        o.straggler_mask = straggler_mask
        o.straggler_slowdown = straggler_slowdown
        o.straggler_after_ms = straggler_after_ms
        o.straggler_mode = _STRAGGLER_MODES[straggler_mode]
        o.worker_sms = worker_sms
        if dist is not None:
            o.dist_rank, o.dist_world, o.dist_port = dist["rank"], dist["world"], dist["port"]
            host = dist.get("host", "127.0.0.1").encode()
            keep.append(host)
            o.dist_host = host
        mat = None
        if matrix is not None:
            mat = np.ascontiguousarray(np.asarray(matrix, dtype=np.int8).reshape(24, 24))
            keep.append(mat)
        if outputs_on_device:
            import torch
            dev = torch.device("cuda", self.devices[0])
            scores = out_scores if out_scores is not None else (
                torch.empty((nq, nd), dtype=torch.int32, device=dev) if want_scores else None)
            hits = out_hits if out_hits is not None else (
                torch.empty((nq, max(top_k, 0), 2), dtype=torch.int32, device=dev) if top_k > 0 else None)
            sp = scores.data_ptr() if scores is not None else None
            hp = hits.data_ptr() if hits is not None else None
        else:
            scores = out_scores if out_scores is not None else (
                np.empty((nq, nd), dtype=np.int32) if want_scores else None)
            hits = out_hits if out_hits is not None else (
                np.empty((nq, max(top_k, 0), 2), dtype=np.int32) if top_k > 0 else None)
            sp = _ptr(scores)
            hp = _ptr(hits)
        st = sw_stats()
        rc = lib().sw_search(ctypes.byref(qs), self._h, mat.ctypes.data if mat is not None else None,
                             gap_open, gap_extend, top_k, sp, hp, ctypes.byref(o), ctypes.byref(st))
        _check(rc)
        hs = hits[..., 0] if hits is not None else None
        hi = hits[..., 1] if hits is not None else None
        return SearchResult(scores, hs, hi, _stats_dict(st))

    def align(self, queries, query_index, db_index, matrix=None, gap_open=10, gap_extend=2):
        """Phase 2 (sw_align): the optimal local alignment of each (query, db) pair.
        Returns a list of dicts: score, q_begin, q_end, d_begin, d_end (0-based, end
        exclusive) and ops ('M' aligned pair, 'I' query residue vs gap, 'D' db residue vs gap)."""
        keep = []
        qs = _seqset(queries, keep)
        qi = np.ascontiguousarray(query_index, dtype=np.int32)
        di = np.ascontiguousarray(db_index, dtype=np.int32)
        n = len(qi)
        out = (sw_alignment * max(n, 1))()
        qlen = np.diff(np.asarray(queries.offsets))
        cap = int(qlen[qi].sum() + self.lengths[di].sum()) if n else 1
        buf = ctypes.create_string_buffer(max(cap, 1))
        mat = None
        if matrix is not None:
            mat = np.ascontiguousarray(np.asarray(matrix, dtype=np.int8).reshape(24, 24))
        _check(lib().sw_align(ctypes.byref(qs), self._h, mat.ctypes.data if mat is not None else None,
                              gap_open, gap_extend, qi.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)),
                              di.ctypes.data_as(ctypes.POINTER(ctypes.c_int32)), n, out, buf, cap))
        res = []
        raw = buf.raw
        for k in range(n):
            a = out[k]
            res.append(dict(score=a.score, q_begin=a.q_begin, q_end=a.q_end, d_begin=a.d_begin,
                            d_end=a.d_end, ops=raw[a.ops_offset:a.ops_offset + a.n_ops].decode()))
        return res

    def merge_hits(self, lists_dev, top_k):
        """sw_merge_hits: lists_dev is a torch CUDA int32 tensor [n_sources, nq, k_in, 2]
        (score, db_index); returns the merged (scores, index) [nq, top_k] on the device."""
        import torch
        n_src, nq, k_in, _ = lists_dev.shape
        lists_dev = lists_dev.contiguous()
        out = torch.empty((nq, top_k, 2), dtype=torch.int32, device=lists_dev.device)
        _check(lib().sw_merge_hits(self._h, lists_dev.data_ptr(), n_src, nq, k_in, top_k, out.data_ptr()))
        return out[..., 0], out[..., 1]

    def topk_device(self, scores_dev, top_k):
        """Top-k of a torch CUDA score matrix (entries < 0 ignored) -> (scores, index)."""
        import torch
        nq, nd = scores_dev.shape
        hits = torch.empty((nq, top_k, 2), dtype=torch.int32, device=scores_dev.device)
        _check(lib().sw_topk_device(self._h, scores_dev.data_ptr(), nq, nd, top_k, hits.data_ptr()))
        return hits[..., 0], hits[..., 1]


def _ptr(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags["C_CONTIGUOUS"]
        return a.ctypes.data
    return a.data_ptr()  # torch (pinned host) tensor


class Scheduler:
    """The master's task table (sw_sched_*), drivable with a simulated clock."""

    def __init__(self, n_workers, unit_cells, policy="pss", wa=True, omega=4):
        cells = np.ascontiguousarray(unit_cells, dtype=np.int64)
        self._cells = cells
        h = lib().sw_sched_create(n_workers, len(cells),
                                  cells.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                  SW_POLICY_SS if policy == "ss" else SW_POLICY_PSS, int(wa), omega)
        if not h:
            raise SwError(SW_EINVAL, "sw_sched_create failed")
        self._h = h

    def __del__(self):
        if getattr(self, "_h", None):
            lib().sw_sched_destroy(self._h)
            self._h = None

    def report(self, worker, now, cells, seconds):
        lib().sw_sched_report(self._h, worker, now, float(cells), float(seconds))

    def request(self, worker, now, cap=64):
        buf = (ctypes.c_int32 * cap)()
        n = lib().sw_sched_request(self._h, worker, now, buf, cap)
        if n < 0:
            return None  # every task finished
        return [buf[i] for i in range(n)]

    def request_wait(self, worker, now, timeout, cap=64):
        buf = (ctypes.c_int32 * cap)()
        n = lib().sw_sched_request_wait(self._h, worker, now, buf, cap, timeout)
        if n < 0:
            return None
        return [buf[i] for i in range(n)]

    def fail_worker(self, worker, now):
        lib().sw_sched_fail_worker(self._h, worker, now)

    def complete(self, worker, unit, now) -> bool:
        return bool(lib().sw_sched_complete(self._h, worker, unit, now))

    def abandon(self, worker, unit, now):
        lib().sw_sched_abandon(self._h, worker, unit, now)

    def start(self, worker, unit, now) -> bool:
        """Worker is about to execute `unit`: False if it is finished or was moved away."""
        return bool(lib().sw_sched_start(self._h, worker, unit, now))

    def is_finished(self, unit) -> bool:
        return bool(lib().sw_sched_is_finished(self._h, unit))

    def state(self, unit):
        return lib().sw_sched_state(self._h, unit)

    def committed_by(self, unit):
        return lib().sw_sched_committed_by(self._h, unit)

    def replicas(self, unit):
        return lib().sw_sched_replicas(self._h, unit)

    def phi(self, worker):
        return lib().sw_sched_phi(self._h, worker)

    def rate(self, worker):
        return lib().sw_sched_rate(self._h, worker)

    def counter(self, which):
        return lib().sw_sched_counter(self._h, which)

    def log(self):
        return json.loads(lib().sw_sched_log_json(self._h).decode())


class Master:
    """The multi-process master (sw_master_start): serves `world` slaves over TCP."""

    def __init__(self, port, world, unit_cells, policy="pss", wa=True, omega=4, plan_hash=0):
        cells = np.ascontiguousarray(unit_cells, dtype=np.int64)
        h = lib().sw_master_start(port, world, len(cells),
                                  cells.ctypes.data_as(ctypes.POINTER(ctypes.c_int64)),
                                  SW_POLICY_SS if policy == "ss" else SW_POLICY_PSS, int(wa), omega,
                                  plan_hash)
        if not h:
            raise SwError(SW_ENET, lib().sw_last_error().decode())
        self._h = h

    def stop(self):
        if self._h:
            lib().sw_master_stop(self._h)
            self._h = None


class Slave:
    """A slave's connection to the master (sw_slave_*)."""

    def __init__(self, host, port, rank, timeout=30.0, plan_hash=0):
        h = lib().sw_slave_connect(host.encode(), port, rank, timeout, plan_hash)
        if not h:
            raise SwError(SW_ENET, lib().sw_last_error().decode())
        self._h = h

    def request(self, cap=64):
        buf = (ctypes.c_int32 * cap)()
        n = lib().sw_slave_request(self._h, buf, cap)
        if n == -2:
            raise SwError(SW_ENET, lib().sw_last_error().decode())
        return None if n < 0 else [buf[i] for i in range(n)]

    def request_wait(self, timeout=0.05, cap=64):
        """One request that waits at the master (long poll) while nothing can be granted."""
        buf = (ctypes.c_int32 * cap)()
        n = lib().sw_slave_request_wait(self._h, buf, cap, timeout)
        if n == -2:
            raise SwError(SW_ENET, lib().sw_last_error().decode())
        return None if n < 0 else [buf[i] for i in range(n)]

    def counter(self, which):
        return lib().sw_slave_counter(self._h, which)

    def report(self, cells, seconds):
        lib().sw_slave_report(self._h, float(cells), float(seconds))

    def complete(self, unit) -> bool:
        return lib().sw_slave_complete(self._h, unit) == 1

    def abandon(self, unit):
        lib().sw_slave_abandon(self._h, unit)

    def start(self, unit) -> bool:
        rc = lib().sw_slave_start(self._h, unit)
        if rc < 0:
            raise SwError(SW_ENET, lib().sw_last_error().decode())
        return rc == 1

    def is_finished(self, unit) -> bool:
        return lib().sw_slave_is_finished(self._h, unit) == 1

    def done(self):
        if self._h:
            lib().sw_slave_done(self._h)
            self._h = None
