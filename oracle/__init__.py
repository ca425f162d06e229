"""ORACLE — plain CPU Smith-Waterman/Gotoh (TEST INFRASTRUCTURE ONLY).

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s ``cpu_baseline`` /
``--impl reference`` legs may import this package.  The product path
(``paper_conf_ipps_mendoncam13_b200``) never imports it and shares no code with it.

The arithmetic lives in ``sw_oracle.c`` (the definition of SURVEY §8(c), citing
PAPER.md P12 §II.A) and ``bruteforce.c`` (exhaustive enumeration, for pins).
This module only builds the C library, marshals arguments and, for top-k, applies
the definition "k best under (score desc, db_index asc)" (reading R13) with a
library sort.

Parity unpinned: nothing here is unpinned except what DESIGN.md §3 lists
(PSS weights for non-integer speed ratios live in the scheduler, not here).
"""
from __future__ import annotations

import ctypes
import os
import subprocess
import threading

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
_LIB_PATH = os.path.join(_HERE, "libsw_oracle.so")
_SOURCES = ["sw_oracle.c", "bruteforce.c"]
_lock = threading.Lock()
_lib = None

NEG_INF = -(1 << 29)
ALPHABET = "ARNDCQEGHILKMFPSTWYVBZX*"


def build(force: bool = False) -> str:
    """Compile liboracle with gcc -O2 -fopenmp (plain C; no SIMD intrinsics)."""
    srcs = [os.path.join(_HERE, s) for s in _SOURCES + ["sw_oracle.h"]]
    if not force and os.path.exists(_LIB_PATH):
        t = os.path.getmtime(_LIB_PATH)
        if all(os.path.getmtime(s) <= t for s in srcs):
            return _LIB_PATH
    cmd = ["gcc", "-O2", "-std=c11", "-fopenmp", "-fPIC", "-shared", "-o", _LIB_PATH + ".tmp"]
    cmd += [os.path.join(_HERE, s) for s in _SOURCES]
    subprocess.check_call(cmd)
    os.replace(_LIB_PATH + ".tmp", _LIB_PATH)
    return _LIB_PATH


def lib():
    global _lib
    with _lock:
        if _lib is None:
            build()
            L = ctypes.CDLL(_LIB_PATH)
            i8p = ctypes.POINTER(ctypes.c_int8)
            i32p = ctypes.POINTER(ctypes.c_int32)
            i64p = ctypes.POINTER(ctypes.c_int64)
            L.sw_oracle_code.argtypes = [ctypes.c_int]
            L.sw_oracle_code.restype = ctypes.c_int
            L.sw_oracle_blosum62.restype = i8p
            L.sw_oracle_pair.argtypes = [ctypes.c_char_p, ctypes.c_int64, ctypes.c_char_p,
                                         ctypes.c_int64, i8p, ctypes.c_int32, ctypes.c_int32,
                                         ctypes.c_int32]
            L.sw_oracle_pair.restype = ctypes.c_int32
            L.sw_oracle_dump.argtypes = [ctypes.c_char_p, ctypes.c_int64, ctypes.c_char_p,
                                         ctypes.c_int64, i8p, ctypes.c_int32, ctypes.c_int32,
                                         i32p, i32p, i32p]
            L.sw_oracle_dump.restype = ctypes.c_int32
            L.sw_oracle_search.argtypes = [ctypes.c_void_p, i64p, ctypes.c_int32, ctypes.c_void_p,
                                           i64p, ctypes.c_int32, i8p, ctypes.c_int32,
                                           ctypes.c_int32, i32p, ctypes.c_int]
            L.sw_oracle_search.restype = ctypes.c_int
            L.sw_oracle_pairs.argtypes = [ctypes.c_void_p, i64p, ctypes.c_void_p, i64p, i32p, i32p,
                                          ctypes.c_int64, i8p, ctypes.c_int32, ctypes.c_int32,
                                          i32p, ctypes.c_int]
            L.sw_oracle_pairs.restype = ctypes.c_int
            L.sw_bruteforce_pair.argtypes = [ctypes.c_char_p, ctypes.c_int, ctypes.c_char_p,
                                             ctypes.c_int, i8p, ctypes.c_int32, ctypes.c_int32]
            L.sw_bruteforce_pair.restype = ctypes.c_int32
            L.sw_alignment_score.argtypes = [ctypes.c_char_p, ctypes.c_char_p, ctypes.c_int64,
                                             i8p, ctypes.c_int32, ctypes.c_int32]
            L.sw_alignment_score.restype = ctypes.c_int32
            _lib = L
    return _lib


def _mat(matrix):
    if matrix is None:
        return None, None
    m = np.ascontiguousarray(np.asarray(matrix, dtype=np.int8).reshape(24, 24))
    return m, m.ctypes.data_as(ctypes.POINTER(ctypes.c_int8))


def _p(a, t):
    return a.ctypes.data_as(ctypes.POINTER(t))


def blosum62() -> np.ndarray:
    """The oracle's own transcription of BLOSUM62 (24x24, NCBI order)."""
    p = lib().sw_oracle_blosum62()
    return np.ctypeslib.as_array(p, shape=(24 * 24,)).reshape(24, 24).copy()


def code(ch: str) -> int:
    return lib().sw_oracle_code(ord(ch))


def pair_score(q, d, matrix=None, gap_open=10, gap_extend=2, border_init=NEG_INF) -> int:
    """Score of one pair (SURVEY §8(c) definition)."""
    qb = q.encode() if isinstance(q, str) else bytes(q)
    db = d.encode() if isinstance(d, str) else bytes(d)
    keep, mp = _mat(matrix)
    s = lib().sw_oracle_pair(qb, len(qb), db, len(db), mp, gap_open, gap_extend, border_init)
    if s < 0:
        raise ValueError("oracle: invalid residue or argument")
    return int(s)


def dump(q, d, matrix=None, gap_open=10, gap_extend=2):
    """Full H, E, F matrices ((m+1) x (n+1)) and the score, for tiny inputs."""
    qb, db = q.encode(), d.encode()
    m, n = len(qb), len(db)
    H = np.zeros((m + 1, n + 1), np.int32)
    E = np.zeros_like(H)
    F = np.zeros_like(H)
    keep, mp = _mat(matrix)
    s = lib().sw_oracle_dump(qb, m, db, n, mp, gap_open, gap_extend, _p(H, ctypes.c_int32),
                             _p(E, ctypes.c_int32), _p(F, ctypes.c_int32))
    if s < 0:
        raise ValueError("oracle: invalid residue or argument")
    return int(s), H, E, F


def bruteforce(q, d, matrix=None, gap_open=10, gap_extend=2) -> int:
    """Exhaustive maximum over all local alignments (len <= 8)."""
    qb, db = q.encode(), d.encode()
    keep, mp = _mat(matrix)
    s = lib().sw_bruteforce_pair(qb, len(qb), db, len(db), mp, gap_open, gap_extend)
    if s < 0:
        raise ValueError("bruteforce: invalid input")
    return int(s)


def alignment_score(row_q: str, row_d: str, matrix=None, gap_open=10, gap_extend=2) -> int:
    assert len(row_q) == len(row_d)
    keep, mp = _mat(matrix)
    s = lib().sw_alignment_score(row_q.encode(), row_d.encode(), len(row_q), mp, gap_open,
                                 gap_extend)
    if s == -(1 << 31):
        raise ValueError("alignment_score: invalid alignment")
    return int(s)


def search(queries, db, matrix=None, gap_open=10, gap_extend=2, n_threads=0) -> np.ndarray:
    """All-pairs scores [nq, nd] for two seqgen.SeqSet (the paper's indexed format)."""
    nq, nd = queries.n, db.n
    out = np.zeros((nq, nd), np.int32)
    if nq == 0 or nd == 0:
        return out
    keep, mp = _mat(matrix)
    qo = np.ascontiguousarray(queries.offsets, np.int64)
    do = np.ascontiguousarray(db.offsets, np.int64)
    qr = np.ascontiguousarray(queries.residues, np.uint8)
    dr = np.ascontiguousarray(db.residues, np.uint8)
    rc = lib().sw_oracle_search(qr.ctypes.data, _p(qo, ctypes.c_int64), nq, dr.ctypes.data,
                                _p(do, ctypes.c_int64), nd, mp, gap_open, gap_extend,
                                _p(out, ctypes.c_int32), n_threads)
    if rc != 0:
        raise ValueError("oracle: invalid residue or argument")
    return out


def pairs(queries, db, qi, di, matrix=None, gap_open=10, gap_extend=2, n_threads=0) -> np.ndarray:
    """Scores of selected (qi[k], di[k]) pairs."""
    qi = np.ascontiguousarray(qi, np.int32)
    di = np.ascontiguousarray(di, np.int32)
    out = np.zeros(len(qi), np.int32)
    if len(qi) == 0:
        return out
    keep, mp = _mat(matrix)
    qo = np.ascontiguousarray(queries.offsets, np.int64)
    do = np.ascontiguousarray(db.offsets, np.int64)
    qr = np.ascontiguousarray(queries.residues, np.uint8)
    dr = np.ascontiguousarray(db.residues, np.uint8)
    rc = lib().sw_oracle_pairs(qr.ctypes.data, _p(qo, ctypes.c_int64), dr.ctypes.data,
                               _p(do, ctypes.c_int64), _p(qi, ctypes.c_int32),
                               _p(di, ctypes.c_int32), len(qi), mp, gap_open, gap_extend,
                               _p(out, ctypes.c_int32), n_threads)
    if rc != 0:
        raise ValueError("oracle: invalid residue or argument")
    return out


def topk(scores: np.ndarray, k: int):
    """Per query: the k best (score, db_index) under (score desc, db_index asc);
    empty slots are (0, -1) (reading R13).  Returns (score[nq,k], index[nq,k])."""
    nq, nd = scores.shape
    s_out = np.zeros((nq, k), np.int32)
    i_out = np.full((nq, k), -1, np.int32)
    for q in range(nq):
        order = np.lexsort((np.arange(nd), -scores[q].astype(np.int64)))[:k]
        s_out[q, :len(order)] = scores[q, order]
        i_out[q, :len(order)] = order
    return s_out, i_out
