"""Parity of the CUDA path (libsw through its C-ABI) with the oracle, bit-exact.

Every score is an integer, so the bar is equality for every pair.
Inputs are seeded (seqgen); expected values come only from oracle/.
"""
import numpy as np
import pytest

import oracle
import seqgen
from paper_conf_ipps_mendoncam13_b200 import Database, SwError

pytestmark = pytest.mark.gpu


def _search(db, qs, **kw):
    D = Database(db, devices=kw.pop("devices", None))
    try:
        return D.search(qs, **kw)
    finally:
        D.close()


def _check_topk(res, scores_ref, k):
    s, i = oracle.topk(scores_ref, k)
    assert (np.asarray(res.hit_scores) == s).all()
    assert (np.asarray(res.hit_index) == i).all()


def test_c1_full_parity():
    """C1 (BASELINE configs[0]): 1 x 100 aa vs 2,000 SwissProt-shaped sequences."""
    w = seqgen.make_workload("C1")
    ref = oracle.search(w.queries, w.db)
    r = _search(w.db, w.queries, top_k=10)
    assert (r.scores == ref).all()
    _check_topk(r, ref, 10)
    assert r.stats["cells"] == int(w.queries.total) * int(w.db.total)


def _mixed_case(seed, nq=8, nd=700, max_len=3500):
    qlens = [1, 15, 16, 17, 127, 129, 600, 1300][:nq]
    qs = seqgen.SeqSet.from_list([seqgen.residues(seqgen.stream_seed(seed, f"q{k}"), 0, L).tobytes()
                                  for k, L in enumerate(qlens)])
    db = seqgen.random_seqset(seed, nd, 0, max_len)
    # some lengths exactly at group/tile boundaries, and a planted copy of a query
    extra = [b"", b"W", seqgen.residues(seed, 0, 16).tobytes(), seqgen.residues(seed, 0, 32).tobytes(),
             qs.seq(nq - 2), qs.seq(nq - 1) + qs.seq(nq - 3)]
    db = seqgen.SeqSet.from_list([db.seq(i) for i in range(db.n)] + extra)
    return qs, db


def test_mixed_lengths_k1_and_k3():
    qs, db = _mixed_case(7)
    ref = oracle.search(qs, db)
    for thr in (0, 256, -1):   # auto (3072), many long sequences via K3, none via K3
        r = _search(db, qs, top_k=12, long_threshold=thr)
        bad = np.argwhere(r.scores != ref)
        assert len(bad) == 0, (thr, bad[:10], r.scores[tuple(bad[0])], ref[tuple(bad[0])])
        _check_topk(r, ref, 12)


@pytest.mark.parametrize("go,ge", [(10, 2), (0, 2), (0, 0), (11, 1), (5, 0), (40, 7)])
def test_gap_settings(go, ge):
    qs, db = _mixed_case(11, nq=6, nd=300, max_len=1200)
    ref = oracle.search(qs, db, gap_open=go, gap_extend=ge)
    r = _search(db, qs, gap_open=go, gap_extend=ge, top_k=5, long_threshold=400)
    assert (r.scores == ref).all()


@pytest.mark.parametrize("seed", [1, 2, 3])
def test_random_matrices(seed):
    M = seqgen.random_matrix(seed, lo=-12, hi=15)
    M[3, 5] = 40    # asymmetric entry: query row vs db column must not be transposed
    qs, db = _mixed_case(20 + seed, nq=5, nd=250, max_len=900)
    ref = oracle.search(qs, db, matrix=M, gap_open=6, gap_extend=3)
    r = _search(db, qs, matrix=M, gap_open=6, gap_extend=3, top_k=4, long_threshold=300)
    assert (r.scores == ref).all()


def test_overflow_rerun_int32():
    """Saturation of the s16x2 lanes is detected and the pair re-scored in int32 (K2):
    an all-W query of 3,200 aa vs a sequence containing it scores 11*3200 = 35,200."""
    wq = "W" * 3200
    qs = seqgen.SeqSet.from_list([wq, seqgen.residues(3, 0, 3100).tobytes(), "WWWW"])
    base = seqgen.random_seqset(4, 120, 10, 4000)
    seqs = [base.seq(i) for i in range(base.n)]
    seqs[5] = b"ACD" + wq.encode() + b"KLM"
    seqs[77] = wq.encode()[:1500]
    db = seqgen.SeqSet.from_list(seqs)
    ref = oracle.search(qs, db)
    assert ref.max() > 32767
    for thr in (0, 1000):
        r = _search(db, qs, top_k=3, long_threshold=thr)
        assert (r.scores == ref).all()
        assert r.stats["n_overflow_pairs"] >= 1
        assert r.stats["n_k2_launches"] >= 1 and r.stats["kernel_seconds_k2"] > 0


def test_big_matrix_forces_many_overflows():
    M = np.full((24, 24), -20, np.int8)
    np.fill_diagonal(M, 120)
    qs = seqgen.SeqSet.from_list([b"A" * 400, b"C" * 300, seqgen.residues(9, 0, 500).tobytes()])
    db = seqgen.SeqSet.from_list([b"A" * 350, b"C" * 280, b"AC" * 200, b"W" * 10] +
                                 [seqgen.residues(10, k * 1000, 300 + k).tobytes() for k in range(60)])
    ref = oracle.search(qs, db, matrix=M, gap_open=10, gap_extend=2)
    r = _search(db, qs, matrix=M, top_k=5)
    assert (r.scores == ref).all()
    assert r.stats["n_overflow_pairs"] >= 2


def test_overflow_rerun_multi_chunk():
    """K2 runs one block per saturated pair with 8,192-row chunks: a 9,500-aa overflowing
    query crosses a chunk border (border row handed from the last active thread to thread
    0), with its best cell below the border, and a gapped copy in a second sequence."""
    q = b"W" * 3000 + seqgen.residues(21, 0, 6000).tobytes() + b"W" * 500
    gapped = q[:8000] + b"PG" + q[8000:9000] + q[9003:]
    base = seqgen.random_seqset(22, 40, 100, 3000)
    seqs = [base.seq(i) for i in range(base.n)]
    seqs[3] = b"KK" + q + b"EE"
    seqs[17] = gapped
    db = seqgen.SeqSet.from_list(seqs)
    qs = seqgen.SeqSet.from_list([q, seqgen.residues(23, 0, 900).tobytes()])
    ref = oracle.search(qs, db)
    assert ref[0, 3] > 32767 and ref[0, 17] > 32767
    r = _search(db, qs, top_k=3)
    assert (r.scores == ref).all()
    assert r.stats["n_overflow_pairs"] >= 2
    # every pair through K2 (alpha + beta > 16384), several chunks, no saturation needed
    ref2 = oracle.search(qs, db, gap_open=20000, gap_extend=3)
    r2 = _search(db, qs, gap_open=20000, gap_extend=3, top_k=3)
    assert (r2.scores == ref2).all()


def test_precision_routing_large_gaps():
    """alpha + beta > 16384: every pair goes to the int32 kernel."""
    qs, db = _mixed_case(5, nq=4, nd=100, max_len=500)
    ref = oracle.search(qs, db, gap_open=20000, gap_extend=1)
    r = _search(db, qs, gap_open=20000, gap_extend=1, top_k=3)
    assert (r.scores == ref).all()


def test_edge_cases():
    db = seqgen.SeqSet.from_list(["", "A", "ACDEFGHIK", ""])
    qs = seqgen.SeqSet.from_list(["", "WWA", "k"])        # lower case accepted
    ref = oracle.search(seqgen.SeqSet.from_list(["", "WWA", "K"]), db)
    r = _search(db, qs, top_k=6)
    assert (r.scores == ref).all()
    assert (np.asarray(r.hit_index)[:, 4:] == -1).all()   # ndb < k: empty slots {0, -1}
    assert (np.asarray(r.hit_scores)[:, 4:] == 0).all()
    # no queries / no database sequences
    r0 = _search(db, seqgen.SeqSet.from_list([]), top_k=3)
    assert r0.scores.shape == (0, 4)
    r1 = _search(seqgen.SeqSet.from_list([]), qs, top_k=3)
    assert r1.scores.shape == (3, 0) and (np.asarray(r1.hit_index) == -1).all()


def test_errors_are_reported():
    db = seqgen.SeqSet.from_list(["ACD", "AJX"])
    with pytest.raises(SwError) as e:
        Database(db)
    assert e.value.code == -2 and "sequence 1" in str(e.value)
    D = Database(seqgen.SeqSet.from_list(["ACD"]))
    with pytest.raises(SwError) as e:
        D.search(seqgen.SeqSet.from_list(["AC1"]))
    assert e.value.code == -2
    with pytest.raises(SwError):
        D.search(seqgen.SeqSet.from_list(["ACD"]), gap_open=-1)
    D.close()


def test_results_independent_of_schedule():
    """Scores are identical for every policy, WA setting, unit size and stream count."""
    qs, db = _mixed_case(31, nq=8, nd=600, max_len=2500)
    ref = oracle.search(qs, db)
    D = Database(db)
    for kw in [dict(policy="ss"), dict(policy="pss", workload_adjust=False),
               dict(target_unit_cells=2_000_000, streams=1),
               dict(target_unit_cells=5_000_000, streams=4, long_threshold=200),
               dict(target_unit_cells=2**62)]:
        r = D.search(qs, top_k=7, **kw)
        assert (r.scores == ref).all(), kw
        _check_topk(r, ref, 7)
    D.close()


@pytest.mark.parametrize("mode", ["sm_cap", "hold", "noise"])
def test_two_workers_one_gpu_with_straggler(mode):
    """Two slave workers on one GPU (two replicas, separate streams); worker 1 is a 6x slower
    PE (GPU-side SM cap, host-side hold, or a local-load kernel).  WA duplicates its late
    units; results stay bit-exact and every pair is merged from the committing worker (the
    in-process data plane: committed segments + top-k lists copied to the first worker)."""
    qs, db = _mixed_case(41, nq=8, nd=800, max_len=2000)
    ref = oracle.search(qs, db)
    r = _search(db, qs, devices=[0, 0], top_k=5, target_unit_cells=3_000_000,
                straggler_mask=0b10, straggler_slowdown=6, straggler_mode=mode)
    assert (r.scores == ref).all()
    _check_topk(r, ref, 5)
    assert r.stats["n_devices"] == 2
    log = r.stats["unit_log"]
    assert {e["worker"] for e in log} == {0, 1}
    assert sum(e["committed"] for e in log) == r.stats["n_units"]
    assert all(e["slowed"] for e in log if e["worker"] == 1)
    assert not any(e["slowed"] for e in log if e["worker"] == 0)


def test_merge_hits_api():
    """sw_merge_hits (K5m) against a host merge: disjoint sources, empty slots, ties broken
    by the lower db index, a source shorter than top_k."""
    import torch
    rng = np.random.default_rng(3)
    n_src, nq, k_in, k = 3, 5, 7, 6
    lists = np.zeros((n_src, nq, k_in, 2), np.int32)
    for r in range(n_src):
        for q in range(nq):
            idx = rng.choice(np.arange(r * 1000, r * 1000 + 50), k_in, replace=False)
            sc = rng.integers(0, 6, k_in)
            o = np.lexsort((idx, -sc))
            lists[r, q, :, 0], lists[r, q, :, 1] = sc[o], idx[o]
    lists[1, 2, 3:] = (0, -1)      # a short list
    D = Database(seqgen.SeqSet.from_list(["ACD"]))
    hs, hi = D.merge_hits(torch.from_numpy(lists).cuda(), k)
    for q in range(nq):
        cand = [(int(s), int(i)) for r in range(n_src) for s, i in lists[r, q] if i >= 0]
        cand.sort(key=lambda t: (-t[0], t[1]))
        exp = (cand + [(0, -1)] * k)[:k]
        assert [tuple(x) for x in zip(hs[q].tolist(), hi[q].tolist())] == exp
    D.close()


def _digest(cfg, scores):
    import hashlib
    import json
    import os
    g = json.load(open(os.path.join(os.path.dirname(os.path.abspath(__file__)), "golden", "oracle_digests.json")))
    sc = np.ascontiguousarray(scores, dtype="<i4")
    return hashlib.sha256(sc.tobytes()).hexdigest() == g[cfg]["sha256_scores"], g[cfg]


def test_wa_beats_a_gpu_side_straggler():
    """workload adjustment against a genuinely slow GPU.  Two workers share the
    B200; worker 1's DP kernels get one SM's worth of blocks.  C2 with the paper's coarse tasks
    (one per pack and kernel kind), one stream per worker: the slow worker takes its first task
    before the master knows its rate, and that task outlives all the others, so without WA it
    decides the end.  With WA on, the fast worker re-executes the
    straggler's last unit, the straggler's replica is cancelled IN its kernel (abort flag polled
    in the group/chunk loops) and abandoned with the cells it really computed; makespan and tail
    drop.  Both runs are bit-exact against the oracle's C2 digest."""
    w = seqgen.make_workload("C2")
    D = Database(w.db, devices=[0, 0])
    kw = dict(top_k=10, target_unit_cells=2**62, straggler_mask=0b10, straggler_slowdown=148,
              straggler_mode="sm_cap", streams=1)
    D.search(w.queries, **kw)   # warm-up (lazy module loading, buffers)
    on = D.search(w.queries, workload_adjust=True, **kw)
    ok_on, e = _digest("C2", on.scores)
    off = D.search(w.queries, workload_adjust=False, **kw)
    ok_off, _ = _digest("C2", off.scores)
    D.close()
    assert ok_on and ok_off
    assert (np.asarray(on.hit_index) == np.asarray(e["top10_index"])).all()
    log = on.stats["unit_log"]
    cancelled = [x for x in log if x["cancelled"]]
    assert on.stats["n_wa_grants"] >= 1 and on.stats["n_cancelled"] >= 1 and cancelled
    for x in cancelled:
        assert x["cells_done"] < x["cells"] and not x["committed"]
        # its committed twin ran on the other worker
        assert any(y["unit"] == x["unit"] and y["committed"] and y["worker"] != x["worker"] for y in log)
    assert on.stats["seconds_device"] < off.stats["seconds_device"]
    assert on.stats["seconds_last_unit"] < off.stats["seconds_last_unit"]
    assert on.stats["tail_seconds"] < 0.5 * off.stats["tail_seconds"]
    assert on.stats["duplicated_cells"] == sum(x["cells_done"] for x in log if not x["committed"])


def test_local_load_midrun_pss_reweights():
    """NEXT-1 (P24 §V.C, Figs. 7/8): worker 1 keeps ceil(148/12) SMs after 30 % of the run.
    The master's per-grant log shows PSS re-weighting (Φ of the unloaded worker rises above 1,
    the loaded worker's stays 1); the result stays bit-exact (C2 digest)."""
    w = seqgen.make_workload("C2")
    D = Database(w.db, devices=[0, 0])
    base = D.search(w.queries, top_k=10)
    after = int(1000 * 0.3 * base.stats["seconds_device"])
    r = D.search(w.queries, top_k=10, straggler_mask=0b10, straggler_slowdown=12,
                 straggler_mode="sm_cap", straggler_after_ms=after)
    D.close()
    assert _digest("C2", r.scores)[0]
    from paper_conf_ipps_mendoncam13_b200 import grant_timeline
    g = grant_timeline(r.stats["sched_log"])
    assert g
    late = [x for x in g if x["t_rel"] > 1e-3 * after + 0.03 and not x["wa"]]
    assert any(x["worker"] == 0 and x["phi"] >= 2 for x in late), late[:10]
    assert all(x["phi"] == 1 for x in late if x["worker"] == 1)
    # v̄ of the loaded worker falls below the other's
    v0 = [x["rate"] for x in late if x["worker"] == 0]
    v1 = [x["rate"] for x in late if x["worker"] == 1]
    assert v0 and (not v1 or max(v1) < max(v0))
    slowed = [x for x in r.stats["unit_log"] if x["slowed"]]
    assert slowed and all(x["worker"] == 1 for x in slowed)


def test_noise_kernel_single_worker():
    """Straggler mode "noise": a local-load kernel fills all but ceil(148/6) SMs of the GPU
    from t0 and is stopped at the end of the search; results unchanged."""
    qs, db = _mixed_case(43, nq=6, nd=500, max_len=3000)
    ref = oracle.search(qs, db)
    r = _search(db, qs, top_k=4, straggler_mask=1, straggler_mode="noise", straggler_after_ms=1)
    assert (r.scores == ref).all()
    _check_topk(r, ref, 4)


def test_outputs_on_device():
    import torch
    qs, db = _mixed_case(51, nq=4, nd=200, max_len=800)
    ref = oracle.search(qs, db)
    r = _search(db, qs, top_k=3, outputs_on_device=True)
    assert r.scores.is_cuda
    assert (r.scores.cpu().numpy() == ref).all()
    s, i = oracle.topk(ref, 3)
    assert (r.hit_index.cpu().numpy() == i).all() and (r.hit_scores.cpu().numpy() == s).all()


def test_c5_long_sequences_small():
    """C5 shape at reduced count: 8 x 5,000-aa queries (one W/C/Y-rich overflow query) vs
    long sequences (10k-35k) on the intra-task kernel; full parity."""
    w = seqgen.make_workload("C5", n_db=24)
    ref = oracle.search(w.queries, w.db)
    r = _search(w.db, w.queries, top_k=5)
    assert (r.scores == ref).all()
    assert r.stats["cells_k3"] > 0 and r.stats["n_overflow_pairs"] >= 1
    _check_topk(r, ref, 5)


def _sampled_parity(w, r, n_sample, seed):
    rng = np.random.default_rng(seed)
    qi = rng.integers(0, w.queries.n, n_sample).astype(np.int32)
    di = rng.integers(0, w.db.n, n_sample).astype(np.int32)
    # always include the longest DB sequences and every planted pair
    longest = np.argsort(-w.db.lengths)[:8]
    pq = [p["query"] for p in w.meta["planted"]]
    pd = [p["slot"] for p in w.meta["planted"]]
    qi = np.concatenate([qi, np.repeat(np.arange(w.queries.n), len(longest)), pq]).astype(np.int32)
    di = np.concatenate([di, np.tile(longest, w.queries.n), pd]).astype(np.int32)
    ref = oracle.pairs(w.queries, w.db, qi, di)
    got = np.asarray(r.scores)[qi, di]
    assert (got == ref).all(), np.argwhere(got != ref)[:5]
    # self-hits (reading R16): each query's best hit is its own DB slot (or an equal score)
    for p in w.meta["planted"]:
        if p["kind"] == "self":
            q = p["query"]
            assert np.asarray(r.hit_scores)[q, 0] == np.asarray(r.scores)[q].max()
            assert np.asarray(r.scores)[q, p["slot"]] == np.asarray(r.hit_scores)[q, 0]


def test_c2_full_size_sampled():
    w = seqgen.make_workload("C2")
    r = _search(w.db, w.queries, top_k=10)
    _sampled_parity(w, r, 1500, 2)
    # every pair's score is a valid non-negative integer
    assert (np.asarray(r.scores) >= 0).all()


@pytest.mark.slow
def test_c4_full_size_sampled():
    w = seqgen.make_workload("C4")
    r = _search(w.db, w.queries, top_k=10)
    _sampled_parity(w, r, 1000, 4)
    assert (np.asarray(r.scores) >= 0).all()


def test_paper_figures_on_gpu():
    """The paper's printed values through the CUDA path: Fig. 2 (GAAGCTA x GCTGACCT,
    linear gap -2, score 3, P12/P14) and Fig. 1's pair (SW >= the printed global 4)."""
    M = np.full((24, 24), -1, np.int8)
    np.fill_diagonal(M, 1)
    qs = seqgen.SeqSet.from_list(["GAAGCTA", "ACTTGTCCG"])
    db = seqgen.SeqSet.from_list(["GCTGACCT", "ATTGTCAG"])
    r = _search(db, qs, matrix=M, gap_open=0, gap_extend=2, top_k=2)
    assert r.scores[0, 0] == 3
    assert r.scores[1, 1] >= 4
    assert (r.scores == oracle.search(qs, db, matrix=M, gap_open=0, gap_extend=2)).all()


@pytest.mark.parametrize("cfg", ["C3", "RAT", "MOUSE"])
def test_other_databases_full_size_sampled(cfg):
    """Table II's other database shapes (RefSeq Human, Ensembl Rat, RefSeq Mouse)."""
    w = seqgen.make_workload(cfg)
    r = _search(w.db, w.queries, top_k=10)
    _sampled_parity(w, r, 600, 7)


def test_c5_full_size_sampled():
    """C5 at full size: 8 x 5,000-aa queries vs 2,048 sequences of 10k-35k aa (K3 + the
    planted overflow pair re-scored in int32)."""
    w = seqgen.make_workload("C5")
    r = _search(w.db, w.queries, top_k=5)
    assert r.stats["n_overflow_pairs"] >= 1 and r.stats["cells_k3"] == r.stats["cells"]
    rng = np.random.default_rng(5)
    qi = rng.integers(0, w.queries.n, 24).astype(np.int32)
    di = rng.integers(0, w.db.n, 24).astype(np.int32)
    pq = np.array([p["query"] for p in w.meta["planted"]], np.int32)
    pd = np.array([p["slot"] for p in w.meta["planted"]], np.int32)
    qi, di = np.concatenate([qi, pq]), np.concatenate([di, pd])
    ref = oracle.pairs(w.queries, w.db, qi, di)
    assert (np.asarray(r.scores)[qi, di] == ref).all()
    assert ref.max() > 32767


def _check_alignment(q, d, a, M=None, go=10, ge=2):
    """An alignment from sw_align is valid and optimal: its ops consume exactly the
    reported substrings and the oracle's alignment scorer gives the pair's SW score."""
    ops = a["ops"]
    assert ops.count("M") + ops.count("I") == a["q_end"] - a["q_begin"]
    assert ops.count("M") + ops.count("D") == a["d_end"] - a["d_begin"]
    if a["score"] == 0:
        assert ops == ""
        return
    rq, rd, i, j = [], [], a["q_begin"], a["d_begin"]
    for op in ops:
        if op == "M":
            rq.append(q[i]); rd.append(d[j]); i += 1; j += 1
        elif op == "I":
            rq.append(q[i]); rd.append("-"); i += 1
        else:
            rq.append("-"); rd.append(d[j]); j += 1
    assert oracle.alignment_score("".join(rq), "".join(rd), M, go, ge) == a["score"]
    if go + ge > 0:
        assert ops[0] == "M" and ops[-1] == "M"


def test_traceback_phase2():
    """NEXT-3 (P12 §II.A.2 Phase 2): alignments of the top hits and of random pairs."""
    qs, db = _mixed_case(71, nq=8, nd=400, max_len=2500)
    D = Database(db)
    r = D.search(qs, top_k=3)
    qi = np.repeat(np.arange(qs.n), 3)
    di = np.asarray(r.hit_index).reshape(-1)
    rng = np.random.default_rng(3)
    qi = np.concatenate([qi, rng.integers(0, qs.n, 40)]).astype(np.int32)
    di = np.concatenate([di, rng.integers(0, db.n, 40)]).astype(np.int32)
    keep = di >= 0
    qi, di = qi[keep], di[keep]
    al = D.align(qs, qi, di)
    ref = oracle.pairs(qs, db, qi, di)
    for k, a in enumerate(al):
        assert a["score"] == ref[k]
        _check_alignment(qs.seq(int(qi[k])).decode(), db.seq(int(di[k])).decode(), a)
    # Fig. 2 through Phase 2: the printed local alignment score 3 (P12/P14)
    M = np.full((24, 24), -1, np.int8)
    np.fill_diagonal(M, 1)
    D2 = Database(seqgen.SeqSet.from_list(["GCTGACCT"]))
    a = D2.align(seqgen.SeqSet.from_list(["GAAGCTA"]), [0], [0], matrix=M, gap_open=0, gap_extend=2)[0]
    assert a["score"] == 3
    _check_alignment("GAAGCTA", "GCTGACCT", a, M, 0, 2)
    D.close(); D2.close()


def test_traceback_long_and_asymmetric():
    """Phase 2 on long sequences (several 256-row chunks, 10k+ columns) and with an
    asymmetric matrix (query residue = row)."""
    w = seqgen.make_workload("C5", n_db=10)
    D = Database(w.db)
    qi = np.array([p["query"] for p in w.meta["planted"]] + [0, 1], np.int32)
    di = np.array([p["slot"] for p in w.meta["planted"]] + [3, 5], np.int32)
    al = D.align(w.queries, qi, di)
    ref = oracle.pairs(w.queries, w.db, qi, di)
    for k, a in enumerate(al):
        assert a["score"] == ref[k]
        _check_alignment(w.queries.seq(int(qi[k])).decode(), w.db.seq(int(di[k])).decode(), a)
    D.close()
    M = seqgen.random_matrix(9, lo=-6, hi=9)
    M[2, 7] = 25
    qs, db = _mixed_case(81, nq=4, nd=60, max_len=700)
    D = Database(db)
    qi = np.repeat(np.arange(qs.n), 15).astype(np.int32)
    di = np.tile(np.arange(15), qs.n).astype(np.int32)
    al = D.align(qs, qi, di, matrix=M, gap_open=4, gap_extend=3)
    ref = oracle.pairs(qs, db, qi, di, matrix=M, gap_open=4, gap_extend=3)
    for k, a in enumerate(al):
        assert a["score"] == ref[k]
        _check_alignment(qs.seq(int(qi[k])).decode(), db.seq(int(di[k])).decode(), a, M, 4, 3)
    D.close()


def test_unusual_inputs():
    """Ambiguity codes B/Z/X and '*', lower case, a query longer than the database
    sequences (12,000 aa; several K1 bands of 128 rows and K3 chunks of 512), many short
    queries (packs of several queries per s16x2 half), and duplicate sequences."""
    rng = np.random.default_rng(17)
    alpha = seqgen.AMINO + "BZX*"
    def rs(n):
        return "".join(alpha[i] for i in rng.integers(0, len(alpha), n))
    queries = [rs(12000), rs(5).lower(), rs(1)] + [rs(int(x)) for x in rng.integers(10, 300, 61)]
    db = [rs(int(x)) for x in rng.integers(0, 4000, 300)] + [queries[3], queries[3], "*" * 50, "X" * 3100]
    qs, dbs = seqgen.SeqSet.from_list(queries), seqgen.SeqSet.from_list(db)
    ref = oracle.search(seqgen.SeqSet.from_list([q.upper() for q in queries]), dbs)
    for thr in (0, 1000):
        r = _search(dbs, qs, top_k=6, long_threshold=thr)
        bad = np.argwhere(r.scores != ref)
        assert len(bad) == 0, (thr, bad[:5])
        _check_topk(r, ref, 6)


def test_extreme_lengths():
    """Beyond the paper's shapes: database sequences of 120,000 and 70,000 residues and a
    60,000-aa query (118 K3 chunks, 469 K1 bands), through K3 (auto threshold) and through
    K1 alone (threshold above every length: 120,000-column groups and border rows)."""
    q_short = seqgen.residues(31, 0, 300).tobytes()
    long1 = seqgen.residues(32, 0, 120000).tobytes()
    long1 = long1[:50000] + q_short + long1[50300:]
    db = [long1, seqgen.residues(33, 0, 70000).tobytes()] + \
         [seqgen.residues(34, k * 1000, 200 + 13 * k).tobytes() for k in range(40)]
    qs = seqgen.SeqSet.from_list([seqgen.residues(35, 0, 2000).tobytes(), q_short,
                                  seqgen.residues(36, 0, 60000).tobytes()])
    dbs = seqgen.SeqSet.from_list(db)
    ref = oracle.search(qs, dbs)
    for thr in (0, 1 << 20):
        r = _search(dbs, qs, top_k=4, long_threshold=thr)
        assert (r.scores == ref).all(), (thr, np.argwhere(r.scores != ref)[:5])
        _check_topk(r, ref, 4)


_CLUSTER_SCRIPT = r"""
import sys; sys.path.insert(0, %r)
import numpy as np, oracle, seqgen
from paper_conf_ipps_mendoncam13_b200 import Database
w = seqgen.make_workload("C5", n_db=24)
ref = oracle.search(w.queries, w.db)
qs = seqgen.SeqSet.from_list([seqgen.residues(41, 0, L).tobytes() for L in (1300, 600, 17, 3000)])
db = seqgen.random_seqset(42, 300, 0, 4000)
db = seqgen.SeqSet.from_list([db.seq(i) for i in range(db.n)] + [b"W" * 3000])
ref2 = oracle.search(qs, db)
D = Database(w.db, devices=[0])
r = D.search(w.queries, top_k=5)
assert (r.scores == ref).all(), np.argwhere(r.scores != ref)[:5]
assert r.stats["n_overflow_pairs"] >= 1
# slower-PE grid cap: fewer resident clusters than sequence blocks (persistent loop)
r = D.search(w.queries, top_k=5, straggler_mask=1, straggler_slowdown=40)
assert (r.scores == ref).all()
D.close()
D = Database(db, devices=[0])
for thr in (0, 500):
    r = D.search(qs, top_k=3, long_threshold=thr)
    assert (r.scores == ref2).all(), np.argwhere(r.scores != ref2)[:5]
D.close()
# WA replicas of clustered units cancelled mid-run (spinning consumers must see the abort)
D = Database(w.db, devices=[0, 0])
r = D.search(w.queries, top_k=5, target_unit_cells=10**9, straggler_mask=2, straggler_slowdown=8)
assert (r.scores == ref).all()
D.close()
print("ok", r.stats["n_cancelled"], r.stats["n_wa_grants"])
"""


@pytest.mark.parametrize("cluster", ["2", "3", "4", "5", "8"])
def test_k3_cluster_split(cluster):
    """K3 with each pair's chunks split over a thread-block cluster (SW_K3_CLUSTER forces the
    size; auto picks it for small long-sequence shares): bit-exact on C5-shaped pairs with an
    overflow, with a capped (persistent) grid, on mixed lengths, and with WA cancellations."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, SW_K3_CLUSTER=cluster)
    out = subprocess.run([sys.executable, "-c", _CLUSTER_SCRIPT % root], env=env, capture_output=True,
                         text=True, timeout=900)
    assert out.returncode == 0 and "ok" in out.stdout, (out.stdout[-2000:], out.stderr[-3000:])


def test_traceback_gaps_across_chunks():
    """K6 linear space: the alignment's insertion / deletion runs cross the 256-row chunk
    boundaries where the backtrack recomputes the chunk above (the H/E/F state carries over)."""
    r = seqgen.residues(91, 0, 900).tobytes()
    q = r[:240] + b"W" * 40 + r[240:600] + r[620:900]   # insertion spanning row 256, deletion near 600
    d = r[:900]
    qs = seqgen.SeqSet.from_list([q, r[:520], b"W" * 300 + r[:300]])
    db = seqgen.SeqSet.from_list([d, r[100:700], r[:260] + b"K" * 30 + r[260:900]])
    D = Database(db)
    qi = np.repeat(np.arange(3), 3).astype(np.int32)
    di = np.tile(np.arange(3), 3).astype(np.int32)
    al = D.align(qs, qi, di)
    ref = oracle.pairs(qs, db, qi, di)
    for k, a in enumerate(al):
        assert a["score"] == ref[k]
        _check_alignment(qs.seq(int(qi[k])).decode(), db.seq(int(di[k])).decode(), a)
    assert "I" * 40 in al[0]["ops"]
    D.close()


_K2_SCRIPT = """
import os, sys; sys.path.insert(0, %r); sys.path.insert(0, os.path.join(sys.path[0], "tests"))
import test_gpu_parity as T
T.test_overflow_rerun_int32()
T.test_big_matrix_forces_many_overflows()
T.test_overflow_rerun_multi_chunk()
T.test_precision_routing_large_gaps()
# every pair through K2 (alpha + beta > 16384): queries whose cluster chunks use 4, 8 and
# 16 rows per thread, against short, ragged and empty sequences
import numpy as np, oracle, seqgen
qs = seqgen.SeqSet.from_list([seqgen.residues(71, 0, L).tobytes() for L in (40000, 20000, 9000, 4000, 33)])
db = seqgen.SeqSet.from_list([seqgen.residues(72, k, L).tobytes() for k, L in enumerate((1500, 7, 0, 2001, 640))])
ref = oracle.search(qs, db, gap_open=20000, gap_extend=3)
r = T._search(db, qs, gap_open=20000, gap_extend=3, top_k=2)
assert (r.scores == ref).all(), np.argwhere(r.scores != ref)[:5]
print("ok")
"""


@pytest.mark.parametrize("big", ["1", "2000000"])
def test_k2_split(big):
    """K2 splits a big saturated pair into chunks run by several blocks at once (chunk tickets
    taken in order, borders through L2 with pair-tagged progress counters, two pair slots).
    SW_K2_BIG lowers the size at which a pair counts as big: "1" sends every re-run pair
    (down to a 4-aa query, one chunk) through the split path -- many pairs, slot reuse --
    "2000000" mixes both paths in one launch.  Queries of 33 to 40,000 aa cover 4, 8 and
    16 rows per thread.  Every overflow / int32-routing case stays bit-exact."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, SW_K2_BIG=big)
    out = subprocess.run([sys.executable, "-c", _K2_SCRIPT % root], env=env, capture_output=True,
                         text=True, timeout=900, cwd=root)
    assert out.returncode == 0 and "ok" in out.stdout, (out.stdout[-2000:], out.stderr[-3000:])


def test_green_partitions_emulated_gpus():
    """Emulated GPUs (worker_sms): four workers on one B200, each on its own green-context SM
    partition (32 SMs: 37 rounded down to a multiple of 8); then back to the whole GPU, and
    to 16-SM partitions with a GPU-side straggler and WA.  C2 stays bit-exact (digest) in
    every layout; the stats report the partition."""
    w = seqgen.make_workload("C2")
    D = Database(w.db, devices=[0, 0, 0, 0])
    try:
        r = D.search(w.queries, top_k=10, worker_sms=37, streams=2)
        assert r.stats["partition_mode"] == 2 and r.stats["partition_sms"] == 32
        assert _digest("C2", r.scores)[0]
        r = D.search(w.queries, top_k=10, streams=2)
        assert r.stats["partition_mode"] == 0
        assert _digest("C2", r.scores)[0]
        r = D.search(w.queries, top_k=10, worker_sms=18, streams=2, straggler_mask=0b1000, straggler_slowdown=4,
                     target_unit_cells=2**62)
        assert r.stats["partition_mode"] == 2 and r.stats["partition_sms"] == 16
        assert _digest("C2", r.scores)[0]
        # under the 8-SM partition granularity: CTA caps (blocks of the workers share SMs)
        r = D.search(w.queries, top_k=10, worker_sms=6, streams=2)
        assert r.stats["partition_mode"] == 1 and r.stats["partition_sms"] == 6
        assert _digest("C2", r.scores)[0]
    finally:
        D.close()
    # long sequences (K3), the planted overflow (K2, started early) and WA replicas cancelled
    # inside their kernels, on 32-SM partitions with a co-running load on the last worker
    w5 = seqgen.make_workload("C5", n_db=24)
    ref = oracle.search(w5.queries, w5.db)
    D = Database(w5.db, devices=[0, 0, 0, 0])
    try:
        r = D.search(w5.queries, top_k=5, worker_sms=37, straggler_mask=0b1000, straggler_slowdown=6,
                     straggler_mode="noise", target_unit_cells=10**9)
        assert r.stats["partition_mode"] == 2
        assert (r.scores == ref).all(), np.argwhere(r.scores != ref)[:5]
        assert r.stats["n_overflow_pairs"] >= 1
    finally:
        D.close()


@pytest.mark.parametrize("script,extra", [("k2", {"SW_K2_BIG": "1"}), ("k2", {}), ("cluster", {"SW_K3_CLUSTER": "5"}),
                                          ("cluster", {"SW_K3_CLUSTER": "2"})])
def test_checked_build(script, extra):
    """The same bit-exact cases on libsw_checked.so (SW_CHECKED=1: bounds of border rows, ring
    slots, profile codes and list entries asserted inside K1/K2/K3; a violation traps and the
    subprocess fails).  compute-sanitizer is closed on this GPU pool; these asserts stand in."""
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ, SW_CHECKED="1", **extra)
    src = (_K2_SCRIPT if script == "k2" else _CLUSTER_SCRIPT) % root
    src += ("\nimport paper_conf_ipps_mendoncam13_b200 as _P\n"
            "assert _P.lib()._name.endswith('libsw_checked.so'), _P.lib()._name\nprint('checked lib ok')\n")
    out = subprocess.run([sys.executable, "-c", src], env=env, capture_output=True, text=True, timeout=1200, cwd=root)
    assert "checked lib ok" in out.stdout, (out.stdout[-2000:], out.stderr[-3000:])
    assert out.returncode == 0 and "ok" in out.stdout, (out.stdout[-2000:], out.stderr[-3000:])
    assert "SW_CHECK failed" not in out.stdout + out.stderr
