"""Small searches that exercise every libsw kernel, for compute-sanitizer (race
detection / sanitizers).  Each case is checked against the oracle, so a run under
memcheck / racecheck / synccheck / initcheck also proves the results unchanged.

  compute-sanitizer --tool racecheck python tools/sanitize.py

Covers: K4 profiles, K1 (8- and 16-column-step instances: groups below and above 144
columns), K3 (sequences above the long threshold, several chunks; SW_K3_CLUSTER=2/4 in the
environment runs the cluster-split instance), K2 (planted int32 overflow; precision
routing), K5u/K5m top-k and merges, the committed-segment gather/scatter of two workers,
WA cancellation of a GPU-side straggler's replicas, K6 linear-space traceback."""
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np  # noqa: E402

import oracle  # noqa: E402
import seqgen  # noqa: E402
from paper_conf_ipps_mendoncam13_b200 import Database  # noqa: E402


def check(name, r, ref, k):
    assert (r.scores == ref).all(), f"{name}: scores differ"
    s, i = oracle.topk(ref, k)
    assert (np.asarray(r.hit_scores) == s).all() and (np.asarray(r.hit_index) == i).all(), f"{name}: top-k"
    print(f"{name}: ok ({r.stats['kernel_launches']} launches, {r.stats['n_overflow_pairs']} overflow pairs)",
          flush=True)


def main():
    # short (K1, 8-column steps), medium (K1, 16-column steps) and long (K3) sequences
    seqs = [seqgen.residues(1, k * 4000, 20 + (k * 37) % 120).tobytes() for k in range(70)]
    seqs += [seqgen.residues(2, k * 4000, 150 + (k * 53) % 300).tobytes() for k in range(70)]
    seqs += [seqgen.residues(3, k * 9000, 1100 + k * 97).tobytes() for k in range(6)]
    wq = b"W" * 3000
    seqs[5] = b"AC" + wq + b"KL"                   # int32 re-run (K2) after K3: 11 * 3000 > 32767 - 11
    db = seqgen.SeqSet.from_list(seqs)
    qs = seqgen.SeqSet.from_list([wq, seqgen.residues(4, 0, 700).tobytes(),
                                  seqgen.residues(5, 0, 90).tobytes(), b"MKV", seqs[100]])
    M = np.full((24, 24), -2, np.int8)
    np.fill_diagonal(M, 100)                        # big diagonal: saturated pairs in K1 and K3
    D = Database(db, devices=[0])
    try:
        ref = oracle.search(qs, db)
        check("default (K1 + K3 + K2)", D.search(qs, top_k=5, long_threshold=1000), ref, 5)
        check("SS, WA off, 2 streams", D.search(qs, top_k=5, long_threshold=1000, policy="ss",
                                                 workload_adjust=False, streams=2), ref, 5)
        ref2 = oracle.search(qs, db, matrix=M)
        check("matrix with many overflows", D.search(qs, matrix=M, top_k=3, long_threshold=1000), ref2, 3)
        ref3 = oracle.search(qs, db, gap_open=20000, gap_extend=1)
        check("precision routing (all int32)", D.search(qs, gap_open=20000, gap_extend=1, top_k=3), ref3, 3)
        al = D.align(qs, [1, 2, 3, 0, 4], [7, 100, 141, 5, 143])
        for a, (qi, di) in zip(al, [(1, 7), (2, 100), (3, 141), (0, 5), (4, 143)]):
            assert a["score"] == ref[qi, di], "traceback score"
        print("traceback (K6, linear space): ok", flush=True)
    finally:
        D.close()
    # two workers on the device: committed segments gathered/scattered, hit lists merged;
    # worker 1 a GPU-side straggler with WA on (cancelled replicas)
    D2 = Database(db, devices=[0, 0])
    try:
        check("two workers, straggler, WA", D2.search(qs, top_k=5, long_threshold=1000, target_unit_cells=2_000_000,
                                                      straggler_mask=2, straggler_slowdown=8), ref, 5)
    finally:
        D2.close()


if __name__ == "__main__":
    main()
