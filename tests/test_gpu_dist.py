"""The multi-process path on one GPU: two slave processes (ranks) share cuda:0, the
master runs inside rank 0 and hands out PSS/WA units over TCP; the per-rank partial
score matrices merge (element-wise max) into the oracle's matrix."""
import multiprocessing as mp
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _rank(rank, world, port, q, straggler):
    import seqgen
    from paper_conf_ipps_mendoncam13_b200 import Database
    qs = seqgen.random_seqset(61, 6, 50, 900)
    db = seqgen.random_seqset(62, 900, 10, 2500)
    D = Database(db, devices=[0])
    r = D.search(qs, top_k=5, target_unit_cells=2_000_000,
                 straggler_mask=(2 if straggler else 0), straggler_slowdown=6,
                 dist=dict(rank=rank, world=world, port=port, host="127.0.0.1"))
    q.put((rank, r.scores.copy(), r.stats["n_units"],
           [(e["unit"], e["committed"]) for e in r.stats["unit_log"]]))
    D.close()


@pytest.mark.parametrize("straggler", [False, True])
def test_two_ranks_one_gpu(straggler):
    import oracle
    import seqgen
    qs = seqgen.random_seqset(61, 6, 50, 900)
    db = seqgen.random_seqset(62, 900, 10, 2500)
    ref = oracle.search(qs, db)
    port = _port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_rank, args=(r, 2, port, q, straggler)) for r in range(2)]
    for p in ps:
        p.start()
    out = [q.get(timeout=300) for _ in ps]
    for p in ps:
        p.join(timeout=60)
    merged = np.maximum(out[0][1], out[1][1])
    assert (merged == ref).all()
    n_units = out[0][2]
    committed = [u for o in out for (u, c) in o[3] if c]
    assert sorted(committed) == list(range(n_units))
    assert all(len(o[3]) > 0 for o in out)   # both ranks executed units
