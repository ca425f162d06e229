"""The multi-process path on one GPU: two slave processes (ranks) share cuda:0, the
master runs inside rank 0 and hands out PSS/WA units over TCP.  Data plane (north_star):
each rank's score slice holds exactly its committed units' pairs (disjoint, -1 elsewhere)
and its top-k over them; the hits are gathered and merged by libsw (sw_merge_hits)."""
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
           [(e["unit"], e["committed"]) for e in r.stats["unit_log"]],
           np.stack([r.hit_scores, r.hit_index], axis=-1).copy()))
    D.close()


@pytest.mark.parametrize("straggler", [False, True])
def test_two_ranks_one_gpu(straggler):
    import torch
    import oracle
    import seqgen
    from paper_conf_ipps_mendoncam13_b200 import Database
    qs = seqgen.random_seqset(61, 6, 50, 900)
    db = seqgen.random_seqset(62, 900, 10, 2500)
    ref = oracle.search(qs, db)
    port = _port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_rank, args=(r, 2, port, q, straggler)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted([q.get(timeout=300) for _ in ps], key=lambda o: o[0])
    for p in ps:
        p.join(timeout=60)
    a, b = out[0][1], out[1][1]
    # disjoint slices that cover every pair exactly once, each bit-exact
    assert ((a >= 0) ^ (b >= 0)).all()
    assert (np.maximum(a, b) == ref).all()
    n_units = out[0][2]
    committed = [u for o in out for (u, c) in o[3] if c]
    assert sorted(committed) == list(range(n_units))
    assert all(len(o[3]) > 0 for o in out)   # both ranks executed units
    # each rank's hits = top-k over its own slice; merged by libsw = the oracle's top-k
    for o, sl in zip(out, (a, b)):
        s, i = oracle.topk(np.where(sl >= 0, sl, -1), 5)
        assert (o[4][..., 1] == i).all() and (o[4][..., 0] == s).all()
    D = Database(seqgen.SeqSet.from_list(["A"]))
    hs, hi = D.merge_hits(torch.from_numpy(np.stack([out[0][4], out[1][4]])).cuda(), 5)
    s, i = oracle.topk(ref, 5)
    assert (hi.cpu().numpy() == i).all() and (hs.cpu().numpy() == s).all()
    D.close()


def _torchrun_rank(rank, world, port, mport, q):
    import os
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank), WORLD_SIZE=str(world))
    import torch
    import torch.distributed as dist
    import seqgen
    from paper_conf_ipps_mendoncam13_b200 import Database
    from paper_conf_ipps_mendoncam13_b200 import dist as swdist
    torch.cuda.set_device(0)
    dist.init_process_group("gloo")
    qs = seqgen.random_seqset(71, 5, 40, 700)
    db = seqgen.random_seqset(72, 700, 10, 2000)
    D = Database(db, devices=[0])
    sc, hs, hi, st = swdist.search(D, qs, rank, world, top_k=4, port=mport, target_unit_cells=1_500_000)
    q.put((rank, sc.cpu().numpy(), hs.cpu().numpy(), hi.cpu().numpy(), st["gather_bytes"]))
    D.close()
    dist.destroy_process_group()


def test_dist_search_gathers_hits_only():
    """dist.search end to end (gloo process group on one GPU): merged hits = the oracle's
    top-k on every rank; scores stay rank-local; the collective moves nq*k*8 bytes per rank."""
    import oracle
    import seqgen
    qs = seqgen.random_seqset(71, 5, 40, 700)
    db = seqgen.random_seqset(72, 700, 10, 2000)
    ref = oracle.search(qs, db)
    s, i = oracle.topk(ref, 4)
    port, mport = _port(), _port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    ps = [ctx.Process(target=_torchrun_rank, args=(r, 2, port, mport, q)) for r in range(2)]
    for p in ps:
        p.start()
    out = sorted([q.get(timeout=300) for _ in ps], key=lambda o: o[0])
    for p in ps:
        p.join(timeout=60)
    for o in out:
        assert (o[3] == i).all() and (o[2] == s).all()
        assert o[4] == 5 * 4 * 8
    assert (np.maximum(out[0][1], out[1][1]) == ref).all()
    assert ((out[0][1] >= 0) ^ (out[1][1] >= 0)).all()
