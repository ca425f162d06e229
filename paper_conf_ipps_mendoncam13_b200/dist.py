"""Multi-process (torchrun, one process per GPU) search: every rank is a slave of one
master (a thread of rank 0's libsw, reached over TCP), then the results are merged.

The merge is the paper's last step ("the slaves send their results to the master, that
merges them and sends the result to the user", P16 §IV).  Each rank's score matrix holds
the pairs of the units it executed (committed or duplicate: identical values) and -1
elsewhere, so an element-wise MAX reduction to rank 0 (NCCL over NVLink) reassembles the
full matrix; rank 0 then takes the top-k on its GPU (libsw K5).
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def master_port(default_offset: int = 17) -> int:
    return int(os.environ.get("SW_MASTER_PORT", int(os.environ.get("MASTER_PORT", "29500")) + default_offset))


def merge_scores(partial: torch.Tensor, group=None, dst: int = 0) -> torch.Tensor:
    """Element-wise MAX of per-rank partial score matrices onto rank `dst` (in place).
    Entries a rank did not compute are -1; computed entries agree across ranks."""
    dist.reduce(partial, dst=dst, op=dist.ReduceOp.MAX, group=group)
    return partial


def merge_hits(scores: torch.Tensor, index: torch.Tensor, k: int, group=None):
    """Merge per-rank top-k lists (score desc, index asc; index -1 = empty) into the
    global top-k, dropping duplicates of the same index (a WA replica computed it twice).
    Used when only hits (not the full matrix) are gathered.  Returns rank-local tensors
    holding the merged lists on every rank."""
    world = dist.get_world_size(group)
    gs = [torch.empty_like(scores) for _ in range(world)]
    gi = [torch.empty_like(index) for _ in range(world)]
    dist.all_gather(gs, scores.contiguous(), group=group)
    dist.all_gather(gi, index.contiguous(), group=group)
    S = torch.cat(gs, dim=1).cpu()
    I = torch.cat(gi, dim=1).cpu()
    nq = S.shape[0]
    out_s = torch.zeros((nq, k), dtype=scores.dtype)
    out_i = torch.full((nq, k), -1, dtype=index.dtype)
    for q in range(nq):
        seen = set()
        cand = sorted(((int(s), int(i)) for s, i in zip(S[q].tolist(), I[q].tolist()) if i >= 0),
                      key=lambda t: (-t[0], t[1]))
        r = 0
        for s, i in cand:
            if i in seen:
                continue
            seen.add(i)
            out_s[q, r], out_i[q, r] = s, i
            r += 1
            if r == k:
                break
    return out_s.to(scores.device), out_i.to(index.device)


def search(database, queries, rank: int, world: int, top_k: int = 10, host: str = "127.0.0.1",
           port: int | None = None, **kw):
    """One distributed search step.  Returns (scores on rank 0 else None, hit scores,
    hit index (rank 0), per-rank libsw stats with "merge_seconds" added: the device time of
    the cross-rank merge and the top-k on this rank, CUDA events on torch's stream)."""
    import torch
    port = port or master_port()
    r = database.search(queries, top_k=top_k, outputs_on_device=True,
                        dist=dict(rank=rank, world=world, port=port, host=host), **kw)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    if dist.get_backend() == "gloo":   # tests / single-GPU runs: the merge goes through the host
        part = r.scores.cpu()
        merge_scores(part)
        merged = part.to(r.scores.device) if rank == 0 else r.scores
    else:
        merged = merge_scores(r.scores)
    hs = hi = None
    if rank == 0 and top_k > 0:
        hs, hi = database.topk_device(merged, top_k)
    ev1.record()
    torch.cuda.synchronize()
    r.stats["merge_seconds"] = ev0.elapsed_time(ev1) * 1e-3
    if rank == 0:
        return merged, hs, hi, r.stats
    return None, None, None, r.stats
