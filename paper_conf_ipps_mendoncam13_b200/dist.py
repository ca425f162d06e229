"""Multi-process (torchrun, one process per GPU) search: every rank is a slave of one
master (a thread of rank 0's libsw, reached over TCP), then the hits are merged.

The merge is the paper's last step ("the slaves send their results to the master, that
merges them and sends the result to the user", P16 §IV), with north_star's data plane:
* per-pair scores stay where they were computed: each rank's `scores` holds exactly the
  pairs of the units it committed (-1 elsewhere), so the ranks' slices are disjoint and no
  score matrix crosses the interconnect;
* each rank's top-k over its committed units (libsw K5u/K5m) is all-gathered with one
  NCCL collective (nq * k * 8 bytes per rank) and merged by libsw's sw_merge_hits (K5m).
This module only marshals: the collective is torch.distributed's, the merge is libsw's.
"""
from __future__ import annotations

import os

import torch
import torch.distributed as dist


def master_port(default_offset: int = 17) -> int:
    return int(os.environ.get("SW_MASTER_PORT", int(os.environ.get("MASTER_PORT", "29500")) + default_offset))


def gather_hits(hits: torch.Tensor, group=None) -> torch.Tensor:
    """All-gather every rank's [nq, k, 2] int32 hits into [world, nq, k, 2] (NCCL on GPU
    tensors; gloo goes through the host)."""
    world = dist.get_world_size(group)
    if dist.get_backend(group) == "gloo":
        src = hits.cpu().contiguous()
        out = [torch.empty_like(src) for _ in range(world)]
        dist.all_gather(out, src, group=group)
        return torch.stack(out).to(hits.device)
    out = torch.empty((world,) + tuple(hits.shape), dtype=hits.dtype, device=hits.device)
    dist.all_gather_into_tensor(out, hits.contiguous(), group=group)
    return out


def search(database, queries, rank: int, world: int, top_k: int = 10, host: str = "127.0.0.1",
           port: int | None = None, want_scores: bool = True, out_scores=None, **kw):
    """One distributed search step.  Returns (this rank's committed-only scores, merged hit
    scores, merged hit index, stats).  stats gets "merge_seconds" (device time of the hits
    all-gather and merge, CUDA events on torch's current stream) and "gather_bytes" (bytes
    this rank contributed to the collective)."""
    port = port or master_port()
    r = database.search(queries, top_k=top_k, outputs_on_device=True, want_scores=want_scores,
                        out_scores=out_scores,
                        dist=dict(rank=rank, world=world, port=port, host=host), **kw)
    ev0, ev1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    ev0.record()
    hs = hi = None
    gbytes = 0
    if top_k > 0 and queries.n > 0:
        local = torch.stack([r.hit_scores, r.hit_index], dim=-1)   # [nq, k, 2]
        allh = gather_hits(local)
        gbytes = local.numel() * local.element_size()
        hs, hi = database.merge_hits(allh, top_k)
    ev1.record()
    torch.cuda.synchronize()
    r.stats["merge_seconds"] = ev0.elapsed_time(ev1) * 1e-3
    r.stats["gather_bytes"] = gbytes
    return r.scores, hs, hi, r.stats
