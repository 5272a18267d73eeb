"""Multi-GPU layouts of the ALGAS search (not in the paper, which
uses one GPU).

* Replicas (query-parallel, no collective): every rank holds the whole index
  and serves its own slice of the query stream -- `replica_slice`.
* Sharded index (one exchange step): rank g holds base points
  [g*n/G, (g+1)*n/G) and a graph built inside its shard; every query is
  searched on every shard, the per-shard top-k (with GLOBAL ids) are
  all-gathered over NCCL (NVLink) and merged by (dist, id) with the same
  host TopK merge & filter as the multi-CTA path --
  `ShardedIndex`, `gather_and_merge`.

torch.distributed is plumbing only (process group + all-gather); the search
and the merge run in libalgas.
"""
from __future__ import annotations

import numpy as np

from . import Index, SENTINEL, merge_topk_parts


def shard_range(n: int, world: int, rank: int) -> tuple[int, int]:
    """Contiguous [lo, hi) of base points owned by `rank` (sizes differ by <= 1)."""
    base, extra = divmod(n, world)
    lo = rank * base + min(rank, extra)
    hi = lo + base + (1 if rank < extra else 0)
    return lo, hi


def replica_slice(nq: int, world: int, rank: int) -> slice:
    """Queries served by `rank` when the index is replicated (contiguous split)."""
    lo, hi = shard_range(nq, world, rank)
    return slice(lo, hi)


def to_global(ids: np.ndarray, offset: int) -> np.ndarray:
    """Local shard ids -> global ids (sentinels stay sentinels)."""
    ids = np.asarray(ids, dtype=np.uint32)
    out = ids.astype(np.uint64) + np.uint64(offset)
    out[ids == SENTINEL] = SENTINEL
    return out.astype(np.uint32)


def gather_and_merge(ids: np.ndarray, dists: np.ndarray, k: int, group=None, device=None):
    """All-gather every rank's [nq, k] (global id, dist) and merge per query.

    ids/dists: host arrays of this rank's per-shard results.  Uses
    torch.distributed.all_gather_into_tensor (NCCL on GPUs, gloo on CPU).
    Returns merged (ids [nq,k] uint32, dists [nq,k] float32), identical on
    every rank."""
    import torch
    import torch.distributed as dist

    world = dist.get_world_size(group)
    nq = ids.shape[0]
    dev = device if device is not None else torch.device("cpu")
    ti = torch.from_numpy(np.ascontiguousarray(ids).view(np.int32)).to(dev)
    td = torch.from_numpy(np.ascontiguousarray(dists, dtype=np.float32)).to(dev)
    gi = torch.empty((world * nq, k), dtype=torch.int32, device=dev)
    gd = torch.empty((world * nq, k), dtype=torch.float32, device=dev)
    dist.all_gather_into_tensor(gi, ti, group=group)
    dist.all_gather_into_tensor(gd, td, group=group)
    gi = gi.cpu().numpy().view(np.uint32).reshape(world, nq, k)
    gd = gd.cpu().numpy().reshape(world, nq, k)
    return merge_topk_parts(gi, gd, k)


class ShardedIndex:
    """This rank's shard of a base set, searched locally and merged globally."""

    def __init__(self, shard_data, offset: int, graph=None, metric: int = 0, degree: int | None = None):
        self.offset = int(offset)
        self.index = Index(shard_data, graph, metric=metric, degree=degree)

    def search(self, queries, params, group=None, tag0: int = 0, dynamic: bool = False, device=None):
        """Search every query on this shard, then exchange + merge (all ranks)."""
        if dynamic:
            r = self.index.search_dynamic(queries, params, tag0=tag0)
        else:
            r = self.index.search(queries, params=params, tag0=tag0)
        ids = np.asarray(r["ids"]) if isinstance(r["ids"], np.ndarray) else r["ids"].cpu().numpy().view(np.uint32)
        ds = np.asarray(r["dists"]) if isinstance(r["dists"], np.ndarray) else r["dists"].cpu().numpy()
        gi, gd = gather_and_merge(to_global(ids, self.offset), ds, params.k, group=group, device=device)
        return dict(ids=gi, dists=gd, local=r)
