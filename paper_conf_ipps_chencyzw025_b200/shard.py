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


class ShardedServer:
    """Sharded-index SERVING: rank g runs a persistent `Server` (its slot ring,
    dynamic batching) on its shard of the base set.  Rank 0 holds the query
    stream; every batch of it is broadcast to all ranks (one collective per
    batch), each rank streams the batch through its own server's host FIFO
    (`enqueue`) and collects its per-shard top-k by tag, and the per-shard
    lists (GLOBAL ids) of each batch are all-gathered and merged on every rank
    with the host TopK merge & filter of the multi-CTA path.

    All batches are broadcast and enqueued before the first is collected, so
    the shards' searches of batch i+1 overlap the exchange of batch i.
    `server`: this rank's Server (or an emulated one in host-logic tests);
    `offset`: first global id of this rank's shard.  The exchange launches
    small torch / NCCL kernels; with CUDA's lazy module loading the first
    launch of a kernel can wait for the device to go idle, which a running
    persistent kernel never does: create the server deferred, call
    `warmup()`, then start it."""

    def __init__(self, server, offset: int, k: int, group=None, device=None):
        self.server = server
        self.offset = int(offset)
        self.k = int(k)
        self.group = group
        self.device = device

    def warmup(self, dim: int, batch: int) -> None:
        """Collective.  Runs every device operation of `serve` once (header
        and batch broadcasts, the all-gather + merge) on dummy data, so their
        kernels are loaded before the persistent kernel starts."""
        import torch
        dev = self.device if self.device is not None else torch.device("cpu")
        hdr = torch.zeros(2, dtype=torch.int64, device=dev)
        hdr[0] = 1
        self._bcast(hdr)
        qb = torch.empty((batch, dim), dtype=torch.float32, device=dev)
        qb.copy_(torch.zeros((batch, dim), dtype=torch.float32))
        self._bcast(qb)
        _ = int(hdr[0]), qb.cpu()
        gather_and_merge(np.full((batch, self.k), SENTINEL, np.uint32), np.full((batch, self.k), np.inf, np.float32),
                         self.k, group=self.group, device=self.device)
        if dev.type == "cuda":
            torch.cuda.synchronize(dev)

    def _bcast(self, t):
        import torch.distributed as dist
        src = dist.get_global_rank(self.group, 0) if self.group is not None else 0
        dist.broadcast(t, src=src, group=self.group)
        return t

    def serve(self, queries=None, batch: int = 256, tag0: int = 0, timeout_s: float = 60.0):
        """Collective (every rank calls it).  queries: [nq, d] fp32 on group
        rank 0 (ignored elsewhere).  Returns merged (ids [nq, k], dists) on
        every rank."""
        import time

        import torch
        import torch.distributed as dist
        dev = self.device if self.device is not None else torch.device("cpu")
        me = dist.get_rank(self.group)
        hdr = torch.zeros(2, dtype=torch.int64, device=dev)
        if me == 0:
            hdr[0], hdr[1] = int(queries.shape[0]), int(queries.shape[1])
        self._bcast(hdr)
        nq, d = int(hdr[0]), int(hdr[1])
        spans = [(lo, min(nq, lo + batch)) for lo in range(0, nq, batch)]
        for lo, hi in spans:  # broadcast + enqueue every batch
            qb = torch.empty((hi - lo, d), dtype=torch.float32, device=dev)
            if me == 0:
                qb.copy_(torch.from_numpy(np.ascontiguousarray(queries[lo:hi], dtype=np.float32)))
            self._bcast(qb)
            self.server.enqueue(np.ascontiguousarray(qb.cpu().numpy()), tag0=tag0 + lo)
        out_i = np.empty((nq, self.k), np.uint32)
        out_d = np.empty((nq, self.k), np.float32)
        got_i = np.full((nq, self.k), SENTINEL, np.uint32)
        got_d = np.full((nq, self.k), np.inf, np.float32)
        have = np.zeros(nq, bool)
        t0 = time.time()
        for lo, hi in spans:  # collect in batch order, exchange + merge each batch
            while not have[lo:hi].all():
                if time.time() - t0 > timeout_s:
                    raise TimeoutError(f"rank {me}: shard results missing after {timeout_s} s")
                tags, ids, ds, _ = self.server.poll(1024)
                for t, i, dd in zip(tags, ids, ds):
                    q = int(t) - tag0
                    got_i[q], got_d[q] = i[:self.k], dd[:self.k]
                    have[q] = True
                if len(tags) == 0:
                    time.sleep(0.0002)
            gi, gd = gather_and_merge(to_global(got_i[lo:hi], self.offset), got_d[lo:hi], self.k,
                                      group=self.group, device=self.device)
            out_i[lo:hi], out_d[lo:hi] = gi, gd
        return out_i, out_d
