"""Seeded synthetic inputs shared by the oracle side and the CUDA side.

Holds none of the method's arithmetic (no distances, no search, no graph
logic): only random-number recipes that shape the inputs like the paper's
workloads (Table III) and BASELINE.json's configs.  The recipe is
stated in DESIGN.md §4 ("Input recipe").

Workloads (BASELINE.json ``configs``):
  C1  10k x 128  fp32 L2, clustered, R=32 plain kNN graph, 100 queries, k=10
  C2  1M  x 128  fp32 L2 (SIFT1M-shaped),  R=64, k=10
  C3  1M  x 960  fp32 L2 (GIST1M-shaped),  R=64, k=10
  C4  1.2M x 100 inner product (GloVe-100-shaped, unit-normalised), R=64, k=100
  C5  100M x 96  fp32 L2 (DEEP-shaped, unit-normalised), sharded: 8 shards
      generated on the device from (seed, shard) (shard_vectors_device);
      C5s = one of them (12.5M x 96), what one B200 holds at G = 8
"""
from __future__ import annotations

import dataclasses

import numpy as np

L2 = 0
IP = 1


@dataclasses.dataclass(frozen=True)
class Workload:
    name: str
    n: int
    dim: int
    metric: int
    degree: int
    k: int
    n_queries: int
    knn_degree: int          # degree of the brute-force kNN graph before pruning
    prune: bool
    clusters: int
    rank: int                # intrinsic rank of each cluster's subspace
    spread: float            # within-cluster scale along the subspace
    noise: float             # isotropic noise
    value_scale: float       # affine map to a dataset-like value range
    value_shift: float
    clip0: bool
    normalize: bool
    seed_base: int
    seed_query: int
    center_scale: float = 1.0  # centers ~ N(0, center_scale^2 I)
    shards: int = 0            # > 0: the base set is shard 0 of `shards` per-shard generated parts (C5)
    build: str = "exact"       # graph build: "exact" (kNN + prune) or "partitioned" (R30 / R33)
    part_clusters: int = 0     # partitioned build: clusters (0: n / 4096), overlap, refinement rounds / fan
    part_overlap: int = 2
    refine_rounds: int = 8
    refine_fan: int = 32


WORKLOADS = {
    "C1": Workload("C1-10kx128-L2", 10_000, 128, L2, 32, 10, 100, 32, False,
                   100, 12, 4.0, 0.05, 1.0, 0.0, False, False, 1001, 1002, 0.5),
    "C2": Workload("C2-SIFT1M-shaped-1Mx128-L2", 1_000_000, 128, L2, 64, 10, 10_000, 128, True,
                   1000, 24, 4.0, 0.3, 12.0, 40.0, True, False, 2001, 2002, 0.5),
    # C3 calibrated on the B200 box (scripts/sweep_cfg.py): with 1000 points
    # per cluster, well-separated 960-d clusters make the kNN graph split into
    # per-cluster components (recall ~0.03 from random seeds); overlapping
    # centres (0.15) and a rank-16 subspace give a connected, GIST-hard graph:
    # recall@10 0.85 / 0.95 at L = 128 / 256 with one CTA per query
    "C3": Workload("C3-GIST1M-shaped-1Mx960-L2", 1_000_000, 960, L2, 64, 10, 1_000, 128, True,
                   1000, 16, 4.0, 0.3, 0.08, 0.3, True, False, 3001, 3002, 0.15),
    "C4": Workload("C4-GloVe100-shaped-1.2Mx100-IP", 1_200_000, 100, IP, 64, 100, 10_000, 128, True,
                   1000, 24, 4.0, 0.3, 1.0, 0.0, False, True, 4001, 4002, 0.5),
    "C5": Workload("C5-DEEP100M-shaped-100Mx96-L2", 100_000_000, 96, L2, 64, 10, 10_000, 128, True,
                   10000, 24, 4.0, 0.3, 1.0, 0.0, False, True, 5001, 5002, 0.5, shards=8, build="partitioned"),
    # one shard of C5 at G = 8 (12.5M x 96), generated on the device from (seed, shard) --
    # what one B200 holds and builds in the sharded mode
    "C5s": Workload("C5-shard0of8-DEEP-shaped-12.5Mx96-L2", 12_500_000, 96, L2, 64, 10, 10_000, 128, True,
                    10000, 24, 4.0, 0.3, 1.0, 0.0, False, True, 5001, 5002, 0.5, shards=8, build="partitioned"),
}


def _mixture(rng: np.random.Generator, n: int, dim: int, centers: np.ndarray,
             bases: np.ndarray, spread: float, noise: float, chunk: int = 1 << 18) -> np.ndarray:
    """Gaussian mixture: center_c + spread * z @ basis_c + noise * e, c uniform."""
    K, rank, _ = bases.shape
    c = rng.integers(0, K, size=n)
    z = rng.standard_normal((n, rank), dtype=np.float32)
    out = np.empty((n, dim), np.float32)
    for s in range(0, n, chunk):
        m = min(chunk, n - s)
        out[s:s + m] = rng.standard_normal((m, dim), dtype=np.float32)
    out *= np.float32(noise)
    order = np.argsort(c, kind="stable")
    bounds = np.searchsorted(c[order], np.arange(K + 1))
    for kk in range(K):
        idx = order[bounds[kk]:bounds[kk + 1]]
        if idx.size == 0:
            continue
        out[idx] += centers[kk] + np.float32(spread) * (z[idx] @ bases[kk])
    return out


def _model(w: Workload, dim: int):
    rng = np.random.default_rng(w.seed_base * 7919 + 17)
    centers = np.float32(w.center_scale) * rng.standard_normal((w.clusters, dim), dtype=np.float32)
    bases = rng.standard_normal((w.clusters, w.rank, dim), dtype=np.float32) / np.sqrt(dim)
    return centers, bases.astype(np.float32)


def _finish(w: Workload, x: np.ndarray) -> np.ndarray:
    x = x * np.float32(w.value_scale) + np.float32(w.value_shift)
    if w.clip0:
        np.maximum(x, 0, out=x)
    if w.normalize:
        nrm = np.sqrt((x.astype(np.float64) ** 2).sum(1, keepdims=True))
        nrm[nrm == 0] = 1.0
        x = (x / nrm).astype(np.float32)
    return np.ascontiguousarray(x, dtype=np.float32)


def base_vectors(w: Workload, n: int | None = None) -> np.ndarray:
    n = w.n if n is None else n
    centers, bases = _model(w, w.dim)
    rng = np.random.default_rng(w.seed_base)
    return _finish(w, _mixture(rng, n, w.dim, centers, bases, w.spread, w.noise))


def shard_vectors_device(w: Workload, shard: int, device, n: int | None = None, chunk: int = 1 << 18):
    """Shard `shard` of a sharded base set (C5), generated ON THE DEVICE from
    (seed_base + shard) with torch's generator: the same mixture model (the
    K centres and bases of `_model`, shared by all shards) as base_vectors,
    another random stream.  Returns an (n x dim) float32 CUDA tensor
    (n = w.n, the shard's size)."""
    import torch
    n = w.n if n is None else n
    centers, bases = _model(w, w.dim)
    C = torch.from_numpy(centers).to(device)
    B = torch.from_numpy(bases).to(device)
    g = torch.Generator(device=device)
    g.manual_seed(int(w.seed_base) * 1000 + int(shard))
    out = torch.empty((n, w.dim), dtype=torch.float32, device=device)
    K = B.shape[0]
    for s in range(0, n, chunk):
        m = min(chunk, n - s)
        c = torch.randint(0, K, (m,), generator=g, device=device)
        z = torch.randn((m, w.rank), generator=g, device=device)
        x = torch.randn((m, w.dim), generator=g, device=device) * w.noise
        x += C[c] + w.spread * torch.einsum("mr,mrd->md", z, B[c])
        x = x * w.value_scale + w.value_shift
        if w.clip0:
            x.clamp_(min=0)
        if w.normalize:
            nrm = x.double().pow(2).sum(1, keepdim=True).sqrt()
            nrm[nrm == 0] = 1.0
            x = (x.double() / nrm).float()
        out[s:s + m] = x
    return out


def query_vectors(w: Workload, nq: int | None = None, stream: int = 0) -> np.ndarray:
    """Queries from the base distribution; `stream` selects an independent
    query set (stream 1 = the calibration set used to pick operating points)."""
    nq = w.n_queries if nq is None else nq
    centers, bases = _model(w, w.dim)
    rng = np.random.default_rng(w.seed_query + 1000003 * stream)
    return _finish(w, _mixture(rng, nq, w.dim, centers, bases, w.spread, w.noise))


def lattice(n: int, dim: int, seed: int, metric: int = L2, clusters: int = 16) -> np.ndarray:
    """Integer-lattice twin: coordinates in [0,15] (L2) or [-8,7] (IP), clustered.

    Every partial sum of an L2/IP distance is an integer below 2**24 for
    dim <= 960, so fp32 is exact in any summation order."""
    rng = np.random.default_rng(seed)
    lo, hi = (0, 15) if metric == L2 else (-8, 7)
    centers = rng.integers(lo + 3, hi - 2, size=(clusters, dim))
    c = rng.integers(0, clusters, size=n)
    x = centers[c] + rng.integers(-3, 4, size=(n, dim))
    return np.clip(x, lo, hi).astype(np.float32)


def uniform(n: int, dim: int, seed: int, lo: float = -1.0, hi: float = 1.0) -> np.ndarray:
    rng = np.random.default_rng(seed)
    return rng.uniform(lo, hi, size=(n, dim)).astype(np.float32)


def random_graph(n: int, degree: int, seed: int, sentinel_frac: float = 0.0) -> np.ndarray:
    """Random fixed-degree graph without self loops or repeated neighbours."""
    rng = np.random.default_rng(seed)
    g = np.empty((n, degree), np.uint32)
    for i in range(n):
        cand = rng.choice(n - 1, size=min(degree, n - 1), replace=False)
        cand = cand + (cand >= i)
        row = np.full(degree, 0xFFFFFFFF, np.uint32)
        row[:cand.shape[0]] = cand
        if sentinel_frac > 0:
            drop = rng.random(degree) < sentinel_frac
            row[drop] = 0xFFFFFFFF
        g[i] = row
    return g
