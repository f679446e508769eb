"""Multi-GPU nu-LPA: one process per GPU, torch.distributed (NCCL) plumbing.

Row a/e of DESIGN.md section 8 (north star "8-GPU mode"): the vertex range
is split into contiguous ranges holding ~|E|/P CSR entries each
(``partition_by_edges``); every rank sweeps its own rows (Algorithm 1's
lpaMove, through ``nulpa_sweep`` on a shard handle)
against a REPLICATED label vector, then

  * the labels of every rank's range are exchanged with an all-gather
    (``all_gather_into_tensor`` over a padded [P, max_rows] staging buffer);
  * the "unprocessed" marks a rank set on other ranks' vertices are merged
    with a reduce-scatter(MAX) over the same padded layout: each rank
    receives the maximum of everybody's marks for its own rows only;
  * dN is all-reduced (SUM) and Algorithm 1's tolerance / Pick-Less loop
     runs identically on every rank.

Within a rank the sweep is asynchronous (in-place labels); across ranks it
is bulk-synchronous (remote labels are one sweep old).  The driver only
moves tensors: all label computation happens in the CUDA kernels behind the
C ABI (``CudaShardRunner``).  A runner is any object with ``N_global``,
``row_begin``, ``row_end``, ``labels`` (int32 [N]), ``flags`` (uint8 [N]),
``reset()`` and ``sweep(pickless) -> int``, so the host logic can be tested
with the gloo backend on CPU.
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import List, Optional, Tuple

import torch
import torch.distributed as dist


def partition_by_edges(offsets: torch.Tensor, world: int) -> List[Tuple[int, int]]:
    """Split [0, N) into `world` contiguous vertex ranges with ~M/world CSR
    entries each: boundary r is the first vertex whose offset >= r*M/world."""
    N = int(offsets.numel() - 1)
    M = int(offsets[-1])
    targets = torch.tensor([(r * M) // world for r in range(1, world)], dtype=torch.int64, device=offsets.device)
    cuts = torch.searchsorted(offsets[:N].contiguous(), targets, right=False).tolist() if world > 1 else []
    b = [0] + [int(c) for c in cuts] + [N]
    for r in range(1, len(b)):
        b[r] = max(b[r], b[r - 1])
    return [(b[r], b[r + 1]) for r in range(world)]


@dataclass
class Shard:
    offsets: torch.Tensor          # int64 [n_rows+1], rebased to 0
    indices: torch.Tensor          # int32 [m] global neighbour IDs
    weights: Optional[torch.Tensor]
    row_begin: int
    row_end: int
    N_global: int
    M_global: int
    bounds: List[Tuple[int, int]]

    @property
    def n_rows(self) -> int:
        return self.row_end - self.row_begin


def shard_graph(offsets, indices, weights, rank: int, world: int) -> Shard:
    bounds = partition_by_edges(offsets, world)
    b, e = bounds[rank]
    e0, e1 = int(offsets[b]), int(offsets[e])
    off = (offsets[b:e + 1] - e0).contiguous().clone()
    idx = indices[e0:e1].contiguous().clone()
    w = None if weights is None else weights[e0:e1].contiguous().clone()
    return Shard(off, idx, w, b, e, int(offsets.numel() - 1), int(offsets[-1]), bounds)


class CudaShardRunner:
    """A shard on this rank's GPU behind the C ABI, with the replicated label
    and flag vectors owned here (torch tensors) and bound into the handle."""

    def __init__(self, shard: Shard, **params):
        import paper_conf_ipps_sahunk25_b200 as nl
        self.nl = nl
        self.shard = shard
        self.N_global = shard.N_global
        self.row_begin, self.row_end = shard.row_begin, shard.row_end
        dev = torch.device("cuda", torch.cuda.current_device())
        self.g = nl.Graph(shard.offsets.to(dev), shard.indices.to(dev),
                          None if shard.weights is None else shard.weights.to(dev),
                          n_global=shard.N_global, row_begin=shard.row_begin)
        self.labels = torch.empty(shard.N_global, dtype=torch.int32, device=dev)
        self.flags = torch.empty(shard.N_global, dtype=torch.uint8, device=dev)
        self.g.bind_state(self.labels, self.flags)
        self.params = nl.nulpa_default_params(**params)
        self.launches = 0

    def reset(self):
        self.g.reset()                       # C <- [0..N), all unprocessed (kernel)

    def sweep(self, pickless: bool) -> int:
        return self.nl.nulpa_sweep(self.g.h, pickless, self.params)

    def modularity_partial(self, Sigma: torch.Tensor):
        return self.nl.nulpa_modularity_partial(self.g.h, self.labels, Sigma)

    def modularity_finish(self, Sigma: torch.Tensor, sigma: float, two_m: float) -> float:
        return self.nl.nulpa_modularity_finish(self.g.h, Sigma, sigma, two_m)


class Exchanger:
    """Per-sweep exchange of labels (all-gather) and flags (reduce-scatter
    MAX: a rank needs only its own rows' flags, so each rank receives the
    element-wise maximum of everybody's marks for its range -- half the bytes
    of an all-reduce of the whole flag vector)."""

    def __init__(self, runner, group=None):
        self.r = runner
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        bounds = getattr(runner, "bounds", None) or runner.shard.bounds
        self.bounds = bounds
        self.maxrows = max(e - b for b, e in bounds)
        dev = runner.labels.device
        self.stage_in = torch.empty(self.maxrows, dtype=torch.int32, device=dev)
        self.stage_out = torch.empty(self.world * self.maxrows, dtype=torch.int32, device=dev)
        self.fstage_in = torch.zeros(self.world * self.maxrows, dtype=torch.uint8, device=dev)
        self.fstage_out = torch.empty(self.maxrows, dtype=torch.uint8, device=dev)
        b, e = bounds[self.rank]
        self.own = (b, e)

    def labels(self):
        b, e = self.own
        self.stage_in[: e - b].copy_(self.r.labels[b:e])
        dist.all_gather_into_tensor(self.stage_out, self.stage_in, group=self.group)
        for q, (qb, qe) in enumerate(self.bounds):
            if q != self.rank and qe > qb:
                self.r.labels[qb:qe].copy_(self.stage_out[q * self.maxrows: q * self.maxrows + (qe - qb)])

    def flags(self):
        f = self.r.flags
        for q, (qb, qe) in enumerate(self.bounds):
            if qe > qb:
                self.fstage_in[q * self.maxrows: q * self.maxrows + (qe - qb)].copy_(f[qb:qe])
        dist.reduce_scatter_tensor(self.fstage_out, self.fstage_in, op=dist.ReduceOp.MAX, group=self.group)
        b, e = self.own
        f[b:e].copy_(self.fstage_out[: e - b])
        self.clear_remote_flags()

    def clear_remote_flags(self):
        b, e = self.own
        self.r.flags[:b].zero_()
        self.r.flags[e:].zero_()

    def changed(self, dn_local: int) -> int:
        t = torch.tensor([dn_local], dtype=torch.int64, device=self.r.labels.device)
        dist.all_reduce(t, op=dist.ReduceOp.SUM, group=self.group)
        return int(t.item())


def lpa_distributed(runner, tolerance: float = 0.05, max_iterations: int = 20, pickless_period: int = 4,
                    group=None, exchanger: Optional[Exchanger] = None) -> dict:
    """Algorithm 1's lpa() over all ranks.  Every rank
    returns the same iteration count and per-iteration global dN; the label
    vector is replicated on every rank at the end."""
    ex = exchanger or Exchanger(runner, group)
    runner.reset()
    ex.clear_remote_flags()                  # each rank owns its rows' flags
    N = runner.N_global
    changed = []
    converged = False
    launches = 0
    for l in range(max_iterations):
        pl = pickless_period > 0 and l % pickless_period == 0
        dn_local = runner.sweep(pl)
        ex.labels()
        ex.flags()
        dn = ex.changed(dn_local)
        changed.append(dn)
        launches += 1
        if not pl and dn / N < tolerance:
            converged = True
            break
    return {"iterations": len(changed), "changed": changed, "converged": converged, "launches": launches}


def modularity_distributed(runner, group=None) -> float:
    """Eq. 1 over all shards: per-shard intra weight and
    K_i scattered into Sigma, all-reduced, finished on every rank."""
    dev = runner.labels.device
    Sigma = torch.zeros(runner.N_global, dtype=torch.float64, device=dev)
    sigma, two_m = runner.modularity_partial(Sigma)
    dist.all_reduce(Sigma, op=dist.ReduceOp.SUM, group=group)
    t = torch.tensor([sigma, two_m], dtype=torch.float64, device=dev)
    dist.all_reduce(t, op=dist.ReduceOp.SUM, group=group)
    return runner.modularity_finish(Sigma, float(t[0]), float(t[1]))
