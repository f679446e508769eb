"""Multi-GPU nu-LPA: one process per GPU, torch.distributed (NCCL) plumbing.

Row a/e of DESIGN.md section 8 (north star "8-GPU mode"): the vertex range
is split into contiguous ranges holding ~|E|/P CSR entries each
(``partition_by_edges``); every rank sweeps its own rows (Algorithm 1's
lpaMove, through ``nulpa_sweep`` on a shard handle)
against a REPLICATED label vector, then

  * only CHANGED labels travel: each rank packs its rows whose label moved
    in this sweep as (vertex, label) pairs (``nulpa_pack_changed``), the
    per-rank counts are all-gathered (their sum is dN), and the pairs are
    all-gathered over a [P, max count] buffer and applied
    (``nulpa_apply_pairs``) -- 8 bytes per changed vertex instead of 4 per
    vertex.  When more than 1/8 of all vertices changed (the first sweeps)
    the label ranges are all-gathered densely instead (4 bytes per vertex,
    ``all_gather_into_tensor`` over a padded [P, max_rows] buffer);
  * the "unprocessed" marks a rank set are exchanged as bitmaps: per rank
    range one bit per vertex (``nulpa_pack_flag_bits``), sent with one
    all-to-all, OR-ed into the owner's flags (``nulpa_or_flag_bits``) --
    N/8 bytes per rank instead of a byte per vertex;
  * Algorithm 1's tolerance / Pick-Less loop runs
    identically on every rank from the global dN.

Within a rank the sweep is asynchronous (in-place labels); across ranks it
is bulk-synchronous (remote labels are one sweep old).  The driver only
moves tensors: all label computation happens in the CUDA kernels behind the
C ABI (``CudaShardRunner``).  A runner is any object with ``N_global``,
``row_begin``, ``row_end``, ``labels`` (int32 [N]), ``flags`` (uint8 [N]),
``reset()``, ``sweep(pickless) -> int`` and the exchange primitives
``snapshot()``, ``pack_changed(pairs) -> int``, ``apply_pairs(pairs, n)``,
``pack_flag_bits(bounds, P, words, bits)``, ``or_flag_bits(bits, P, words)``,
so the host logic can be tested with the gloo backend on CPU.
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

    # exchange primitives (kernels behind the C ABI)
    def snapshot(self):
        if not hasattr(self, "prev"):
            self.prev = torch.empty(max(1, self.row_end - self.row_begin), dtype=torch.int32, device=self.labels.device)
        self.prev[: self.row_end - self.row_begin].copy_(self.labels[self.row_begin:self.row_end])

    def pack_changed(self, pairs: torch.Tensor) -> int:
        return self.nl.nulpa_pack_changed(self.g.h, self.prev, pairs)

    def apply_pairs(self, pairs: torch.Tensor, n: int):
        self.nl.nulpa_apply_pairs(self.g.h, pairs, n)

    def pack_flag_bits(self, bounds: torch.Tensor, P: int, words: int, bits: torch.Tensor):
        self.nl.nulpa_pack_flag_bits(self.g.h, bounds, P, words, bits)

    def or_flag_bits(self, bits: torch.Tensor, P: int, words: int):
        self.nl.nulpa_or_flag_bits(self.g.h, bits, P, words)

    def modularity_partial(self, Sigma: torch.Tensor):
        return self.nl.nulpa_modularity_partial(self.g.h, self.labels, Sigma)

    def modularity_finish(self, Sigma: torch.Tensor, sigma: float, two_m: float) -> float:
        return self.nl.nulpa_modularity_finish(self.g.h, Sigma, sigma, two_m)


class Exchanger:
    """Per-sweep exchange between the ranks (module docstring): changed
    labels as pairs (dense all-gather of the label ranges when more than
    `dense_above` of all vertices changed), marks as bitmaps (all-to-all),
    dN from the all-gathered per-rank change counts.  `log` keeps, per
    sweep, the label mode and the bytes each rank sent."""

    def __init__(self, runner, group=None, dense_above: float = 1.0 / 8.0):
        self.r = runner
        self.group = group
        self.world = dist.get_world_size(group)
        self.rank = dist.get_rank(group)
        bounds = getattr(runner, "bounds", None) or runner.shard.bounds
        self.bounds = bounds
        self.N = runner.N_global
        self.maxrows = max(1, max(e - b for b, e in bounds))
        self.dense_above = dense_above
        dev = runner.labels.device
        self.dev = dev
        self.stage_in = torch.empty(self.maxrows, dtype=torch.int32, device=dev)
        self.stage_out = torch.empty(self.world * self.maxrows, dtype=torch.int32, device=dev)
        self.pairs = torch.empty(self.maxrows, dtype=torch.int64, device=dev)
        self.words = (self.maxrows + 31) // 32
        self.bits_out = torch.empty(self.world * self.words, dtype=torch.int32, device=dev)
        self.bits_in = torch.empty(self.world * self.words, dtype=torch.int32, device=dev)
        self.bounds_t = torch.tensor([b for b, _ in bounds] + [bounds[-1][1]], dtype=torch.int64, device=dev)
        b, e = bounds[self.rank]
        self.own = (b, e)
        self.log = []

    def before_sweep(self):
        self.r.snapshot()

    def exchange(self) -> int:
        """After a sweep: labels, marks; returns the global dN."""
        n_loc = self.r.pack_changed(self.pairs)
        cnt = torch.tensor([n_loc], dtype=torch.int64, device=self.dev)
        counts = torch.empty(self.world, dtype=torch.int64, device=self.dev)
        dist.all_gather_into_tensor(counts, cnt, group=self.group)
        counts = counts.tolist()
        dn = int(sum(counts))
        if dn > self.dense_above * self.N:
            self.labels()
            mode, sent = "dense", 4 * (self.own[1] - self.own[0])
        else:
            m = max(counts)
            if m > 0:
                self.pairs[n_loc:m].fill_(-1)                  # padding, skipped by apply
                recv = torch.empty(self.world * m, dtype=torch.int64, device=self.dev)
                dist.all_gather_into_tensor(recv, self.pairs[:m], group=self.group)
                self.r.apply_pairs(recv, self.world * m)
            mode, sent = "sparse", 8 * m
        self.flags()
        self.log.append({"dn": dn, "labels": mode, "label_bytes_sent": sent,
                         "flag_bytes_sent": 4 * self.words * self.world})
        return dn

    def labels(self):
        """Dense: every rank's label range, all-gathered."""
        b, e = self.own
        self.stage_in[: e - b].copy_(self.r.labels[b:e])
        dist.all_gather_into_tensor(self.stage_out, self.stage_in, group=self.group)
        for q, (qb, qe) in enumerate(self.bounds):
            if q != self.rank and qe > qb:
                self.r.labels[qb:qe].copy_(self.stage_out[q * self.maxrows: q * self.maxrows + (qe - qb)])

    def flags(self):
        """Marks of every rank range as bitmaps, all-to-all, OR-ed into the owner's flags."""
        self.r.pack_flag_bits(self.bounds_t, self.world, self.words, self.bits_out)   # also clears remote flags
        dist.all_to_all_single(self.bits_in, self.bits_out, group=self.group)
        self.r.or_flag_bits(self.bits_in, self.world, self.words)

    def clear_remote_flags(self):
        b, e = self.own
        self.r.flags[:b].zero_()
        self.r.flags[e:].zero_()


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
        ex.before_sweep()
        runner.sweep(pl)
        dn = ex.exchange()
        changed.append(dn)
        launches += 1
        if not pl and dn / N < tolerance:
            converged = True
            break
    return {"iterations": len(changed), "changed": changed, "converged": converged, "launches": launches,
            "exchange": ex.log[-len(changed):]}


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
