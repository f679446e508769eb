"""Seeded synthetic graph generators -- the ONLY module shared by the oracle
side (tests, cpu_baseline) and the CUDA side (tests, bench, smoke).

Holds none of the method's arithmetic: it only builds CSR graphs (int64
offsets, int32 indices, optional float32 weights) shaped like the paper's
workloads (Table 1: web graphs, social networks, road
networks, protein k-mer graphs) and like BASELINE.json's configs.  Every
generator is a pure function of its arguments and a seed; it runs with torch
on any device (the 2.2B-edge web graph is generated on the GPU).

All graphs are undirected (every edge stored in both directions, PAPER.md:434
"We ensure that the edges are undirected"), simple (no duplicate edges) and,
unless noted, free of self-loops.  Weighted variants draw one float32 weight
in (0, 1] per undirected edge, so w_ij = w_ji.
"""
from __future__ import annotations

import math
import os
from dataclasses import dataclass, field
from typing import Optional

import torch

_DATA = os.path.join(os.path.dirname(os.path.abspath(__file__)), "data")


@dataclass
class Graph:
    offsets: torch.Tensor            # int64 [N+1]
    indices: torch.Tensor            # int32 [M]
    weights: Optional[torch.Tensor]  # float32 [M] or None (unit weights)
    name: str = "graph"
    truth: Optional[torch.Tensor] = None   # planted community per vertex (int64), if any
    meta: dict = field(default_factory=dict)

    @property
    def N(self) -> int:
        return int(self.offsets.numel() - 1)

    @property
    def M(self) -> int:
        return int(self.indices.numel())

    @property
    def device(self):
        return self.indices.device

    def to(self, device) -> "Graph":
        mv = lambda t: None if t is None else t.to(device)
        return Graph(mv(self.offsets), mv(self.indices), mv(self.weights), self.name, mv(self.truth), dict(self.meta))

    def degrees(self) -> torch.Tensor:
        return self.offsets[1:] - self.offsets[:-1]

    def with_unit_weights(self) -> "Graph":
        return Graph(self.offsets, self.indices, None, self.name, self.truth, dict(self.meta))


def _gen(seed: int, device) -> torch.Generator:
    g = torch.Generator(device=device)
    g.manual_seed(int(seed))
    return g


_CHUNK = 1 << 29   # elements per sort / unique call (CUB handles < 2^31)


def from_edges(src: torch.Tensor, dst: torch.Tensor, N: int, *, weighted: bool = False,
               seed: int = 0, name: str = "graph", keep_self_loops: bool = False,
               truth: Optional[torch.Tensor] = None) -> Graph:
    """Build an undirected simple CSR graph from a list of (src, dst) pairs.

    Pairs are canonicalised to (min, max), deduplicated, optionally given one
    weight each, then emitted in both directions and sorted by (src, dst).
    Large inputs are processed in vertex-range buckets (sorts stay < 2^31)."""
    device = src.device
    src = src.to(torch.int64)
    dst = dst.to(torch.int64)
    if not keep_self_loops:
        keep = src != dst
        src, dst = src[keep], dst[keep]
    lo = torch.minimum(src, dst)
    hi = torch.maximum(src, dst)
    del src, dst
    key = lo * N + hi
    del hi
    nb = max(1, -(-key.numel() // _CHUNK))
    if nb == 1:
        del lo
        key = torch.unique(key)                  # sorted, deduplicated undirected edges
    else:
        # bucket by the smaller endpoint: sorted order is preserved bucket by bucket
        bucket = (lo * nb) // max(N, 1)
        del lo
        parts = []
        for bk in range(nb):
            parts.append(torch.unique(key[bucket == bk]))
        del bucket, key
        key = torch.cat(parts)
        del parts
    u = key // N
    v = key - u * N
    del key
    w_und = None
    if weighted:
        g = _gen(seed ^ 0x5EED, device)
        # float32 in (0, 1]: 1 - U[0,1)
        w_und = 1.0 - torch.rand(u.numel(), generator=g, device=device, dtype=torch.float32)
    # directed entries, bucketed by source vertex range
    m_dir = 2 * u.numel()
    nbd = max(1, -(-m_dir // _CHUNK))
    ind_parts, w_parts = [], []
    counts = torch.zeros(N, dtype=torch.int64, device=device)
    for bk in range(nbd):
        a0, a1 = (N * bk) // nbd, (N * (bk + 1)) // nbd
        mu = (u >= a0) & (u < a1)
        mv = (v >= a0) & (v < a1) & (u != v)          # a self-loop is stored once
        s_b = torch.cat([u[mu], v[mv]])
        d_b = torch.cat([v[mu], u[mv]])
        w_b = None if w_und is None else torch.cat([w_und[mu], w_und[mv]])
        del mu, mv
        dkey = s_b * N + d_b
        del d_b
        if w_b is None:
            dkey, _ = torch.sort(dkey)
        else:
            dkey, perm = torch.sort(dkey)
            w_parts.append(w_b[perm])
            del perm, w_b
        srt_s = dkey // N
        ind_parts.append((dkey - srt_s * N).to(torch.int32))
        counts += torch.bincount(srt_s, minlength=N)
        del dkey, srt_s, s_b
    del u, v, w_und
    indices = torch.cat(ind_parts) if len(ind_parts) > 1 else ind_parts[0]
    weights = None if not w_parts else (torch.cat(w_parts) if len(w_parts) > 1 else w_parts[0])
    del ind_parts, w_parts
    offsets = torch.zeros(N + 1, dtype=torch.int64, device=device)
    torch.cumsum(counts, 0, out=offsets[1:])
    return Graph(offsets, indices, weights, name, truth)


# --------------------------------------------------------------------------
# tiny / hand-made graphs
# --------------------------------------------------------------------------

def karate(device="cpu") -> Graph:
    """Zachary's karate club (34 vertices, 78 edges), BASELINE.json configs[0]."""
    rows = []
    with open(os.path.join(_DATA, "karate.edges")) as f:
        for line in f:
            line = line.strip()
            if line and not line.startswith("#"):
                a, b = line.split()
                rows.append((int(a), int(b)))
    e = torch.tensor(rows, dtype=torch.int64, device=device)
    g = from_edges(e[:, 0], e[:, 1], 34, name="karate")
    return g


def cliques(sizes, *, permute: bool = False, seed: int = 0, device="cpu", weighted: bool = False) -> Graph:
    """Disjoint cliques of the given sizes (a size-1 clique is an isolated vertex).
    `truth` holds the clique index of every vertex."""
    N = int(sum(sizes))
    ids = torch.arange(N, dtype=torch.int64, device=device)
    if permute:
        ids = torch.randperm(N, generator=_gen(seed, device), device=device)
    src, dst, truth = [], [], torch.empty(N, dtype=torch.int64, device=device)
    base = 0
    for k, s in enumerate(sizes):
        members = ids[base:base + s]
        truth[members] = k
        if s > 1:
            a, b = torch.triu_indices(s, s, 1, device=device)
            src.append(members[a])
            dst.append(members[b])
        base += s
    if src:
        src = torch.cat(src)
        dst = torch.cat(dst)
    else:
        src = dst = torch.empty(0, dtype=torch.int64, device=device)
    return from_edges(src, dst, N, weighted=weighted, seed=seed, name="cliques", truth=truth)


def path(n: int, device="cpu") -> Graph:
    a = torch.arange(n - 1, dtype=torch.int64, device=device)
    return from_edges(a, a + 1, n, name="path")


def star(n_leaves: int, device="cpu") -> Graph:
    leaves = torch.arange(1, n_leaves + 1, dtype=torch.int64, device=device)
    return from_edges(torch.zeros_like(leaves), leaves, n_leaves + 1, name="star")


def erdos_renyi(n: int, m: int, *, seed: int = 0, device="cpu", weighted: bool = False) -> Graph:
    g = _gen(seed, device)
    s = torch.randint(0, n, (m,), generator=g, device=device)
    d = torch.randint(0, n, (m,), generator=g, device=device)
    return from_edges(s, d, n, weighted=weighted, seed=seed, name="er")


# --------------------------------------------------------------------------
# paper-shaped workloads
# --------------------------------------------------------------------------

def sbm(n: int = 1_000_000, community_size: int = 1000, avg_degree: float = 20.0, mu: float = 0.15, *,
        seed: int = 0, device="cpu", weighted: bool = False, permute: bool = True) -> Graph:
    """Planted-partition SBM (BASELINE.json configs[1]: 1M vertices / 20M edges).

    Vertex v belongs to community (v' // community_size) where v' is v's
    position before a seeded random relabelling (so communities are not
    contiguous ID ranges).  Each vertex draws avg_degree/2 edge endpoints: a
    fraction 1-mu inside its community (uniform), mu anywhere (uniform)."""
    g = _gen(seed, device)
    k = (n + community_size - 1) // community_size
    half = int(round(avg_degree / 2))
    src = torch.arange(n, dtype=torch.int64, device=device).repeat_interleave(half)
    comm = src // community_size
    cstart = comm * community_size
    csize = torch.clamp(torch.full_like(cstart, n) - cstart, max=community_size)
    local = torch.rand(src.numel(), generator=g, device=device) >= mu
    r = torch.rand(src.numel(), generator=g, device=device, dtype=torch.float64)
    dst_local = cstart + torch.clamp((r * csize).to(torch.int64), max=community_size - 1)
    dst_local = torch.minimum(dst_local, cstart + csize - 1)
    dst_global = torch.randint(0, n, (src.numel(),), generator=g, device=device)
    dst = torch.where(local, dst_local, dst_global)
    truth = torch.arange(n, dtype=torch.int64, device=device) // community_size
    if permute:
        perm = torch.randperm(n, generator=g, device=device)   # old id -> new id
        src, dst = perm[src], perm[dst]
        t2 = torch.empty_like(truth)
        t2[perm] = truth
        truth = t2
    gr = from_edges(src, dst, n, weighted=weighted, seed=seed, name="sbm", truth=truth)
    gr.meta.update(dict(community_size=community_size, mu=mu, communities=k))
    return gr


def rmat(scale: int = 22, edge_factor: float = 8.8, abcd=(0.57, 0.19, 0.19, 0.05), *, seed: int = 0,
         device="cpu", weighted: bool = False, chunk: int = 1 << 26) -> Graph:
    """R-MAT graph (Chakrabarti et al.), social-network shaped
    (BASELINE.json configs[2]: ~4M vertices / 70M edges, com-LiveJournal-like)."""
    g = _gen(seed, device)
    n = 1 << scale
    m = int(n * edge_factor)
    a, b, c, _ = abcd
    srcs, dsts = [], []
    for s0 in range(0, m, chunk):
        cnt = min(chunk, m - s0)
        src = torch.zeros(cnt, dtype=torch.int64, device=device)
        dst = torch.zeros(cnt, dtype=torch.int64, device=device)
        for lvl in range(scale):
            r = torch.rand(cnt, generator=g, device=device)
            bit_s = (r >= a + b).to(torch.int64)                 # quadrant c or d
            bit_d = (((r >= a) & (r < a + b)) | (r >= a + b + c)).to(torch.int64)  # b or d
            src |= bit_s << lvl
            dst |= bit_d << lvl
        srcs.append(src)
        dsts.append(dst)
    src = torch.cat(srcs)
    dst = torch.cat(dsts)
    # relabel so vertex 0 is not always the mega-hub (seeded permutation)
    perm = torch.randperm(n, generator=g, device=device)
    return from_edges(perm[src], perm[dst], n, weighted=weighted, seed=seed, name="rmat")


def road(R: int = 1600, mean_chain: float = 9.5, keep: float = 0.92, *, seed: int = 0, device="cpu",
         weighted: bool = False) -> Graph:
    """Road-network-like mesh (BASELINE.json configs[3]: ~50M vertices /
    110M edges, europe_osm-shaped, average degree ~2.1).

    An R x R lattice of intersections; each lattice edge is kept with
    probability `keep` and subdivided by a chain of Uniform{0..2*mean_chain}
    degree-2 vertices.  IDs are spatially local: intersection p is followed by
    the chain vertices of its right and down edges."""
    g = _gen(seed, device)
    P = R * R
    pid = torch.arange(P, dtype=torch.int64, device=device)
    row, col = pid // R, pid % R
    has_r = (col < R - 1) & (torch.rand(P, generator=g, device=device) < keep)
    has_d = (row < R - 1) & (torch.rand(P, generator=g, device=device) < keep)
    hi = int(round(2 * mean_chain))
    s_r = torch.randint(0, hi + 1, (P,), generator=g, device=device) * has_r
    s_d = torch.randint(0, hi + 1, (P,), generator=g, device=device) * has_d
    block = 1 + s_r + s_d
    base = torch.cumsum(block, 0) - block            # id of intersection p
    N = int(block.sum())

    def chains(has, s, nbr, first):
        # edges along: p -> c_1 -> ... -> c_s -> nbr, chain ids first..first+s-1
        p = pid[has]
        s = s[has]
        a = base[p]
        b = base[nbr[has]]
        f = first[has]
        L = s + 1                                     # edges per chain
        tot = int(L.sum())
        e_chain = torch.repeat_interleave(torch.arange(p.numel(), device=device), L)
        start = torch.cumsum(L, 0) - L
        k = torch.arange(tot, device=device) - start[e_chain]   # 0..s
        sc = s[e_chain]
        fc = f[e_chain]
        u = torch.where(k == 0, a[e_chain], fc + k - 1)
        v = torch.where(k == sc, b[e_chain], fc + k)
        return u, v

    nbr_r = torch.clamp(pid + 1, max=P - 1)
    nbr_d = torch.clamp(pid + R, max=P - 1)
    u1, v1 = chains(has_r, s_r, nbr_r, base + 1)
    u2, v2 = chains(has_d, s_d, nbr_d, base + 1 + s_r)
    gr = from_edges(torch.cat([u1, u2]), torch.cat([v1, v2]), N, weighted=weighted, seed=seed, name="road")
    return gr


def kmer(n: int = 1_000_000, branch: float = 0.05, *, seed: int = 0, device="cpu", weighted: bool = False) -> Graph:
    """Protein k-mer-graph-like (kmer_A2a/kmer_V1r: average
    degree ~2.1, mostly long unbranched paths, vertex IDs with no locality):
    a random ordering of the vertices is cut into paths, plus a fraction
    `branch` of random extra edges joining path vertices."""
    g = _gen(seed, device)
    order = torch.randperm(n, generator=g, device=device)
    cut = torch.rand(n - 1, generator=g, device=device) < 0.002   # break into paths
    a = order[:-1][~cut]
    b = order[1:][~cut]
    nb = int(n * branch / 2)
    xa = torch.randint(0, n, (nb,), generator=g, device=device)
    xb = torch.randint(0, n, (nb,), generator=g, device=device)
    return from_edges(torch.cat([a, xa]), torch.cat([b, xb]), n, weighted=weighted, seed=seed, name="kmer")


def web(n: int = 40_000_000, avg_out: float = 58.0, p_local: float = 0.95, gamma: float = 3.6,
        host_alpha: float = 1.4, host_min: int = 16, host_max: int = 400_000, max_out: int = 20_000, *,
        locality: str = "loguniform", global_target: str = "page", seed: int = 0, device="cpu",
        weighted: bool = False,
        chunk: int = 1 << 28) -> Graph:
    """Web-graph-like power-law graph (BASELINE.json configs[4]: ~40M vertices /
    2.2B edges, it-2004-shaped).

    Shape of the LAW crawls: vertex IDs in URL order, so pages of one host are
    a contiguous ID range (host sizes ~ Pareto(host_alpha) in
    [host_min, host_max]); out-degrees log-normal with mean `avg_out`; each
    link stays inside its host with probability p_local (uniform target),
    uniform over the host (locality="uniform") or at a log-uniform ID distance
    (locality="loguniform", the default: URL-ordered crawls link mostly to
    nearby pages), otherwise it points to a globally popular page: rank floor(n * U^gamma)
    through a seeded permutation, which gives power-law in-degrees
    (rank^(1/gamma - 1)) and hubs with ~10^6 neighbours at full size."""
    g = _gen(seed, device)
    # host partition
    est = int(n / max(host_min, 1)) + 16
    u = torch.rand(est, generator=g, device=device, dtype=torch.float64)
    hs = torch.clamp((host_min * u.pow(-1.0 / host_alpha)).to(torch.int64), max=host_max)
    cs = torch.cumsum(hs, 0)
    nh = int(torch.searchsorted(cs, torch.tensor([n], device=device)).item()) + 1
    hs = hs[:nh].clone()
    hs[-1] -= int(cs[nh - 1].item()) - n
    hstart = torch.cumsum(hs, 0) - hs
    host_of = torch.repeat_interleave(torch.arange(nh, device=device), hs)
    # out-degrees
    sigma = 1.1
    mu_ln = math.log(avg_out) - sigma * sigma / 2
    z = torch.randn(n, generator=g, device=device)
    deg = torch.clamp(torch.exp(mu_ln + sigma * z).round().to(torch.int64), 1, max_out)
    perm = torch.randperm(n, generator=g, device=device)
    hperm = torch.randperm(nh, generator=g, device=device)
    total = int(deg.sum())
    srcs, dsts = [], []
    cdeg = torch.cumsum(deg, 0)
    v0 = 0
    while v0 < n:
        # vertices [v0, v1) whose edges fit in one chunk
        lim = (cdeg[v0 - 1] if v0 > 0 else 0) + chunk
        v1 = int(torch.searchsorted(cdeg, torch.as_tensor([lim], device=device), right=True).item())
        v1 = max(v1, v0 + 1)
        v1 = min(v1, n)
        vv = torch.arange(v0, v1, device=device)
        src = torch.repeat_interleave(vv, deg[v0:v1])
        cnt = src.numel()
        h = host_of[src]
        loc = torch.rand(cnt, generator=g, device=device) < p_local
        r = torch.rand(cnt, generator=g, device=device, dtype=torch.float64)
        if locality == "uniform":
            dl = hstart[h] + (r * hs[h]).to(torch.int64)
        else:
            # URL-order locality: distance to the target page log-uniform in
            # [1, host size], either direction, wrapped inside the host
            hsz = hs[h]
            dist = torch.exp(r * torch.log(hsz.to(torch.float64))).to(torch.int64)
            sign = torch.rand(cnt, generator=g, device=device) < 0.5
            dist = torch.where(sign, dist, -dist)
            dl = hstart[h] + torch.remainder(src - hstart[h] + dist, hsz)
        r2 = torch.rand(cnt, generator=g, device=device, dtype=torch.float64)
        if global_target == "page":
            dg = perm[torch.clamp((n * r2.pow(gamma)).to(torch.int64), max=n - 1)]
        else:
            # links into another host land on its home page (first ID of the
            # host: the root URL sorts first); hosts chosen by popularity
            hp = hperm[torch.clamp((nh * r2.pow(gamma)).to(torch.int64), max=nh - 1)]
            dg = hstart[hp]
        dst = torch.where(loc, dl, dg)
        srcs.append(src)
        dsts.append(dst)
        del h, loc, r, dl, r2, dg
        v0 = v1
    src = torch.cat(srcs)
    dst = torch.cat(dsts)
    del srcs, dsts
    gr = from_edges(src, dst, n, weighted=weighted, seed=seed, name="web",
                    truth=host_of.to(torch.int64))
    gr.meta.update(dict(hosts=nh, directed_links=total))
    return gr


# named BASELINE.json configurations --------------------------------------------

CONFIGS = {
    "karate": dict(fn="karate", kw={}),
    "sbm_1m_20m": dict(fn="sbm", kw=dict(n=1_000_000, community_size=1000, avg_degree=20.0, mu=0.15)),
    "rmat_4m_70m": dict(fn="rmat", kw=dict(scale=22, edge_factor=8.8)),
    "road_50m_110m": dict(fn="road", kw=dict(R=1600, mean_chain=9.5)),
    "web_40m_2200m": dict(fn="web", kw=dict(n=40_000_000)),
    # north star "k-mer workloads": kmer_A2a-shaped (171M / 361M)
    "kmer_171m_360m": dict(fn="kmer", kw=dict(n=171_000_000)),
}


def make(config: str, *, device="cpu", seed: int = 0, weighted: bool = False, **overrides) -> Graph:
    c = CONFIGS[config]
    fn = globals()[c["fn"]]
    kw = dict(c["kw"])
    kw.update(overrides)
    if c["fn"] == "karate":
        return fn(device=device)
    return fn(seed=seed, device=device, weighted=weighted, **kw)
