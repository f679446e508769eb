"""Host logic of the multi-GPU mode (paper_conf_ipps_sahunk25_b200/distributed.py)
on CPU: world_size 2 over gloo, the per-shard sweep played by the oracle's
per-vertex decision (oracle.vertex_best), compared with a single-process
emulation of the same bulk-synchronous protocol."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_ipps_sahunk25_b200 import distributed as D


class OracleShardRunner:
    """Asynchronous lpaMove restricted to rows [b, e) (Algorithm 1 with the
    oracle's c* per vertex), on a replicated label vector."""

    def __init__(self, g, b, e, bounds):
        self.h = oracle.CSR.from_graph(g)
        self.N_global = g.N
        self.row_begin, self.row_end = b, e
        self.bounds = bounds
        self.labels = torch.empty(g.N, dtype=torch.int32)
        self.flags = torch.empty(g.N, dtype=torch.uint8)

    def reset(self):
        self.labels.copy_(torch.arange(self.N_global, dtype=torch.int32))
        self.flags.fill_(1)

    # exchange primitives (reference semantics of the CUDA kernels behind
    # nulpa_pack_changed / nulpa_apply_pairs / nulpa_pack_flag_bits /
    # nulpa_or_flag_bits)
    def snapshot(self):
        self.prev = self.labels[self.row_begin:self.row_end].clone()

    def pack_changed(self, pairs):
        cur = self.labels[self.row_begin:self.row_end]
        idx = torch.nonzero(cur != self.prev).flatten()
        k = idx.numel()
        pairs[:k] = ((idx + self.row_begin).to(torch.int64) << 32) | cur[idx].to(torch.int64)
        return k

    def apply_pairs(self, pairs, n):
        p = pairs[:n]
        p = p[p >= 0]
        self.labels[p >> 32] = (p & 0xFFFFFFFF).to(torch.int32)

    def pack_flag_bits(self, bounds, P, words, bits):
        weights = (torch.ones(32, dtype=torch.int64) << torch.arange(32))
        for q in range(P):
            b, e = int(bounds[q]), int(bounds[q + 1])
            seg = torch.zeros(words * 32, dtype=torch.int64)
            seg[: e - b] = self.flags[b:e].to(torch.int64) != 0
            x = (seg.view(words, 32) * weights).sum(1)
            bits[q * words:(q + 1) * words] = (x - ((x >> 31) << 32)).to(torch.int32)   # two's complement int32
        self.flags[:self.row_begin] = 0
        self.flags[self.row_end:] = 0

    def or_flag_bits(self, bits, P, words):
        x = torch.zeros(words, dtype=torch.int64)
        for q in range(P):
            x |= bits[q * words:(q + 1) * words].to(torch.int64) & 0xFFFFFFFF
        n = self.row_end - self.row_begin
        unpacked = ((x.view(words, 1) >> torch.arange(32)) & 1).flatten()[:n]
        self.flags[self.row_begin:self.row_end] = unpacked.to(torch.uint8)

    def sweep(self, pickless):
        C = self.labels.numpy()
        U = self.flags.numpy()
        off, idx = self.h.offsets, self.h.indices
        dn = 0
        for i in range(self.row_begin, self.row_end):
            if not U[i]:
                continue
            U[i] = 0
            c, _, _ = oracle.vertex_best(self.h, i, C)
            if c != oracle.EMPTY and c != C[i] and (not pickless or c <= C[i]):
                C[i] = c
                dn += 1
                U[idx[off[i]:off[i + 1]]] = 1
        return dn


def emulate(g, world, tol=0.05, max_it=20, rho=4):
    """Single-process emulation: every shard sweeps from the same snapshot."""
    bounds = D.partition_by_edges(g.offsets, world)
    N = g.N
    C = np.arange(N, dtype=np.int32)
    owned = [np.zeros(N, dtype=np.uint8) for _ in range(world)]
    for r, (b, e) in enumerate(bounds):
        owned[r][b:e] = 1
    changed = []
    for l in range(max_it):
        pl = rho > 0 and l % rho == 0
        newC = C.copy()
        newU = np.zeros(N, dtype=np.uint8)
        dn = 0
        for r, (b, e) in enumerate(bounds):
            run = OracleShardRunner(g, b, e, bounds)
            run.labels = torch.from_numpy(C.copy())
            run.flags = torch.from_numpy((U_all if l else np.ones(N, dtype=np.uint8)) * owned[r])
            dn += run.sweep(pl)
            newC[b:e] = run.labels.numpy()[b:e]
            newU = np.maximum(newU, run.flags.numpy())
        C, U_all = newC, newU
        changed.append(dn)
        if not pl and dn / N < tol:
            break
    return C, changed


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    g = synth.sbm(n=1500, community_size=50, avg_degree=10, mu=0.2, seed=5)
    bounds = D.partition_by_edges(g.offsets, world)
    b, e = bounds[rank]
    run = OracleShardRunner(g, b, e, bounds)
    res = D.lpa_distributed(run)
    out[rank] = (run.labels.numpy().copy(), res)
    dist.barrier()
    dist.destroy_process_group()


def test_partition_by_edges_balanced():
    g = synth.web(n=20000, avg_out=20, host_min=4, host_max=3000, seed=3)
    for world in (1, 2, 3, 4, 8):
        bounds = D.partition_by_edges(g.offsets, world)
        assert bounds[0][0] == 0 and bounds[-1][1] == g.N
        assert all(bounds[r][1] == bounds[r + 1][0] for r in range(world - 1))
        edges = [int(g.offsets[e] - g.offsets[b]) for b, e in bounds]
        assert sum(edges) == g.M
        maxdeg = int(g.degrees().max())
        assert max(edges) <= g.M / world + maxdeg


def test_shard_graph_rebases_rows():
    g = synth.sbm(n=1000, community_size=50, avg_degree=8, seed=1)
    for r in range(3):
        sh = D.shard_graph(g.offsets, g.indices, None, r, 3)
        assert int(sh.offsets[0]) == 0
        assert int(sh.offsets[-1]) == sh.indices.numel()
        b = sh.row_begin
        for i in [0, sh.n_rows // 2, sh.n_rows - 1]:
            got = sh.indices[sh.offsets[i]:sh.offsets[i + 1]]
            ref = g.indices[g.offsets[b + i]:g.offsets[b + i + 1]]
            assert torch.equal(got, ref)


def test_two_rank_gloo_matches_emulation():
    world = 2
    port = _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(world, port, out), nprocs=world, join=True)
    (C0, r0), (C1, r1) = out[0], out[1]
    assert np.array_equal(C0, C1), "replicated labels differ between ranks"
    strip = lambda r: {k: v for k, v in r.items() if k != "exchange"}   # bytes sent differ per rank
    assert strip(r0) == strip(r1)
    assert [x["labels"] for x in r0["exchange"]] == [x["labels"] for x in r1["exchange"]]
    g = synth.sbm(n=1500, community_size=50, avg_degree=10, mu=0.2, seed=5)
    C, changed = emulate(g, world)
    assert r0["changed"] == changed
    assert np.array_equal(C0, C)
    assert r0["converged"]
    q = oracle.modularity(oracle.CSR.from_graph(g), C0)
    assert q > 0.5
    # the first sweep changes every label (dense all-gather), later sweeps
    # send only the changed ones as pairs
    modes = [x["labels"] for x in r0["exchange"]]
    assert modes[0] == "dense" and "sparse" in modes, modes
    assert [x["dn"] for x in r0["exchange"]] == changed


def test_exchange_primitives_reference():
    """The pair / bitmap encodings used by the exchange round-trip."""
    g = synth.sbm(n=300, community_size=30, avg_degree=6, seed=2)
    bounds = D.partition_by_edges(g.offsets, 3)
    run = OracleShardRunner(g, *bounds[1], bounds)
    run.reset()
    run.snapshot()
    b, e = bounds[1]
    run.labels[b + 3] = 7
    run.labels[e - 1] = 0
    pairs = torch.full((e - b,), -5, dtype=torch.int64)
    k = run.pack_changed(pairs)
    assert k == 2
    other = OracleShardRunner(g, *bounds[0], bounds)
    other.reset()
    other.apply_pairs(torch.cat([pairs[:k], torch.tensor([-1])]), k + 1)
    assert int(other.labels[b + 3]) == 7 and int(other.labels[e - 1]) == 0
    assert int((other.labels != torch.arange(g.N, dtype=torch.int32)).sum()) == 2
    # bitmaps: rank 1's marks on every range, OR-ed into each owner
    rng = np.random.default_rng(0)
    fl = torch.from_numpy((rng.random(g.N) < 0.3).astype(np.uint8))
    run.flags.copy_(fl)
    words = (max(e_ - b_ for b_, e_ in bounds) + 31) // 32
    bits = torch.zeros(3 * words, dtype=torch.int32)
    bt = torch.tensor([x for x, _ in bounds] + [bounds[-1][1]])
    run.pack_flag_bits(bt, 3, words, bits)
    assert int(run.flags[:b].sum()) == 0 and int(run.flags[e:].sum()) == 0
    for q in range(3):
        own = OracleShardRunner(g, *bounds[q], bounds)
        own.flags.zero_()
        recv = torch.zeros(3 * words, dtype=torch.int32)
        recv[words:2 * words] = bits[q * words:(q + 1) * words]     # from rank 1
        own.or_flag_bits(recv, 3, words)
        qb, qe = bounds[q]
        assert torch.equal(own.flags[qb:qe], fl[qb:qe])
