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
    assert r0 == r1
    g = synth.sbm(n=1500, community_size=50, avg_degree=10, mu=0.2, seed=5)
    C, changed = emulate(g, world)
    assert r0["changed"] == changed
    assert np.array_equal(C0, C)
    assert r0["converged"]
    q = oracle.modularity(oracle.CSR.from_graph(g), C0)
    assert q > 0.5
