"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (default parameters):

* one whole synchronous sweep (lpaMove, Algorithm 1) of
  the 2.2B-edge web graph, the 4M/70M social graph and the 50M/110M road
  graph, compared element by element (all labels, all flags, dN) with
  oracle.lpa_move_sync from the same state;
* the north star's headline quality bar on the 2.2B-edge web graph: every
  one of 6 production (asynchronous) GPU runs on each of 2 generator seeds
  reaches modularity (Eq. 1) >= the asynchronous oracle's
  - 0.02;
* SBM 1M/20M: full oracle runs (sync bit-exact, async quality + NMI).

The oracle is plain single-threaded C; independent oracle calls run in
threads (ctypes releases the GIL), so the module fits the GPU test budget.
"""
import json
import os
import time
from concurrent.futures import ThreadPoolExecutor

import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_ipps_sahunk25_b200 as nl

pytestmark = [pytest.mark.gpu, pytest.mark.slow]

QUALITY_SEEDS = tuple(int(x) for x in os.environ.get("NULPA_FULLSIZE_SEEDS", "0,1").split(","))
QUALITY_RUNS = 6


def host_csr(g, weights=None):
    """The oracle's copy of a device graph (unit weights when None)."""
    return oracle.CSR(g.offsets.cpu().numpy(), g.indices.cpu().numpy(),
                      None if weights is None else weights.cpu().numpy())


def sync_sweep_whole(g, h, weights, C0, U0, pickless):
    """One synchronous sweep on the GPU (bench launch configuration) and in
    the oracle from the same state; every label, every flag and dN equal."""
    gg = nl.Graph(g.offsets, g.indices, weights)
    gg.set_labels(torch.from_numpy(C0).cuda(), torch.from_numpy(U0).cuda())
    gdn = gg.sweep(pickless, mode=nl.SYNC)
    gC = gg.labels(device=False).numpy()
    gU = gg.flags(device=False).numpy()
    gg.close()
    dn, C1, U1, _, _ = oracle.lpa_move_sync(h, C0, U0, pickless)
    assert gdn == dn
    bad = np.nonzero(gC != C1)[0]
    assert bad.size == 0, f"{bad.size} labels differ, e.g. {bad[:10]}"
    badf = np.nonzero(gU != U1)[0]
    assert badf.size == 0, f"{badf.size} flags differ, e.g. {badf[:10]}"
    return dn


def states(N, seed):
    """Two sweep inputs: the first sweep of a run (C = [0..N), all
    unprocessed, Pick-Less on) and a mid-run-like state (labels constant on
    blocks of 32 IDs with a random 1/8 relabelled to a random block, 80% of
    the vertices unprocessed, Pick-Less off)."""
    rng = np.random.default_rng(seed)
    C_init = np.arange(N, dtype=np.int32)
    U_all = np.ones(N, dtype=np.uint8)
    C_mid = (np.arange(N, dtype=np.int64) // 32 * 32).astype(np.int32)
    pick = rng.random(N) < 0.125
    C_mid[pick] = (rng.integers(0, N, int(pick.sum())) // 32 * 32).astype(np.int32)
    U_mid = (rng.random(N) < 0.8).astype(np.uint8)
    return [(C_init, U_all, True), (C_mid, U_mid, False)]


def test_web_2200m_sync_sweep_whole_vector():
    g = synth.make("web_40m_2200m", device="cuda")
    assert 2.0e9 < g.M < 2.4e9
    ones = torch.ones(g.M, dtype=torch.float32, device="cuda")     # the bench's stored weights
    h = host_csr(g)                                                # unit weights: the same exact sums
    for C0, U0, pl in states(g.N, 5):
        sync_sweep_whole(g, h, ones, C0, U0, pl)
    del ones


@pytest.mark.parametrize("config", ["rmat_4m_70m", "road_50m_110m"])
def test_social_and_road_sync_sweep_whole_vector(config):
    g = synth.make(config, device="cuda")
    h = host_csr(g)
    for C0, U0, pl in states(g.N, 6):
        sync_sweep_whole(g, h, None, C0, U0, pl)
    # the production run at full size: converges, modularity >= the
    # asynchronous oracle's - 0.02 (bench configuration: stored weights = ones)
    ones = torch.ones(g.M, dtype=torch.float32, device="cuda")
    gg = nl.Graph(g.offsets, g.indices, ones)
    st = gg.run()
    assert st["converged"] or st["iterations"] == 20
    C_o, _, _ = oracle.lpa(h)
    q_o = oracle.modularity(h, C_o)
    q_g = gg.modularity()
    assert q_g >= q_o - 0.02, (config, q_g, q_o)
    gg.close()


def test_web_2200m_quality_vs_full_oracle():
    """North star headline: on the full 2.2B-edge web graph, every
    asynchronous GPU run (6 per seed, 2 generator seeds, default parameters,
    stored weights = ones as in bench.py) reaches modularity >= the
    asynchronous oracle's - 0.02, converges, and keeps every final label a
    vertex ID.  Eq. 1 on the GPU equals the oracle's on the oracle's labels."""
    out = {"graph": "web_40m_2200m, stored weights = ones", "seeds": {}}
    pool = ThreadPoolExecutor(max_workers=len(QUALITY_SEEDS))

    def run_oracle(h):
        t0 = time.time()
        C, it, dN = oracle.lpa(h)
        return C, it, [int(x) for x in dN], oracle.modularity(h, C), time.time() - t0

    futures, gpu = {}, {}
    for seed in QUALITY_SEEDS:
        g = synth.make("web_40m_2200m", device="cuda", seed=seed)
        h = host_csr(g)
        futures[seed] = (h, pool.submit(run_oracle, h))          # oracle on the host meanwhile
        ones = torch.ones(g.M, dtype=torch.float32, device="cuda")
        gg = nl.Graph(g.offsets, g.indices, ones)
        runs = []
        for _ in range(QUALITY_RUNS):
            st = gg.run()
            C = gg.labels()
            assert st["converged"] and st["iterations"] <= 20
            assert int(C.min()) >= 0 and int(C.max()) < g.N
            runs.append(dict(modularity=gg.modularity(), iterations=st["iterations"], changed=st["changed"]))
        gpu[seed] = (g, gg, runs)
    for seed in QUALITY_SEEDS:
        h, fut = futures[seed]
        C, it, dN, q_or, secs = fut.result()
        g, gg, runs = gpu[seed]
        q_or_gpu = gg.modularity(torch.from_numpy(C).cuda())
        out["seeds"][seed] = dict(oracle=dict(modularity=q_or, iterations=it, changed=dN, seconds=round(secs, 1)),
                                  gpu_async_runs=runs)
        assert abs(q_or - q_or_gpu) < 1e-6             # Eq. 1 on the GPU agrees with the oracle's
        gg.close()
    pool.shutdown()
    print(json.dumps(out))
    path = os.environ.get("NULPA_FULLSIZE_OUT")
    if path:
        with open(path, "w") as f:
            json.dump(out, f, indent=1)
    for seed, d in out["seeds"].items():
        q_or = d["oracle"]["modularity"]
        qs = [r["modularity"] for r in d["gpu_async_runs"]]
        assert min(qs) >= q_or - 0.02, (seed, qs, q_or)


def test_sbm_1m_full_oracle_runs():
    g = synth.make("sbm_1m_20m")
    h = oracle.CSR.from_graph(g)
    gg = nl.Graph(g.offsets.cuda(), g.indices.cuda())
    # synchronous mode: the full run is bit-exact
    C, it, dn = oracle.lpa(h, sync=True)
    st = gg.run(mode=nl.SYNC)
    assert st["iterations"] == it and st["changed"] == list(dn)
    assert np.array_equal(gg.labels(device=False).numpy(), C)
    # asynchronous: modularity within 0.02 of the oracle's, NMI >= 0.9x
    Co, _, _ = oracle.lpa(h)
    qo = oracle.modularity(h, Co)
    st = gg.run()
    Cg = gg.labels(device=False).numpy()
    qg = oracle.modularity(h, Cg)
    assert st["converged"]
    assert qg >= qo - 0.02, (qg, qo)
    t = g.truth.numpy()
    assert oracle.nmi(Cg, t) >= 0.9 * oracle.nmi(Co, t)
    assert abs(gg.modularity() - qg) < 1e-9


def test_web_2200m_async_first_sweep_invariants():
    """The production first sweep (Pick-Less) at full size: no label
    increases, every changed vertex took a label one of its neighbours held
    before or after the sweep (sampled), dN = number of changed labels."""
    g = synth.make("web_40m_2200m", device="cuda")
    ones = torch.ones(g.M, dtype=torch.float32, device="cuda")
    gg = nl.Graph(g.offsets, g.indices, ones)
    gg.reset()
    C0 = gg.labels()
    dn = gg.sweep(True)
    C1 = gg.labels()
    assert dn == int((C1 != C0).sum())
    assert bool((C1 <= C0).all())
    rng = np.random.default_rng(2)
    for i in rng.choice(g.N, 3000, replace=False):
        if int(C1[i]) == int(C0[i]):
            continue
        nb = g.indices[g.offsets[i]:g.offsets[i + 1]].to(torch.int64)
        assert bool(((C0[nb] == C1[i]) | (C1[nb] == C1[i])).any())
    gg.close()


def test_permuted_web_quality():
    """The first-sweep schedule on a web graph without ID locality: a 4M-vertex
    synth.web graph with its vertex IDs randomly permuted (hosts are no
    longer contiguous ID ranges, so the measured-locality gate gives the
    full-grid first sweep).  Every one of 4 asynchronous GPU runs reaches
    modularity (Eq. 1) >= the asynchronous oracle's on the same graph - 0.02
    (measured: GPU 0.862-0.875, oracle 0.871, `scripts/exp_permuted_web.py`)."""
    n = 4_000_000
    g = synth.web(n=n, seed=0, device="cuda")
    perm = torch.randperm(n, generator=torch.Generator(device="cuda").manual_seed(100), device="cuda")
    src = torch.repeat_interleave(torch.arange(n, device="cuda"), g.offsets[1:] - g.offsets[:-1])
    gp = synth.from_edges(perm[src], perm[g.indices.to(torch.int64)], n, name="web-permuted")
    del g, src
    ones = torch.ones(gp.M, dtype=torch.float32, device="cuda")
    gg = nl.Graph(gp.offsets, gp.indices, ones)
    qs = []
    for _ in range(4):
        st = gg.run()
        assert st["converged"] or st["iterations"] == 20
        qs.append(gg.modularity())
    gg.close()
    h = host_csr(gp)
    C, _, _ = oracle.lpa(h)
    q_o = oracle.modularity(h, C)
    assert min(qs) >= q_o - 0.02, (qs, q_o)

