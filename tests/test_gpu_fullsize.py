"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (default parameters), on outputs the oracle can compute one by one:
a synchronous sweep's label for sampled vertices (oracle.vertex_best on the
vertex's own row), plus properties that hold at any size for the
asynchronous production run.  SBM 1M/20M is small enough for full oracle
runs."""
import os

import numpy as np
import pytest
import torch

import oracle
import synth
import paper_conf_ipps_sahunk25_b200 as nl

pytestmark = [pytest.mark.gpu, pytest.mark.slow]


def row_csr(g, i, labels):
    """The oracle's view of vertex i alone: a one-row CSR whose column 0 is i
    itself, so Algorithm 1's "if j = i continue" still applies."""
    o0, o1 = int(g.offsets[i]), int(g.offsets[i + 1])
    nb = g.indices[o0:o1].to(torch.int64)
    w = None if g.weights is None else g.weights[o0:o1].cpu().numpy()
    lab_nb = labels[nb].cpu().numpy().astype(np.int32)
    nbh = nb.cpu().numpy()
    local_idx = np.where(nbh == i, 0, np.arange(1, nbh.size + 1)).astype(np.int32)
    loc_labels = np.concatenate([[int(labels[i])], lab_nb]).astype(np.int32)
    offs = np.zeros(nbh.size + 2, dtype=np.int64)
    offs[1:] = nbh.size
    return oracle.CSR(offs, local_idx, w), loc_labels


def sample_vertices(g, n, seed):
    """Uniform sample plus the highest-degree vertices (giant / block bins)."""
    rng = np.random.default_rng(seed)
    s = rng.choice(g.N, size=n, replace=False)
    top = torch.topk(g.degrees(), 64).indices.cpu().numpy()
    return np.unique(np.concatenate([s, top]))


def check_sync_sweep_sampled(g, weights, labels0, n_sample=3000, pickless=False):
    gg = nl.Graph(g.offsets, g.indices, weights)
    flags0 = torch.ones(g.N, dtype=torch.uint8, device="cuda")
    gg.set_labels(labels0, flags0)
    gg.sweep(pickless, mode=nl.SYNC)
    C1 = gg.labels()
    gw = synth.Graph(g.offsets, g.indices, weights)
    bad = 0
    for i in sample_vertices(g, n_sample, 1):
        h, loc = row_csr(gw, int(i), labels0)
        c, w1, w2 = oracle.vertex_best(h, 0, loc)
        ci = int(labels0[i])
        expect = c if (c != oracle.EMPTY and c != ci and (not pickless or c <= ci)) else ci
        got = int(C1[i])
        if got != expect:
            bad += 1
            assert weights is not None and weights.min() != weights.max(), f"vertex {i}: {got} != {expect}"
    gg.close()
    return bad


def test_web_2200m_sync_sweep_sampled():
    g = synth.make("web_40m_2200m", device="cuda")
    assert 2.0e9 < g.M < 2.4e9
    ones = torch.ones(g.M, dtype=torch.float32, device="cuda")
    # a mid-run-like state: labels constant over blocks of 32 vertex IDs
    labels0 = (torch.arange(g.N, device="cuda", dtype=torch.int32) // 32) * 32
    assert check_sync_sweep_sampled(g, ones, labels0) == 0
    # the first sweep from the initial state (all labels distinct), Pick-Less on
    labels0 = torch.arange(g.N, device="cuda", dtype=torch.int32)
    assert check_sync_sweep_sampled(g, ones, labels0, pickless=True) == 0


def test_web_2200m_async_run_properties():
    g = synth.make("web_40m_2200m", device="cuda")
    ones = torch.ones(g.M, dtype=torch.float32, device="cuda")
    gg = nl.Graph(g.offsets, g.indices, ones)
    st = gg.run()
    assert st["converged"] and st["iterations"] <= 20
    assert st["changed"][-1] / g.N < 0.05
    C = gg.labels()
    # every final label is a vertex ID
    assert int(C.min()) >= 0 and int(C.max()) < g.N
    q = gg.modularity()
    assert 0.2 < q <= 1.0
    # first (Pick-Less) sweep never increases a label, and every changed
    # vertex took a label held by a neighbour before or after the sweep
    gg.reset()
    C0 = gg.labels()
    gg.sweep(True)
    C1 = gg.labels()
    assert bool((C1 <= C0).all())
    for i in sample_vertices(g, 2000, 2):
        if int(C1[i]) == int(C0[i]):
            continue
        nb = g.indices[g.offsets[i]:g.offsets[i + 1]].to(torch.int64)
        assert bool(((C0[nb] == C1[i]) | (C1[nb] == C1[i])).any())
    gg.close()


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


@pytest.mark.parametrize("config", ["rmat_4m_70m", "road_50m_110m"])
def test_social_and_road_sync_sweep_sampled(config):
    g = synth.make(config, device="cuda")
    labels0 = (torch.arange(g.N, device="cuda", dtype=torch.int32) // 8) * 8
    assert check_sync_sweep_sampled(g, None, labels0) == 0
    gg = nl.Graph(g.offsets, g.indices)
    st = gg.run()
    assert st["converged"] or st["iterations"] == 20
    gg.close()


@pytest.mark.skipif(not os.environ.get("NULPA_FULLSIZE_ORACLE"),
                    reason="opt-in (NULPA_FULLSIZE_ORACLE=1): ~4 min of single-threaded oracle on the host")
def test_web_2200m_quality_vs_full_oracle():
    """The production asynchronous run on the full 2.2B-edge bench graph next
    to the oracle's full asynchronous run on the same graph (the north star's
    "modularity within 0.02 of the CPU oracle").  Asynchronous LPA's result
    depends on the schedule, so several GPU runs
    are recorded; the test asserts the neighbour-label invariant and records
    the comparison (NULPA_FULLSIZE_OUT: JSON path)."""
    import json, time
    seed = int(os.environ.get("NULPA_FULLSIZE_SEED", "0"))
    g = synth.make("web_40m_2200m", device="cuda", seed=seed)
    gg = nl.Graph(g.offsets, g.indices, None)
    runs = []
    for r in range(int(os.environ.get("NULPA_FULLSIZE_RUNS", "6"))):
        st = gg.run()
        runs.append(dict(modularity=gg.modularity(), iterations=st["iterations"], changed=st["changed"]))
    sync_st = gg.run(mode=nl.SYNC)
    sync_q = gg.modularity()
    h = oracle.CSR(g.offsets.cpu().numpy(), g.indices.cpu().numpy(), None)
    t0 = time.time()
    C, it, dN = oracle.lpa(h)
    t_or = time.time() - t0
    q_or = oracle.modularity(h, C)
    q_or_gpu = gg.modularity(torch.from_numpy(C).cuda())
    assert abs(q_or - q_or_gpu) < 1e-6          # Eq. 1 on the GPU agrees with the oracle's
    out = dict(graph=f"web_40m_2200m seed {seed}, unit weights", N=g.N, M=g.M,
               gpu_async_runs=runs, gpu_sync=dict(modularity=sync_q, iterations=sync_st["iterations"]),
               oracle=dict(modularity=q_or, iterations=it, changed=[int(x) for x in dN], seconds=round(t_or, 1)))
    print(json.dumps(out))
    path = os.environ.get("NULPA_FULLSIZE_OUT")
    if path:
        with open(path, "w") as f:
            json.dump(out, f, indent=1)
    gg.close()
