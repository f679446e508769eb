"""The seeded input generators (synth/): shape, symmetry, simplicity,
determinism, and that the bucketed large-graph path equals the direct one."""
import numpy as np
import pytest
import torch

import synth


def check_simple_undirected(g):
    off, idx = g.offsets.numpy(), g.indices.numpy().astype(np.int64)
    N = g.N
    src = np.repeat(np.arange(N), np.diff(off))
    assert np.all((idx >= 0) & (idx < N))
    assert not np.any(src == idx), "self-loop"
    key = src * N + idx
    assert np.all(np.diff(key) > 0), "rows not sorted / duplicate edge"
    rkey = idx * N + src
    assert np.array_equal(np.sort(rkey), key), "not symmetric"
    if g.weights is not None:
        w = g.weights.numpy()
        order = np.argsort(rkey)
        assert np.array_equal(w[order], w), "w_ij != w_ji"
        assert np.all((w > 0) & (w <= 1))


@pytest.mark.parametrize("make", [
    lambda: synth.karate(),
    lambda: synth.sbm(n=5000, community_size=100, avg_degree=12, seed=1),
    lambda: synth.rmat(scale=12, edge_factor=8, seed=2),
    lambda: synth.road(R=30, mean_chain=4, seed=3),
    lambda: synth.kmer(n=5000, seed=4),
    lambda: synth.web(n=20000, avg_out=20, host_min=4, host_max=3000, seed=5),
    lambda: synth.web(n=20000, avg_out=20, seed=5, weighted=True),
    lambda: synth.cliques([3, 1, 5], permute=True),
])
def test_generators_simple_symmetric(make):
    check_simple_undirected(make())


def test_generators_deterministic():
    a = synth.web(n=10000, seed=9)
    b = synth.web(n=10000, seed=9)
    assert torch.equal(a.indices, b.indices) and torch.equal(a.offsets, b.offsets)
    c = synth.web(n=10000, seed=10)
    assert not torch.equal(a.offsets, c.offsets)


def test_bucketed_path_matches_direct():
    old = synth._CHUNK
    try:
        synth._CHUNK = 1 << 29
        g1 = synth.web(n=30000, seed=2, weighted=True)
        synth._CHUNK = 5000
        g2 = synth.web(n=30000, seed=2, weighted=True)
    finally:
        synth._CHUNK = old
    assert torch.equal(g1.offsets, g2.offsets)
    assert torch.equal(g1.indices, g2.indices)
    assert torch.equal(g1.weights, g2.weights)


def test_shapes_match_paper_families():
    road = synth.road(R=100, seed=1)
    assert 1.9 < road.M / road.N < 2.3          # europe_osm: avg degree 2.1
    km = synth.kmer(n=50000, seed=1)
    assert 1.9 < km.M / km.N < 2.3              # kmer_A2a: 2.1
    sbm = synth.sbm(n=50000, community_size=1000, avg_degree=20, seed=1)
    assert 18 < sbm.M / sbm.N < 21              # configs[1]: 1M / 20M
    web = synth.web(n=100000, seed=1)
    d = web.degrees()
    assert int(d.max()) > 50 * float(d.float().mean())   # power-law hubs
