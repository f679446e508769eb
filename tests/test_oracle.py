"""Pins for the oracle (oracle/oracle.c) against what the paper and the
mathematics fix -- never against the oracle itself or the CUDA path.

Each test names the passage of PAPER.md it checks.  Independent checks used:
closed forms, hand-derived and published karate-club modularity values,
brute-force (dense / candidate-enumeration) reimplementations on tiny graphs,
and invariants of the method (labels come from neighbours, Pick-Less never
increases a label, disjoint cliques collapse to one label each).
"""
import json
import math
import os

import numpy as np
import pytest

import oracle
import synth

GOLDEN = os.path.join(os.path.dirname(__file__), "golden")


def np_graph(g):
    return oracle.CSR.from_graph(g)


def adjacency(g):
    """CSR -> python lists of (j, w) in CSR order (unit weight when None)."""
    off, idx = g.offsets, g.indices
    w = g.weights
    return [[(int(idx[e]), float(w[e]) if w is not None else 1.0) for e in range(off[i], off[i + 1])]
            for i in range(g.N)]


def naive_best(i, adj_i, C, tie_rule=0):
    """Brute force Eq. 3: enumerate candidate labels in
    tie order (R6: increasing label; tie rule 1: increasing home slot
    c mod p1 with p1 = nextPow2(D)-1, then label), sum float32 weights in CSR
    order, keep the strictly larger."""
    cands = sorted({C[j] for j, _ in adj_i if j != i})
    if tie_rule == 1:
        D = len(adj_i)
        p1 = 1
        while p1 <= D:
            p1 *= 2
        p1 -= 1
        cands = sorted(cands, key=lambda c: ((c % p1), c))
    best, bw, all_w = None, None, []
    for c in cands:
        s = np.float32(0.0)
        for j, w in adj_i:
            if j != i and C[j] == c:
                s = np.float32(s + np.float32(w))
        all_w.append(s)
        if best is None or s > bw:
            best, bw = c, s
    second = max([x for c, x in zip(cands, all_w) if c != best], default=np.float32(-1.0))
    return best, (np.float32(-1.0) if bw is None else bw), second


def naive_lpa(g, tau, max_iter, rho, sync):
    """Algorithm 1 written out naively on python lists."""
    adj = adjacency(g)
    N = g.N
    C = list(range(N))
    U = [1] * N
    dns = []
    it = 0
    for l in range(max_iter):
        pl = rho > 0 and l % rho == 0
        dn = 0
        if sync:
            Cold = list(C)
            Unew = [0] * N
            for i in range(N):
                if not U[i]:
                    continue
                c, _, _ = naive_best(i, adj[i], Cold)
                if c is not None and c != Cold[i] and (not pl or c <= Cold[i]):
                    C[i] = c
                    dn += 1
                    for j, _ in adj[i]:
                        Unew[j] = 1
            U = Unew
        else:
            for i in range(N):
                if not U[i]:
                    continue
                U[i] = 0
                c, _, _ = naive_best(i, adj[i], C)
                if c is not None and c != C[i] and (not pl or c <= C[i]):
                    C[i] = c
                    dn += 1
                    for j, _ in adj[i]:
                        U[j] = 1
        dns.append(dn)
        it = l + 1
        if not pl and dn / N < tau:
            break
    return np.array(C, dtype=np.int32), it, dns


# ---------------------------------------------------------------------------
# hashtable (Algorithm 2)
# ---------------------------------------------------------------------------

def test_capacity_and_secondary_prime():
    # capacity nextPow2(D)-1 must hold every neighbour label (>= D)
    # inside the 2*D slots reserved per vertex; p2 > p1, co-prime.
    for D in range(1, 5000):
        p1, p2 = oracle.hashtable_primes(D)
        assert D <= p1 < 2 * D
        assert p1 + 1 & p1 == 0            # Mersenne number 2^a - 1 (mod-friendly)
        assert p2 > p1 and math.gcd(p1, p2) == 1


@pytest.mark.parametrize("D", [1, 2, 3, 7, 8, 31, 100, 1000, 4095])
def test_hashtable_matches_dictionary(D):
    rng = np.random.default_rng(D)
    ht = oracle.Hashtable(D)
    # D insertions drawn from at most D distinct keys spread over a large range
    keys_pool = rng.choice(1 << 30, size=D, replace=False)
    stream_k = rng.choice(keys_pool, size=D)
    stream_v = rng.random(D).astype(np.float32)
    ref = {}
    for k, v in zip(stream_k, stream_v):
        probes, slot = ht.accumulate(int(k), float(v))
        assert probes >= 1 and 0 <= slot < ht.p1
        ref[int(k)] = np.float32(ref.get(int(k), np.float32(0)) + v)
    got = {int(k): v for k, v in zip(ht.Hk, ht.Hv) if k != oracle.EMPTY}
    assert got.keys() == ref.keys()
    for k in ref:
        assert got[k] == ref[k]            # same float32 summation order -> exact
    # hashtableMaxKey: max weight, smallest label on ties
    best = min(ref, key=lambda k: (-ref[k], k))
    k, w1, w2 = ht.max_key()
    assert k == best and np.float32(w1) == ref[best]
    others = [v for kk, v in ref.items() if kk != best]
    assert np.float32(w2) == (max(others) if others else np.float32(-1))


def test_hashtable_completely_full():
    # p1 distinct keys in a table of p1 slots: the R5 linear continuation must place all.
    for D in [7, 15, 63, 255]:
        ht = oracle.Hashtable(D)
        assert ht.p1 >= D
        keys = np.arange(ht.p1) * 7919 + 3
        for k in keys:
            assert ht.accumulate(int(k), 1.0)[0] >= 1
        for k in keys:                     # second pass hits existing keys
            assert ht.accumulate(int(k), 1.0)[0] >= 1
        assert sorted(ht.Hk.tolist()) == sorted(keys.tolist())
        assert np.all(ht.Hv == 2.0)


def test_hashtable_tie_takes_smallest_label():
    ht = oracle.Hashtable(4)
    for k in [9, 5, 7, 5, 9]:
        ht.accumulate(k, 1.0)
    assert ht.max_key()[0] == 5            # 5 and 9 both weigh 2.0


# ---------------------------------------------------------------------------
# one vertex / one sweep against brute force
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("tie_rule", [0, 1])
@pytest.mark.parametrize("weighted", [False, True])
@pytest.mark.parametrize("seed", [0, 1, 2])
def test_vertex_best_bruteforce(weighted, seed, tie_rule):
    g = np_graph(synth.erdos_renyi(60, 400, seed=seed, weighted=weighted))
    rng = np.random.default_rng(seed)
    C = rng.integers(0, 40, g.N).astype(np.int32)   # few labels -> many collisions/ties
    adj = adjacency(g)
    for i in range(g.N):
        c, w1, w2 = oracle.vertex_best(g, i, C, tie_rule=tie_rule)
        nc, nw1, nw2 = naive_best(i, adj[i], C, tie_rule)
        if nc is None:
            assert c == oracle.EMPTY
            continue
        assert c == nc and np.float32(w1) == nw1 and np.float32(w2) == nw2


def test_self_loops_are_skipped():
    # PAPER.md:338 "if j = i continue": a heavy self-loop must not pull the label.
    import torch
    src = torch.tensor([0, 0, 1])
    dst = torch.tensor([0, 1, 2])
    g = synth.from_edges(src, dst, 3, keep_self_loops=True)
    g = np_graph(g)
    C = np.array([0, 1, 2], dtype=np.int32)
    assert oracle.vertex_best(g, 0, C)[0] == 1
    iso = np_graph(synth.from_edges(torch.tensor([0]), torch.tensor([0]), 2, keep_self_loops=True))
    assert oracle.vertex_best(iso, 0, np.array([0, 1], dtype=np.int32))[0] == oracle.EMPTY


@pytest.mark.parametrize("pickless", [False, True])
@pytest.mark.parametrize("weighted", [False, True])
def test_sync_sweep_bruteforce(pickless, weighted):
    g = np_graph(synth.erdos_renyi(80, 300, seed=5, weighted=weighted))
    rng = np.random.default_rng(7)
    C = rng.integers(0, 80, g.N).astype(np.int32)
    U = (rng.random(g.N) < 0.7).astype(np.uint8)
    dn, C2, U2, w1, w2 = oracle.lpa_move_sync(g, C, U, pickless)
    adj = adjacency(g)
    eC, eU, edn = C.copy(), np.zeros_like(U), 0
    for i in range(g.N):
        if not U[i]:
            assert math.isnan(w1[i])
            continue
        c, bw, sw = naive_best(i, adj[i], C)
        if c is not None:
            assert np.float32(w1[i]) == bw and np.float32(w2[i]) == sw
        if c is not None and c != C[i] and (not pickless or c <= C[i]):
            eC[i] = c
            edn += 1
            for j, _ in adj[i]:
                eU[j] = 1
    assert dn == edn
    np.testing.assert_array_equal(C2, eC)
    np.testing.assert_array_equal(U2, eU)


@pytest.mark.parametrize("sync", [False, True])
@pytest.mark.parametrize("weighted", [False, True])
@pytest.mark.parametrize("seed", [0, 1])
def test_full_lpa_bruteforce(sync, weighted, seed):
    gs = [synth.erdos_renyi(50, 120, seed=seed, weighted=weighted),
          synth.karate(),
          synth.sbm(n=300, community_size=30, avg_degree=8, mu=0.2, seed=seed, weighted=weighted)]
    for g in gs:
        g = np_graph(g)
        for rho in [4, 0, 1]:
            C, it, dn = oracle.lpa(g, tolerance=0.05, max_iterations=20, pickless_period=rho, sync=sync)
            nC, nit, ndn = naive_lpa(g, 0.05, 20, rho, sync)
            assert it == nit and list(dn) == ndn
            np.testing.assert_array_equal(C, nC)


# ---------------------------------------------------------------------------
# invariants of the method
# ---------------------------------------------------------------------------

@pytest.mark.parametrize("sync", [False, True])
def test_disjoint_cliques_one_label_each(sync):
    # Brute force: every clique's vertices end with one label, the smallest
    # vertex ID of the clique (the only label PL sweep 0 lets everyone adopt).
    sizes = [1, 2, 3, 5, 8, 13, 2, 1, 21, 4]
    g = synth.cliques(sizes, permute=True, seed=3)
    truth = g.truth.numpy()
    C, it, dn = oracle.lpa(np_graph(g), sync=sync)
    for k in range(len(sizes)):
        members = np.nonzero(truth == k)[0]
        assert np.all(C[members] == members.min())
    assert it == 2 and dn[-1] == 0


def test_pickless_resolves_swap():
    # two adjacent vertices swap labels forever under
    # synchronous updates; Pick-Less breaks the symmetry.
    g = np_graph(synth.cliques([2]))
    C, it, dn = oracle.lpa(g, tolerance=0.05, max_iterations=20, pickless_period=0, sync=True)
    assert it == 20 and np.all(dn == 2)
    C, it, dn = oracle.lpa(g, tolerance=0.05, max_iterations=20, pickless_period=4, sync=True)
    assert it == 2 and list(C) == [0, 0]


@pytest.mark.parametrize("sync", [False, True])
def test_sweep_invariants(sync):
    """Every new label is the vertex's old label or a neighbour's label (Eq. 3
    takes the argmax over neighbour labels), and a Pick-Less sweep never
    increases a label."""
    g = np_graph(synth.sbm(n=3000, community_size=100, avg_degree=12, mu=0.3, seed=1))
    C = np.arange(g.N, dtype=np.int32)
    U = np.ones(g.N, dtype=np.uint8)
    off, idx = g.offsets, g.indices
    for l in range(12):
        pl = l % 4 == 0
        old = C.copy()
        if sync:
            _, C, U, _, _ = oracle.lpa_move_sync(g, C, U, pl)
        else:
            oracle.lpa_move_async(g, C, U, pl)
        for i in np.nonzero(C != old)[0]:
            nb = idx[off[i]:off[i + 1]]
            allowed = set(old[nb].tolist()) | (set() if sync else set(C[nb].tolist()))
            assert C[i] in allowed
        if pl:
            assert np.all(C <= old)


def test_tolerance_and_iteration_semantics():
    g = np_graph(synth.sbm(n=2000, community_size=50, avg_degree=10, mu=0.3, seed=2))
    # PL on iteration 0 can never stop the loop: huge tau -> 2 iterations
    _, it, _ = oracle.lpa(g, tolerance=10.0)
    assert it == 2
    _, it, _ = oracle.lpa(g, max_iterations=1)
    assert it == 1
    _, it, dn = oracle.lpa(g, tolerance=0.0, max_iterations=50)
    assert it == 50 or dn[-1] == 0


def test_sbm_planted_partition_recovered():
    # LPA reaches high NMI relative to ground truth.
    g = synth.sbm(n=20000, community_size=200, avg_degree=20, mu=0.1, seed=4)
    C, it, _ = oracle.lpa(np_graph(g))
    assert oracle.nmi(C, g.truth.numpy()) > 0.9
    assert oracle.modularity(np_graph(g), C) > 0.8


# ---------------------------------------------------------------------------
# modularity (Equation 1)
# ---------------------------------------------------------------------------

def test_modularity_karate_golden():
    spec = json.load(open(os.path.join(GOLDEN, "karate_modularity.json")))["partitions"]
    g = np_graph(synth.karate())
    assert g.N == 34 and g.M == 156
    hi = [0, 1, 2, 3, 4, 5, 6, 7, 8, 10, 11, 12, 13, 16, 17, 19, 21]
    club = np.ones(34, dtype=np.int32)
    club[hi] = 0
    opt = np.zeros(34, dtype=np.int32)
    for k, part in enumerate(spec["optimum_4"]["labels"]):
        opt[part] = k
    cases = {"one_community": np.zeros(34, dtype=np.int32),
             "singletons": np.arange(34, dtype=np.int32),
             "club_split": club, "optimum_4": opt}
    for name, labels in cases.items():
        q = oracle.modularity(g, labels)
        tol = spec[name].get("tol", 1e-12)
        assert abs(q - spec[name]["Q"]) <= tol, (name, q)


@pytest.mark.parametrize("seed", [0, 1, 2, 3])
def test_modularity_dense_first_form(seed):
    # Eq. 1 first form over ALL vertex pairs (R11), dense numpy, float64.
    g = synth.erdos_renyi(40, 150, seed=seed, weighted=bool(seed % 2))
    g = np_graph(g)
    A = np.zeros((g.N, g.N))
    for i in range(g.N):
        for e in range(g.offsets[i], g.offsets[i + 1]):
            A[i, g.indices[e]] += g.weights[e] if g.weights is not None else 1.0
    K = A.sum(1)
    two_m = A.sum()
    rng = np.random.default_rng(seed)
    C = rng.integers(0, 6, g.N).astype(np.int32)
    delta = C[:, None] == C[None, :]
    q_dense = ((A - np.outer(K, K) / two_m) * delta).sum() / two_m
    assert abs(oracle.modularity(g, C) - q_dense) < 1e-12


def test_modularity_equal_cliques_closed_form():
    for k in [1, 2, 5, 10]:
        g = synth.cliques([6] * k, permute=True, seed=k)
        q = oracle.modularity(np_graph(g), g.truth.numpy().astype(np.int32))
        assert abs(q - (1 - 1 / k)) < 1e-12


# ---------------------------------------------------------------------------
# NMI (evaluation metric)
# ---------------------------------------------------------------------------

def test_nmi_pins():
    rng = np.random.default_rng(0)
    a = rng.integers(0, 10, 5000)
    assert abs(oracle.nmi(a, a) - 1) < 1e-12
    perm = rng.permutation(10)
    assert abs(oracle.nmi(a, perm[a] + 100) - 1) < 1e-12
    b = rng.integers(0, 10, 5000)
    assert oracle.nmi(a, b) < 0.01
    # hand example: A = [0,0,1,1], B = [0,0,0,1]: H(A)=ln2, H(B)=H(1/4,3/4),
    # I = H(B) - H(B|A) = H(B) - (1/2) ln 2
    hb = -(0.25 * math.log(0.25) + 0.75 * math.log(0.75))
    mi = hb - 0.5 * math.log(2)
    assert abs(oracle.nmi([0, 0, 1, 1], [0, 0, 0, 1]) - 2 * mi / (math.log(2) + hb)) < 1e-12
