"""Experiment: modularity of GPU async/sync runs under tie rules and bin orders."""
import sys, os, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, ctypes
import oracle, synth
import paper_conf_ipps_sahunk25_b200 as nl
L = oracle._L(); L.oracle_set_tie_rule.argtypes = [ctypes.c_int]
gs = {'web30k': synth.web(n=30000, avg_out=20, host_min=4, host_max=3000, seed=3),
      'web300k': synth.web(n=300000, seed=3),
      'web2m': synth.web(n=2_000_000, seed=3, device='cuda').to('cpu'), 'web30k_uniform': synth.web(n=30000, avg_out=20, host_min=4, host_max=3000, seed=3, p_local=0.85, locality='uniform'),
      'sbm': synth.sbm(n=100000, community_size=100, avg_degree=16, mu=0.25, seed=2),
      'road': synth.road(R=200, seed=5), 'kmer': synth.kmer(n=200000, seed=6), 'rmat': synth.rmat(scale=16, seed=4)}
for name, g in gs.items():
    h = oracle.CSR.from_graph(g)
    gg = nl.Graph(g.offsets.cuda(), g.indices.cuda())
    for rule in (0, 1):
        L.oracle_set_tie_rule(rule)
        res = []
        if g.N <= 300000:
            for sync in (False, True):
                C, it, _ = oracle.lpa(h, sync=sync)
                res.append(f"oracle-{'sync' if sync else 'async'} {oracle.modularity(h, C):.3f}/{it}")
        for mode in (nl.ASYNC, nl.SYNC):
            for order in (0, 1):
                st = gg.run(mode=mode, tie_rule=rule, bin_order=order)
                q = gg.modularity()
                res.append(f"gpu-{'sync' if mode else 'async'}-o{order} {q:.3f}/{st['iterations']}")
        print(f"{name:8s} rule{rule}: " + "  ".join(res), flush=True)
