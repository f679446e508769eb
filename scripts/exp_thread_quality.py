"""Modularity of GPU async runs vs the async oracle on small k-mer / road /
SBM graphs over several seeds (thread-bin schedule experiments)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import oracle, synth
import paper_conf_ipps_sahunk25_b200 as nl
for name, fn in [("kmer", lambda s, w: synth.kmer(n=20000, seed=s, weighted=w)),
                 ("road", lambda s, w: synth.road(R=40, mean_chain=4, seed=s, weighted=w))]:
    for w in (False, True):
        d = []
        for seed in range(6, 16):
            g = fn(seed, w)
            h = oracle.CSR.from_graph(g)
            C, _, _ = oracle.lpa(h)
            qo = oracle.modularity(h, C)
            gg = nl.Graph(g.offsets.cuda(), g.indices.cuda(), None if g.weights is None else g.weights.cuda())
            st = gg.run()
            qg = oracle.modularity(h, gg.labels(device=False).numpy())
            d.append(qg - qo)
            gg.close()
        print(name, "weighted" if w else "unit", "min dQ %.4f mean %.4f" % (min(d), float(np.mean(d))), flush=True)
