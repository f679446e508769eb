import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "tests"))
import numpy as np, torch, oracle, synth
import paper_conf_ipps_sahunk25_b200 as nl
from test_gpu_parity import GRAPHS, to_gpu, host
for name in ["sbm", "web", "rmat", "road", "kmer", "hub"]:
    for w in (False, True):
        g = GRAPHS[name](w); h = host(g)
        Co, _, _ = oracle.lpa(h); qo = oracle.modularity(h, Co)
        gg = to_gpu(g)
        qs = []
        for order in (1, 0):
            q = []
            for rep in range(5):
                gg.run(bin_order=order); q.append(round(gg.modularity(), 3))
            qs.append(q)
        print(f"{name:6s} w={int(w)} oracle {qo:.3f}  order1 {qs[0]}  order0 {qs[1]}", flush=True)
