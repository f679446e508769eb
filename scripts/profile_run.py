"""Run nu-LPA on a synthetic workload a few times (for ncu / nsight capture)."""
import argparse, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import synth
import paper_conf_ipps_sahunk25_b200 as nl
ap = argparse.ArgumentParser()
ap.add_argument("--config", default="web_40m_2200m")
ap.add_argument("--n", type=int, default=0)
ap.add_argument("--runs", type=int, default=2)
ap.add_argument("--weights", default="ones")
ap.add_argument("--iters", type=int, default=0, help="force exactly this many sweeps (tolerance 0)")
a = ap.parse_args()
kw = {"n": a.n} if a.n else {}
g = synth.make(a.config, device="cuda", **kw)
w = torch.ones(g.M, dtype=torch.float32, device="cuda") if a.weights == "ones" else None
gg = nl.Graph(g.offsets, g.indices, w)
for i in range(a.runs):
    kw = dict(max_iterations=a.iters, tolerance=0.0) if a.iters else {}
    st = gg.run(timing=1, **kw)
    torch.cuda.synchronize()
    print(i, st["iterations"], st["changed"], [round(x, 2) for x in st["kernel_ms"]], round(st["run_ms"], 2), flush=True)
print("Q", gg.modularity())
