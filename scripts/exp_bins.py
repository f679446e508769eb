"""Sweep the degree-bin switch points on a workload; print per-bin kernel ms."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_ipps_sahunk25_b200 as nl
ap = argparse.ArgumentParser()
ap.add_argument("--config", default="web_40m_2200m")
ap.add_argument("--weights", default="ones")
ap.add_argument("--grid", default="16,256,4096;8,256,4096;24,256,4096;33,256,4096;16,128,4096;16,256,1024;16,256,2048")
a = ap.parse_args()
g = synth.make(a.config, device="cuda")
w = torch.ones(g.M, dtype=torch.float32, device="cuda") if a.weights == "ones" else None
gg = nl.Graph(g.offsets, g.indices, w)
print(a.config, g.N, g.M, flush=True)
for spec in a.grid.split(";"):
    s, b, gi = map(int, spec.split(","))
    kw = dict(switch_degree=s, block_degree=b, giant_degree=gi, timing=1)
    gg.run(**kw)
    res = []
    for _ in range(3):
        st = gg.run(**kw)
        res.append(st)
    ms = sorted(r["run_ms"] for r in res)[1]
    k = [round(sum(r["kernel_ms"][i] for r in res) / 3, 2) for i in range(4)]
    print(f"switch={s:3d} block={b:4d} giant={gi:5d}  run_ms={ms:7.2f}  bins_ms={k}  it={res[-1]['iterations']} "
          f"bin_v={res[-1]['bin_vertices']}", flush=True)
