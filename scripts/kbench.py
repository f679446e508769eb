"""Deterministic kernel A/B timing: synchronous sweeps from fixed states, so
the work is identical across builds.  State A: the initial labels (all
distinct, all active -- like sweep 0).  State B: labels of a converged async
run, all active (like the confirming sweeps)."""
import argparse, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_ipps_sahunk25_b200 as nl
ap = argparse.ArgumentParser()
ap.add_argument("--config", default="web_40m_2200m")
ap.add_argument("--weights", default="ones")
ap.add_argument("--reps", type=int, default=5)
ap.add_argument("--async-too", action="store_true")
ap.add_argument("--capture", default="", help="A or B: one synchronous sweep inside cudaProfilerStart/Stop (ncu --profile-from-start off)")
ap.add_argument("--param", action="append", default=[], metavar="KEY=INT", help="nulpa_params override for the timed sweeps")
a = ap.parse_args()
P = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in a.param}
g = synth.make(a.config, device="cuda")
w = torch.ones(g.M, dtype=torch.float32, device="cuda") if a.weights == "ones" else None
gg = nl.Graph(g.offsets, g.indices, w)
torch.manual_seed(0)
gg.run()
Lconv = gg.labels().clone()
ones = torch.ones(g.N, dtype=torch.uint8, device="cuda")
Linit = torch.arange(g.N, dtype=torch.int32, device="cuda")
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
if a.capture:
    L = Linit if a.capture == "A" else Lconv
    gg.set_labels(L, ones)
    torch.cuda.synchronize()
    torch.cuda.profiler.start()
    gg.sweep(a.capture == "A", mode=nl.SYNC, **P)
    torch.cuda.synchronize()
    torch.cuda.profiler.stop()
    sys.exit(0)
modes = [("sync", nl.SYNC)] + ([("async", nl.ASYNC)] if a.async_too else [])
for name, L in (("A:init", Linit), ("B:converged", Lconv)):
    for mname, mode in modes:
        ts = []
        for r in range(a.reps):
            gg.set_labels(L, ones)
            torch.cuda.synchronize()
            e0.record()
            gg.sweep(name.startswith("A"), mode=mode, **P)
            e1.record()
            torch.cuda.synchronize()
            ts.append(e0.elapsed_time(e1))
        st = gg.stats()
        print(f"{name:12s} {mname:5s} min {min(ts):7.3f} ms  median {sorted(ts)[len(ts)//2]:7.3f} ms", flush=True)
