"""Run time of nu-LPA with the device-side loop (timing=0: one CUDA graph with a
conditional while node, one host sync per run) vs the host loop with per-bin
CUDA events (timing=1), per workload (CUDA events around 10 runs each)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_ipps_sahunk25_b200 as nl
for cfg in sys.argv[1:] or ["sbm_1m_20m", "rmat_4m_70m", "road_50m_110m", "web_40m_2200m"]:
    g = synth.make(cfg, device="cuda")
    w = torch.ones(g.M, dtype=torch.float32, device="cuda")
    gg = nl.Graph(g.offsets, g.indices, w)
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    res = {}
    for timing in (0, 1, 0, 1):
        for _ in range(3):
            gg.run(timing=timing)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(10):
            st = gg.run(timing=timing)
        e1.record()
        torch.cuda.synchronize()
        res.setdefault(timing, []).append(round(e0.elapsed_time(e1) / 10, 3))
    print(cfg, "ms per run: device loop", res[0], "host loop + events", res[1], "iterations", st["iterations"], flush=True)
    gg.close()
    del g, w
