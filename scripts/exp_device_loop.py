"""nulpa_run with the host loop (device_loop=0) vs the CUDA-graph device loop
(device_loop=1): same counters, run time per workload (CUDA events around
nulpa_run on the caller's stream, 10 runs after 3 warm-ups)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_ipps_sahunk25_b200 as nl
for cfg in sys.argv[1:] or ["sbm_1m_20m", "road_50m_110m", "rmat_4m_70m", "web_40m_2200m"]:
    g = synth.make(cfg, device="cuda")
    w = torch.ones(g.M, dtype=torch.float32, device="cuda")
    gg = nl.Graph(g.offsets, g.indices, w)
    out = {}
    for dl in (0, 1):
        for _ in range(3):
            gg.run(device_loop=dl, mode=nl.SYNC)
        st_sync = gg.run(device_loop=dl, mode=nl.SYNC)
        lab_sync = gg.labels().clone()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        torch.cuda.synchronize()
        e0.record()
        for _ in range(10):
            st = gg.run(device_loop=dl)
        e1.record()
        torch.cuda.synchronize()
        out[dl] = (e0.elapsed_time(e1) / 10, st["iterations"], st_sync["iterations"], st_sync["changed"], lab_sync, st["launches"])
    same = out[0][2:4] == out[1][2:4] and torch.equal(out[0][4], out[1][4])
    print(f"{cfg}: host loop {out[0][0]:.3f} ms ({out[0][1]} it), device loop {out[1][0]:.3f} ms ({out[1][1]} it); "
          f"sync runs identical: {same}; launches {out[0][5]} / {out[1][5]}", flush=True)
    gg.close()
    del g, w
    torch.cuda.empty_cache()
