import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import time, torch, synth, paper_conf_ipps_sahunk25_b200 as nl
g = synth.make("web_40m_2200m", device="cuda")
w = torch.ones(g.M, dtype=torch.float32, device="cuda")
off_h = g.offsets.cpu().pin_memory(); idx_h = g.indices.cpu().pin_memory(); w_h = w.cpu().pin_memory()
lab_h = torch.empty(g.N, dtype=torch.int32).pin_memory()
d_idx = torch.empty_like(idx_h, device="cuda"); d_w = torch.empty_like(w_h, device="cuda")
for rep in range(2):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    d_idx.copy_(idx_h, non_blocking=True); d_w.copy_(w_h, non_blocking=True); torch.cuda.synchronize()
    t1 = time.perf_counter()
    print("raw H2D %.1f GB in %.1f ms = %.1f GB/s" % ((idx_h.numel()*8)/1e9, (t1-t0)*1e3, idx_h.numel()*8/(t1-t0)/1e9))
del d_idx, d_w; torch.cuda.empty_cache()
for rep in range(3):
    torch.cuda.synchronize(); t0 = time.perf_counter()
    h = nl.nulpa_create(off_h, idx_h, w_h); torch.cuda.synchronize(); t1 = time.perf_counter()
    nl.nulpa_run(h, nl.nulpa_default_params()); torch.cuda.synchronize(); t2 = time.perf_counter()
    nl.nulpa_labels(h, lab_h); torch.cuda.synchronize(); t3 = time.perf_counter()
    nl.nulpa_destroy(h); t4 = time.perf_counter()
    print("create %.1f ms run %.1f ms labels %.1f ms destroy %.1f ms" % ((t1-t0)*1e3, (t2-t1)*1e3, (t3-t2)*1e3, (t4-t3)*1e3))
