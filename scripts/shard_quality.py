"""Quality of the multi-GPU protocol (bulk-synchronous across ranks,
asynchronous within a rank) emulated on ONE GPU: P shard handles of the
web_40m_2200m graph, each with its own replicated label / flag vectors,
sweep one after another; after every sweep the labels of each range are
copied to every replica (the all-gather) and the flags are merged with a max
and restricted to the owner's rows (the reduce-scatter).  Prints the
modularity and per-sweep changes for P = 1, 2, 4, 8 -- the same numbers an
8-GPU run would produce, up to the asynchronous schedule.  Also reports,
per sweep, what the exchange of distributed.py sends per rank: changed
labels as 8-byte pairs (padded to the largest count) or, when more than
N/8 changed, the dense 4-byte label range; marks as bitmaps (N/8 bytes)."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, synth
import paper_conf_ipps_sahunk25_b200 as nl
from paper_conf_ipps_sahunk25_b200 import distributed as D

g = synth.make(sys.argv[1] if len(sys.argv) > 1 else "web_40m_2200m", device="cuda")
out = {}
for P in [int(x) for x in os.environ.get("SHARDS", "1,2,4,8").split(",")]:
    runners = [D.CudaShardRunner(D.shard_graph(g.offsets, g.indices, None, r, P)) for r in range(P)]
    bounds = runners[0].shard.bounds
    qs = []
    for rep in range(3):
        for run in runners:
            run.reset()
            run.flags[:run.row_begin].zero_()
            run.flags[run.row_end:].zero_()
        changed = []
        ts = []
        xbytes = []
        for l in range(20):
            pl = l % 4 == 0
            d = 0
            counts = []
            for run in runners:
                prev = run.labels[run.row_begin:run.row_end].clone()
                e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
                e0.record()
                d += run.sweep(pl)
                e1.record()
                torch.cuda.synchronize()
                ts.append(e0.elapsed_time(e1))
                counts.append(int((run.labels[run.row_begin:run.row_end] != prev).sum()))
            maxrows = max(e - b for b, e in bounds)
            dense = sum(counts) > g.N / 8
            lab_b = 4 * maxrows if dense else 8 * max(counts)
            xbytes.append({"labels": "dense" if dense else "sparse", "label_bytes_per_rank": lab_b,
                           "dense_label_bytes_per_rank": 4 * maxrows,
                           "flag_bitmap_bytes_per_rank": 4 * ((maxrows + 31) // 32) * P})
            for q, (qb, qe) in enumerate(bounds):
                for run in runners:
                    if run is not runners[q]:
                        run.labels[qb:qe].copy_(runners[q].labels[qb:qe])
            F = runners[0].flags.clone()
            for run in runners[1:]:
                torch.maximum(F, run.flags, out=F)
            for run in runners:
                run.flags.copy_(F)
                run.flags[:run.row_begin].zero_()
                run.flags[run.row_end:].zero_()
            changed.append(d)
            if not pl and d / g.N < 0.05:
                break
        Sigma = torch.zeros(g.N, dtype=torch.float64, device="cuda")
        sig = m2 = 0.0
        for run in runners:
            s_, m_ = run.modularity_partial(Sigma)
            sig += s_
            m2 += m_
        qs.append(round(runners[0].modularity_finish(Sigma, sig, m2), 4))
    out[P] = {"modularity_runs": qs, "changed_last_run": changed, "exchange_last_run": xbytes,
              "max_shard_sweep_ms_last_run": [round(max(ts[i * P:(i + 1) * P]), 2) for i in range(len(ts) // P)]}
    print(P, json.dumps(out[P]), flush=True)
    for run in runners:
        run.g.close()
    del runners
    torch.cuda.empty_cache()
