"""Merge DRAM traffic per sweep of one degree bin into profiles/traffic.json.

Input: an ncu launch list with dram__bytes_read/write of one nu-LPA run
(`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
--clock-control none --csv --log-file X python scripts/profile_run.py --config C --runs 1`).

    python scripts/make_traffic.py X <config> <weights> warp|thread

warp bin of a sweep = the k_frontier launch right before each k_warp<..., 512,
...> launch; thread bin = each k_thread launch.  The bench reads
traffic.json["<config>/<weights>/<bin>"]["dram_bytes_per_sweep"] as the
roofline's `traffic` (same per-sweep unit as algorithmic_bytes_per_sweep).
"""
import collections
import csv
import json
import os
import sys

path, config, weights, binname = sys.argv[1:5]
rows = [r for r in csv.reader(open(path)) if r]
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hi]
ik, im, iv, iid = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per = collections.defaultdict(dict)
name = {}
for r in rows[hi + 1:]:
    if len(r) <= iv:
        continue
    per[r[iid]][r[im]] = float(r[iv].replace(",", ""))
    name[r[iid]] = r[ik]


def dram(k):
    return per[k]["dram__bytes_read.sum"] + per[k]["dram__bytes_write.sum"]


ids = sorted(per, key=int)
if binname == "warp":
    # per sweep: the warp-bin k_frontier, k_warp_easy (two-pass sweeps) and k_warp
    main = [k for k in ids if "k_warp<" in name[k] and ", 512" in name[k]]
    front, easy = [], []
    for k in main:
        j = ids.index(k) - 1
        e = None
        if "k_warp_easy" in name[ids[j]]:
            e = ids[j]
            j -= 1
        assert "k_frontier" in name[ids[j]], name[ids[j]]
        front.append(ids[j])
        easy.append(e)
    b = [dram(f) + dram(w) + (dram(e) if e else 0.0) for f, w, e in zip(front, main, easy)]
    kernels = ["k_frontier", "k_warp_easy", "k_warp"] if any(easy) else ["k_frontier", "k_warp"]
    extra = {"k_warp_per_launch": [dram(w) for w in main], "k_frontier_per_launch": [dram(f) for f in front],
             "k_warp_easy_per_launch": [dram(e) if e else 0.0 for e in easy]}
elif binname == "block":
    # per sweep: the block-bin k_frontier (the one right before a k_block launch) and the k_block
    # launches that follow it (4-warp TMA k_block below wide_degree, 8-warp above)
    front = [k for i, k in enumerate(ids[:-1]) if "k_frontier" in name[k] and "k_block" in name[ids[i + 1]]]
    blks = []
    for f in front:
        j = ids.index(f) + 1
        bl = []
        while j < len(ids) and "k_block" in name[ids[j]]:
            bl.append(ids[j])
            j += 1
        blks.append(bl)
    b = [dram(f) + sum(dram(c) for c in bl) for f, bl in zip(front, blks)]
    kernels = ["k_frontier", "k_block"]
    extra = {"k_block_per_sweep": [sum(dram(c) for c in bl) for bl in blks]}
else:
    # thread bin: every k_thread launch of a sweep (synchronous mode, thin bins), or the
    # compacted path's k_tscan + k_tact pairs (asynchronous bulk bins; one wave per sweep
    # at full size)
    main = [k for k in ids if "k_thread" in name[k]]
    if main:
        b = [dram(k) for k in main]
        kernels = ["k_thread"]
        extra = {}
    else:
        scan = [k for k in ids if "k_tscan" in name[k]]
        act = [ids[ids.index(k) + 1] for k in scan]
        assert all("k_tact" in name[k] for k in act), [name[k] for k in act]
        b = [dram(x) + dram(y) for x, y in zip(scan, act)]
        kernels = ["k_tscan", "k_tact"]
        extra = {"k_tscan_per_launch": [dram(x) for x in scan], "k_tact_per_launch": [dram(y) for y in act]}
out_path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "traffic.json")
db = json.load(open(out_path)) if os.path.exists(out_path) else {}
if "workload" in db:          # round-1 single-entry format
    db = {}
db[f"{config}/{weights}/{binname}"] = {
    "kernels": kernels, "sweeps": len(b), "dram_bytes_per_sweep": sum(b) / len(b), "per_sweep": b, **extra,
    "source": os.path.basename(path),
    "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none (cold, serialised launches)"}
json.dump(db, open(out_path, "w"), indent=1)
print(config, binname, sum(b) / len(b) / 1e9, "GB per sweep over", len(b), "sweeps")
