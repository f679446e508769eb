"""profiles/traffic.json from an ncu launch list with dram__bytes_read/write
(`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
-k regex:^k_ --csv --log-file X python bench.py ...`): DRAM bytes per sweep of
the warp bin (one k_frontier + one k_warp launch per sweep)."""
import csv, collections, json, sys
path, workload, weights = sys.argv[1], sys.argv[2], sys.argv[3]
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
# the warp bin of a sweep = the k_frontier launch right before each k_warp<..., 512> launch
warp = [k for k in ids if "k_warp" in name[k] and "512>" in name[k]]
front = [ids[ids.index(k) - 1] for k in warp]
assert all("k_frontier" in name[f] for f in front)
b = [dram(f) + dram(w) for f, w in zip(front, warp)]
out = {"workload": workload, "weights": weights, "bin": "warp", "kernels": ["k_frontier", "k_warp"],
       "sweeps": len(b), "dram_bytes_per_sweep": sum(b) / len(b), "per_sweep": b,
       "k_warp_per_launch": [dram(w) for w in warp], "k_frontier_per_launch": [dram(f) for f in front],
       "source": path, "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none (cold, serialised launches)"}
json.dump(out, open("profiles/traffic.json", "w"), indent=1)
print(out["dram_bytes_per_sweep"] / 1e9, "GB per sweep over", len(b), "sweeps")
