"""profiles/traffic.json from an ncu launch list with dram__bytes_read/write
(`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum
-k regex:^k_ --csv --log-file X python bench.py ...`)."""
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
warp = [d for k, d in per.items() if "k_warp" in name[k]]
b = [d["dram__bytes_read.sum"] + d["dram__bytes_write.sum"] for d in warp]
out = {"workload": workload, "weights": weights, "kernel": "k_warp", "launches": len(b),
       "dram_bytes_per_launch": sum(b) / len(b), "per_launch": b,
       "source": path, "how": "ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum --clock-control none (cold, serialised launches)"}
json.dump(out, open("profiles/traffic.json", "w"), indent=1)
print(out["dram_bytes_per_launch"] / 1e9, "GB per launch over", len(b), "launches")
