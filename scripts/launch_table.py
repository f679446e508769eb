"""Summarise an ncu launch list (--metrics gpu__time_duration.sum[,dram__bytes_*] --csv):
per kernel name: launches, total ms, share, DRAM GB.  Only this repo's kernels
(k_*) unless --all."""
import collections, csv, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if r]
hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
h = rows[hi]
ik, im, iv, iid = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID")
per = collections.defaultdict(dict)
name = {}
for r in rows[hi + 1:]:
    if len(r) > iv:
        per[r[iid]][r[im]] = float(r[iv].replace(",", ""))
        name[r[iid]] = r[ik].split("(")[0].replace("void ", "").replace("<unnamed>::", "")
agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
ours = "--all" not in sys.argv
for k, m in per.items():
    if ours and not name[k].startswith("k_"):
        continue                                   # torch kernels of the graph generator
    a = agg[name[k]]
    a[0] += 1
    a[1] += m.get("gpu__time_duration.sum", 0) / 1e6
    a[2] += (m.get("dram__bytes_read.sum", 0) + m.get("dram__bytes_write.sum", 0)) / 1e9
tot = sum(a[1] for a in agg.values())
print(f"{'kernel':60s} {'n':>4s} {'ms':>9s} {'share':>6s} {'DRAM GB':>8s}")
for k, a in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k[:60]:60s} {a[0]:4d} {a[1]:9.3f} {a[1] / tot * 100:5.1f}% {a[2]:8.2f}")
print(f"{'total':60s} {'':4s} {tot:9.3f}")
