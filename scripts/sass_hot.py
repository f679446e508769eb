"""Per-SASS-instruction view of an ncu source page export (--page source --csv
--print-source sass): executions per unit (e.g. per vertex) and stall samples.
usage: python scripts/sass_hot.py <export.csv> <units> [min_per_unit]"""
import csv, sys
rows = list(csv.reader(open(sys.argv[1])))
units = float(sys.argv[2]); thr = float(sys.argv[3]) if len(sys.argv) > 3 else 0.02
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
ia, isrc, iss, iex = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
ith = h.index("Avg. Predicated-On Threads Executed")
data = [(int(r[ia], 16), r[isrc].strip(), int(r[iss] or 0), int(r[iex] or 0), r[ith]) for r in rows[hi + 1:] if len(r) > iex and r[ia].startswith("0x")]
base = data[0][0]
tot_e = sum(d[3] for d in data); tot_s = sum(d[2] for d in data)
print(f"total inst {tot_e:.4e} = {tot_e/units:.1f} per unit; stall samples {tot_s}")
skipped = 0
for a, src, s, e, th in data:
    if e / units < thr and s / tot_s < 0.002:
        skipped += 1
        continue
    if skipped:
        print(f"   ... {skipped} cold")
        skipped = 0
    print(f"{a-base:6x} {e/units:7.3f} {s/tot_s*100:5.2f}% {th:>5} {src[:90]}")
