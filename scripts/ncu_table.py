"""Print an ncu --csv --metrics capture as one row per launch."""
import csv, sys
rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
hdr = rows[0]
ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
idi = hdr.index("ID")
by = {}
for r in rows[1:]:
    by.setdefault((r[idi], r[ki][:40]), {})[r[mi]] = r[vi]
for (i, k), m in by.items():
    print(i, k)
    for n, v in sorted(m.items()):
        print(f"   {n:75s} {v}")
