"""Markdown table (one row per launch) of an ncu capture with
gpu__time_duration, thread-instructions per warp-instruction (warp execution
efficiency = ratio / 32), issue active, warps active, instructions.
usage: python scripts/wexec_md.py <capture.csv> [...]"""
import csv, sys, collections
for path in sys.argv[1:]:
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    rows = rows[next(i for i, r in enumerate(rows) if "Kernel Name" in r):]
    h = rows[0]
    ik, im, iv, iid, iu = h.index("Kernel Name"), h.index("Metric Name"), h.index("Metric Value"), h.index("ID"), h.index("Metric Unit")
    per, name = collections.defaultdict(dict), {}
    for r in rows[1:]:
        per[int(r[iid])][r[im]] = (float(r[iv].replace(",", "")), r[iu])
        name[int(r[iid])] = r[ik].split("(")[0].replace("void ", "").replace("<unnamed>::", "")
    print(f"\n### {path.split('/')[-1]}\n")
    print("| launch | kernel | ms | warp exec. efficiency | issue % | warps active % | G warp inst |")
    print("|---|---|---|---|---|---|---|")
    for k in sorted(per):
        m = per[k]
        t, u = m["gpu__time_duration.sum"]
        ms = t / 1e6 if u in ("nsecond", "ns") else (t / 1e3 if u in ("usecond", "us") else t)
        print(f"| {k} | {name[k][:34]} | {ms:.3f} | {m['smsp__thread_inst_executed_per_inst_executed.ratio'][0] / 32 * 100:.1f}% | "
              f"{m['smsp__issue_active.avg.pct_of_peak_sustained_active'][0]:.1f} | {m['sm__warps_active.avg.pct_of_peak_sustained_active'][0]:.1f} | "
              f"{m['smsp__inst_executed.sum'][0] / 1e9:.3f} |")
