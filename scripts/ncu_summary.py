"""Summarise ncu captures for profiles/: per-kernel launch table (from a
--metrics gpu__time_duration.sum CSV log) and key counters of a --set full
report (ncu -i ... --page raw --csv)."""
import csv, io, json, subprocess, sys, collections

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__inst_executed.sum",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__sass_inst_executed_op_global_ld.sum",
        "smsp__sass_inst_executed_op_shared.sum", "smsp__inst_executed_op_shared_atom.sum"]


def launches(csv_path):
    rows = [r for r in csv.reader(open(csv_path)) if r]
    hdr_i = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    hdr = rows[hdr_i]
    ik, iv, im = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Name")
    agg = collections.defaultdict(lambda: [0, 0.0])
    order = []
    for r in rows[hdr_i + 1:]:
        if len(r) <= iv or r[im] != "gpu__time_duration.sum":
            continue
        name = r[ik].split("(")[0].replace("void ", "").replace("<unnamed>::", "")
        v = float(r[iv].replace(",", ""))
        agg[name][0] += 1
        agg[name][1] += v
        order.append((name, v))
    return agg, order


def full(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")].split("(")[0]}
        for k in KEYS:
            if k in hdr:
                d[k] = f"{r[hdr.index(k)]} {units[hdr.index(k)]}".strip()
        res.append(d)
    return res


if __name__ == "__main__":
    mode, path = sys.argv[1], sys.argv[2]
    if mode == "launches":
        agg, order = launches(path)
        tot = sum(v[1] for v in agg.values())
        print("| kernel | launches | total time (ns) | share |\n|---|---|---|---|")
        for k, (n, t) in sorted(agg.items(), key=lambda x: -x[1][1]):
            print(f"| {k} | {n} | {t:.0f} | {t / tot * 100:.1f}% |")
    else:
        for d in full(path):
            print(json.dumps(d))
