"""Per-source-line view of an ncu --set full capture: joins the SASS source
page (instructions executed, stall samples per instruction) with the line
table of the cubin (nvdisasm -g), so hot spots read as nulpa.cu lines.

usage: python scripts/ncu_lines.py <report.ncu-rep> <mangled-kernel-substring> [top] [launch-index]
(BY=0 sorts by stall samples, BY=1 (default) by instructions executed)
"""
import collections, csv, io, os, re, subprocess, sys, tempfile

rep, kname = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
launch = sys.argv[4] if len(sys.argv) > 4 else "0"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
lib = os.path.join(ROOT, "paper_conf_ipps_sahunk25_b200", "libnulpa.so")

d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=d, capture_output=True, check=True)
cubin = os.path.join(d, [f for f in os.listdir(d) if f.endswith(".cubin")][0])
dis = subprocess.run(["nvdisasm", "-g", cubin], capture_output=True, text=True).stdout

# offset -> line within the function whose name contains kname
line_of, cur_fn, cur_line = {}, None, None
for ln in dis.splitlines():
    m = re.match(r"\s*\.text\.(\S+):", ln)
    if m:
        cur_fn = m.group(1)
        continue
    m = re.search(r"//## File \".*?\", line (\d+)", ln)
    if m:
        cur_line = int(m.group(1))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m and cur_fn and kname in cur_fn:
        line_of[int(m.group(1), 16)] = cur_line

out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass",
                      "--launch-skip", launch, "--launch-count", "1"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
hdr = rows[hi]
ia, isrc = hdr.index("Address"), hdr.index("Source")
iss = hdr.index("Warp Stall Sampling (All Samples)")
iex = hdr.index("Instructions Executed")
base = None
agg = collections.defaultdict(lambda: [0, 0, []])
tot_s = tot_e = 0
for r in rows[hi + 1:]:
    if len(r) <= iex or not r[ia].startswith("0x"):
        continue
    a = int(r[ia], 16)
    base = a if base is None else base
    off = a - base
    s, e = int(r[iss] or 0), int(r[iex] or 0)
    L = line_of.get(off)
    agg[L][0] += s
    agg[L][1] += e
    agg[L][2].append(r[isrc].strip().split()[0] if r[isrc].strip() else "")
    tot_s += s
    tot_e += e
src = open(os.path.join(ROOT, "paper_conf_ipps_sahunk25_b200", "csrc", "nulpa.cu")).read().splitlines()
print(f"total samples {tot_s}, instructions {tot_e:.3e}; mapped offsets {len(line_of)}")
for L, (s, e, ops) in sorted(agg.items(), key=lambda kv: -kv[1][int(os.environ.get("BY", "1"))])[:top]:
    txt = src[L - 1].strip()[:70] if L else "?"
    print(f"{L!s:>5} inst {e / tot_e * 100:5.1f}% stall {s / max(tot_s, 1) * 100:5.1f}%  n={len(ops):3d}  {txt}")
