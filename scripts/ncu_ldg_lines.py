"""Global-load sectors by source line from an ncu --set full capture: for
every LDG of a kernel, ncu's "L2 Theoretical Sectors Global" (sectors the
instruction requests from L2) summed per nulpa.cu line, so the label
gathers C[j] (Algorithm 1) separate from the CSR streams.

usage: python scripts/ncu_ldg_lines.py <report.ncu-rep> <mangled-kernel-substring> [launch-index]
"""
import collections, csv, io, os, re, subprocess, sys, tempfile

rep, kname = sys.argv[1], sys.argv[2]
launch = sys.argv[3] if len(sys.argv) > 3 else "0"
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
lib = os.path.join(ROOT, "paper_conf_ipps_sahunk25_b200", "libnulpa.so")
src_lines = open(os.path.join(ROOT, "paper_conf_ipps_sahunk25_b200", "csrc", "nulpa.cu")).read().split("\n")
d = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=d, capture_output=True, check=True)
cubin = os.path.join(d, [f for f in os.listdir(d) if f.endswith(".cubin")][0])
dis = subprocess.run(["nvdisasm", "-g", cubin], capture_output=True, text=True).stdout
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
                      "--launch-skip", launch, "--launch-count", "1"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
h = rows[hi]
ia, isrc, isec = h.index("Address"), h.index("Source"), h.index("L2 Theoretical Sectors Global")
ireq = h.index("L1 Tag Requests Global")
agg = collections.defaultdict(lambda: [0, 0])
base, seen = None, set()
for r in rows[hi + 1:]:
    if len(r) <= isec or not r[ia].startswith("0x"):
        continue
    a = int(r[ia], 16)
    base = a if base is None else base
    if a in seen:
        continue
    seen.add(a)
    if "LDG" not in r[isrc]:
        continue
    L = line_of.get(a - base)
    agg[L][0] += int(r[isec] or 0)
    agg[L][1] += int(r[ireq] or 0)
tot = sum(v[0] for v in agg.values())
print(f"{'line':>5} {'sectors':>10} {'share':>6} {'per req':>7}  source")
for L, (sec, req) in sorted(agg.items(), key=lambda kv: -kv[1][0]):
    txt = src_lines[L - 1].strip()[:90] if L else "?"
    print(f"{L or 0:5d} {sec / 1e6:9.1f}M {sec / tot * 100:5.1f}% {sec / max(req, 1):7.2f}  {txt}")
print(f"total {tot / 1e6:.1f}M sectors")
