"""Write profiles/<tag>_launches_<config>.md from a campaign's ncu CSVs:
the launch list of the bench command (bench.py --steps 2 --warmup 1, timing
only) and of one nu-LPA run with DRAM bytes (scripts/profile_run.py --runs 1).
usage: python scripts/launch_md.py <tag> <config>"""
import subprocess, sys, os
tag, cfg = sys.argv[1], sys.argv[2]
R = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
def table(path):
    return subprocess.run([sys.executable, os.path.join(R, "scripts", "launch_table.py"), path], capture_output=True, text=True).stdout
out = [f"# {tag}: ncu launch lists, {cfg}", "",
       "Cold, serialised launches (`ncu --clock-control none`); absolute times are not bench values, shares are.", "",
       f"## Bench command: `python bench.py --config {cfg} --steps 2 --warmup 1 --no-e2e --no-cpu-baseline --quality-runs 0`", "",
       "(`ncu --metrics gpu__time_duration.sum`; includes the untimed warm-up, serialised and modularity runs)", "", "```",
       table(os.path.join(R, "gpurun_out", f"{tag}_launches_{cfg}.csv")).rstrip(), "```", "",
       f"## One run with DRAM bytes: `python scripts/profile_run.py --config {cfg} --runs 1`", "",
       "(`ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum`; per-sweep DRAM bytes of the dominant bin in profiles/traffic.json)", "", "```",
       table(os.path.join(R, "gpurun_out", f"{tag}_traffic_{cfg}.csv")).rstrip(), "```", ""]
open(os.path.join(R, "profiles", f"{tag}_launches_{cfg}.md"), "w").write("\n".join(out))
print("wrote", f"profiles/{tag}_launches_{cfg}.md")
