"""Per-kernel table (means over launches) of an ncu_summary.py text file."""
import collections
import re
import sys

KEYS = {"gpu__time_duration.sum": "ms", "dram__bytes_read.sum": "rdGB", "dram__bytes_write.sum": "wrGB",
        "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue%",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed": "L2%",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram%",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio": "lsb",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio": "bar",
        "sm__warps_active.avg.per_cycle_active": "warps", "launch__registers_per_thread": "regs",
        "smsp__inst_executed.sum": "Minst"}
acc = collections.defaultdict(lambda: collections.defaultdict(list))
name = None
for ln in open(sys.argv[1]):
    if ln.startswith("-----"):
        name = re.sub(r"\(.*", "", ln[6:].strip()).replace("void ", "")
        continue
    parts = ln.split()
    if name and len(parts) >= 2 and parts[0] in KEYS:
        acc[name][KEYS[parts[0]]].append(float(parts[1]))
cols = ["n", "ms", "rdGB", "wrGB", "dram%", "L2%", "issue%", "lsb", "bar", "warps", "regs", "Minst"]
print(f"{'kernel':42s}" + "".join(f"{c:>8s}" for c in cols))
for k, d in sorted(acc.items(), key=lambda kv: -sum(kv[1]["ms"])):
    row = [len(d["ms"])] + [sum(d[c]) / len(d[c]) if d[c] else 0 for c in cols[1:]]
    row[-1] /= 1e6
    print(f"{k[:42]:42s}" + "".join(f"{x:8.3f}" if isinstance(x, float) else f"{x:8d}" for x in row))
