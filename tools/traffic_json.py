"""DRAM traffic per launch of every phase-1 kernel class, from one `ncu --set full` capture of a
whole gala_run (tools/profile_run.py, cuda_graph=0), written to profiles/traffic.json for
bench.py's roofline `traffic` field.

traffic[class] = sum over the class's kernels of (dram__bytes_read.sum + dram__bytes_write.sum)
                 / number of class launches (= launches of the class's anchor kernel, matching
                 the library's per-class launch counter: one Timer interval per anchor).
usage: python tools/traffic_json.py <report.ncu-rep> <config> [out.json]   (merged per config)
"""
import csv
import json
import re
import subprocess
import sys

# (class, kernel-name regex, is-anchor)
CLASSES = [
    ("prune_bin", r"^k_prune_bin", True),
    ("decide_single", r"^k_decide_single", True),          # k_decide_single_small + k_decide_single
    ("decide_small", r"^k_decide_small", True),
    ("decide_warp", r"^k_decide_warp<32, 128", True),
    ("decide_warp512", r"^k_decide_warp<32, 512", True),
    ("decide_block", r"^k_decide_block", True),
    ("decide_hub", r"^k_hub_prep[(<]", True),
    ("decide_hub", r"^k_decide_cluster", True),             # hubs on a thread-block cluster
    ("decide_hub", r"^k_hub_(agg|prep2|eval|final|single)", False),
    ("apply", r"^k_apply", True),
    ("dp_update", r"^k_dp_delta", True),
    ("dp_update", r"^k_(dp_full|sm_flags)", False),
    ("reduce", r"^k_reduce", True),
]


def to_bytes(v, unit):
    f = float(v.replace(",", ""))
    return f * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit, 1)


def main(path, config, out):
    raw = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(raw.splitlines()))
    h, units, data = rows[0], rows[1], rows[2:]
    ki, ri, wi = h.index("Kernel Name"), h.index("dram__bytes_read.sum"), h.index("dram__bytes_write.sum")
    acc = {}
    for r in data:
        name = re.sub(r"^void ", "", r[ki])
        for cls, rx, anchor in CLASSES:
            if re.search(rx, name):
                a = acc.setdefault(cls, {"bytes": 0.0, "launches": 0, "kernels": 0})
                a["bytes"] += to_bytes(r[ri], units[ri]) + to_bytes(r[wi], units[wi])
                a["kernels"] += 1
                a["launches"] += int(anchor)
                break
    res = {c: {"dram_bytes_per_launch": a["bytes"] / max(a["launches"], 1), "launches": a["launches"],
               "kernels": a["kernels"], "source": path} for c, a in acc.items()}
    try:
        allres = json.load(open(out))
    except (OSError, ValueError):
        allres = {}
    allres[config] = res
    json.dump(allres, open(out, "w"), indent=1, sort_keys=True)
    print(json.dumps(res, indent=1, sort_keys=True))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], sys.argv[3] if len(sys.argv) > 3 else "profiles/traffic.json")
