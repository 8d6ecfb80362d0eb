"""Fold gpurun_out/traffic_<W>.csv (tools/traffic.sh) into profiles/traffic.json:
{workload: {kernel: dram read+write bytes of its LAST launch in the run}}."""
import csv
import glob
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12,
        "nsecond": 1, "usecond": 1e3, "msecond": 1e6, "second": 1e9,
        "inst": 1, "Kinst": 1e3, "Minst": 1e6, "Ginst": 1e9}


def parse(path):
    rows = [r for r in csv.reader(open(path)) if r]
    hi = next(i for i, r in enumerate(rows) if "Kernel Name" in r)
    h = rows[hi]
    per = {}
    for r in rows[hi + 1:]:
        if len(r) != len(h):
            continue
        name = r[h.index("Kernel Name")]
        k = re.search(r"(tile_reduce_kernel|brick_reduce_kernel|reduce_kernel|table_scan_kernel)", name)
        if not k:
            continue
        lid = r[h.index("ID")]
        m = r[h.index("Metric Name")]
        v = float(r[h.index("Metric Value")].replace(",", "")) * UNIT.get(r[h.index("Metric Unit")], 1)
        per.setdefault((k.group(1), int(lid)), {})[m] = v
    out = {}
    for (k, lid), ms in sorted(per.items(), key=lambda x: x[0][1]):
        out[k] = int(ms.get("dram__bytes_read.sum", 0) + ms.get("dram__bytes_write.sum", 0))
        if "smsp__inst_executed.sum" in ms:
            out[k + ":inst"] = int(ms["smsp__inst_executed.sum"])
        if "gpu__time_duration.sum" in ms:
            out[k + ":ncu_ms"] = ms["gpu__time_duration.sum"] / 1e6  # nsecond -> ms
    return out


def main():
    tp = os.path.join(ROOT, "profiles", "traffic.json")
    data = json.load(open(tp)) if os.path.exists(tp) else {}
    for p in sorted(glob.glob(os.path.join(ROOT, "gpurun_out", "traffic_*.csv"))):
        w = os.path.basename(p)[len("traffic_"):-4]
        if w not in ("C1", "C2a", "C2b", "C3", "C4", "C5", "T", "R"):  # experiment captures are not bench workloads
            continue
        try:
            data[w] = parse(p)
        except StopIteration:
            print("no kernels in", p, file=sys.stderr)
    data["_source"] = ("ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum,"
                       "gpu__time_duration.sum --clock-control none on the reduce kernels of a 1-warm-up + 1-step "
                       "bench.py run per workload (tools/traffic.sh); <kernel> = DRAM read + write bytes of its last "
                       "launch (per launch = per batch), <kernel>:inst = warp instructions executed by that launch, "
                       "<kernel>:ncu_ms its (serialised, cold-cache) duration")
    json.dump(data, open(tp, "w"), indent=1, sort_keys=True)
    print(json.dumps(data, indent=1, sort_keys=True))


if __name__ == "__main__":
    main()
