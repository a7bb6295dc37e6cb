#!/usr/bin/env python
"""DRAM traffic per launch of one kernel from an `ncu --set full` report, into
profiles/traffic.json (read by bench.py for roofline.traffic).

    python tools/ncu_traffic.py gpurun_out/prof_persist.ncu-rep k_persist s24 [--out profiles/traffic.json]
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def to_bytes(val: str, unit: str) -> float:
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    return float(val.replace(",", "")) * scale.get(unit, 1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("kernel")
    ap.add_argument("config")
    ap.add_argument("--out", default=os.path.join(ROOT, "profiles", "traffic.json"))
    args = ap.parse_args()
    import bench
    raw = subprocess.run(["ncu", "-i", args.report, "--page", "raw", "--csv"], capture_output=True, text=True,
                         check=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    ci = {h: i for i, h in enumerate(hdr)}
    per = []
    for r in data:
        if args.kernel not in r[ci["Kernel Name"]]:
            continue
        rd = to_bytes(r[ci["dram__bytes_read.sum"]], units[ci["dram__bytes_read.sum"]])
        wr = to_bytes(r[ci["dram__bytes_write.sum"]], units[ci["dram__bytes_write.sum"]])
        t = float(r[ci["gpu__time_duration.sum"]].replace(",", ""))
        tu = units[ci["gpu__time_duration.sum"]]
        t_ms = t * {"nsecond": 1e-6, "ns": 1e-6, "usecond": 1e-3, "us": 1e-3, "msecond": 1.0, "ms": 1.0,
                     "second": 1e3, "s": 1e3}[tu]
        per.append((rd, wr, t_ms))
    if not per:
        sys.exit(f"no launches of {args.kernel} in {args.report}")
    n = len(per)
    rec = {"dram_bytes_per_launch": int(sum(a + b for a, b, _ in per) / n),
           "dram_read_bytes_per_launch": int(sum(a for a, _, _ in per) / n),
           "dram_write_bytes_per_launch": int(sum(b for _, b, _ in per) / n),
           "launches": n, "ncu_ms_per_launch": round(sum(t for *_, t in per) / n, 4),
           "source": f"{os.path.basename(args.report)} (ncu --set full --clock-control none, bench.py timed roots)"}
    d = {}
    if os.path.exists(args.out):
        d = json.load(open(args.out))
    d.setdefault(bench.workload_name(args.config), {})[args.kernel] = rec
    json.dump(d, open(args.out, "w"), indent=1)
    print(json.dumps(rec))


if __name__ == "__main__":
    main()
