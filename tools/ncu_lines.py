#!/usr/bin/env python
"""Warp-stall samples of an `ncu --set full --import-source on` report folded
onto CUDA source lines (innermost inlined line) via nvdisasm line info.

    python tools/ncu_lines.py gpurun_out/prof_persist.ncu-rep _ZN4xbfs9k_persistENS_5KArgsEPiS1_PKjx \
        [--so paper_conf_sc_yangls0w24_b200/libxbfs.so] [--top 40] [--launch 0]
"""
import argparse
import collections
import csv
import glob
import io
import os
import re
import subprocess
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def line_map(so: str, func: str):
    tmp = tempfile.mkdtemp()
    subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(so)], cwd=tmp, capture_output=True, check=True)
    for cub in glob.glob(os.path.join(tmp, "*.cubin")):
        full = subprocess.run(["nvdisasm", "-gi", cub], capture_output=True, text=True).stdout
        start = full.find(f".text.{func}:")
        if start < 0:
            continue
        lines = full[start:].splitlines()
        stop = next((i for i, l in enumerate(lines[1:], 1)
                     if l.startswith(".text.") or l.lstrip().startswith(".section")), len(lines))
        out = "\n".join(lines[:stop])
        m, cur = {}, None
        for ln in out.splitlines():
            a = re.match(r'\s*//## File "([^"]+)", line (\d+)', ln)
            if a:
                if cur is None:
                    cur = (os.path.basename(a.group(1)), int(a.group(2)))
                continue
            b = re.match(r"\s*/\*([0-9a-f]{4,})\*/\s+(.*)", ln)
            if b:
                if cur is not None:
                    m[int(b.group(1), 16)] = cur
                    last = cur
                else:
                    m[int(b.group(1), 16)] = last if m else ("?", 0)
                cur = None
        return m
    raise SystemExit(f"{func} not found in {so}")


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("report")
    ap.add_argument("func")
    ap.add_argument("--so", default=os.path.join(ROOT, "paper_conf_sc_yangls0w24_b200", "libxbfs.so"))
    ap.add_argument("--top", type=int, default=40)
    ap.add_argument("--launch", type=int, default=0)
    args = ap.parse_args()
    lm = line_map(args.so, args.func)
    raw = subprocess.run(["ncu", "-i", args.report, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True, check=True).stdout
    blocks = [b for b in raw.split('"Kernel Name"') if b.strip()]
    body = blocks[min(args.launch, len(blocks) - 1)]
    rows = list(csv.reader(io.StringIO(body.split("\n", 1)[1])))
    hdr = rows[0]
    ci = {h: i for i, h in enumerate(hdr)}
    stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
    base = min(int(r[ci["Address"]], 16) for r in rows[1:] if r and r[0].startswith("0x"))
    agg = collections.defaultdict(lambda: collections.Counter())
    tot = 0
    for r in rows[1:]:
        if not r or not r[0].startswith("0x"):
            continue
        off = int(r[ci["Address"]], 16) - base
        key = lm.get(off, ("?", 0))
        s = int(r[ci["Warp Stall Sampling (All Samples)"]] or 0)
        agg[key]["samples"] += s
        tot += s
        for c in stall_cols:
            v = r[ci[c]]
            if v and v != "0":
                agg[key][c] += int(float(v))
    src = {}
    for f in ("bfs.cu", "bu_core.cuh", "common.cuh"):
        p = os.path.join(ROOT, "paper_conf_sc_yangls0w24_b200", "csrc", f)
        if os.path.exists(p):
            src[f] = open(p).read().splitlines()
    print(f"total samples {tot}")
    for key, c in sorted(agg.items(), key=lambda kv: -kv[1]["samples"])[: args.top]:
        f, ln = key
        text = src.get(f, [""] * (ln + 1))[ln - 1].strip()[:70] if ln else ""
        top = ", ".join(f"{k[6:]}={v}" for k, v in c.most_common(4) if k != "samples")
        print(f"{100 * c['samples'] / max(tot, 1):5.1f}% {f}:{ln:<5} {text:<70} | {top}")


if __name__ == "__main__":
    main()
