#!/usr/bin/env python
"""Summarise ncu captures into profiles/ (committed evidence).

  python scripts/ncu_summary.py --launches gpurun_out/launches.csv --full gpurun_out/prof.ncu-rep \
      --tag r01_v2 [--batch 256]

Writes profiles/<tag>_launches.md (per-kernel share of the step from the
`--metrics gpu__time_duration.sum` launch list: cold-cache, serialised, so compare
SHARES) and profiles/<tag>_conv_full.md (DRAM bytes, tensor-pipe activity, ... per conv
launch from the `--set full` capture), and updates profiles/ncu_summary.json, which
bench.py reads for roofline.traffic."""
import argparse
import csv
import io
import json
import os
import re
import subprocess
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")


def short(name: str) -> str:
    m = re.search(r"otif::(\w+)", name)
    return m.group(1) if m else name.split("(")[0].split("<")[0]


def launches(path, tag):
    text = open(path).read().splitlines()
    start = next(i for i, l in enumerate(text) if l.startswith('"ID"'))
    rows = list(csv.DictReader(io.StringIO("\n".join(text[start:]))))
    rows = [r for r in rows if r.get("Metric Name") == "gpu__time_duration.sum"]
    tot = defaultdict(float)
    cnt = defaultdict(int)
    unit = rows[0]["Metric Unit"] if rows else ""
    for r in rows:
        k = short(r["Kernel Name"])
        v = float(r["Metric Value"].replace(",", ""))
        tot[k] += v
        cnt[k] += 1
    s = sum(tot.values())
    lines = [f"# ncu launch list ({tag})", "", f"Source: `{os.path.basename(path)}` "
             "(`ncu --metrics gpu__time_duration.sum --clock-control none`, cold-cache and serialised: "
             "compare shares, not absolutes).", "",
             f"| kernel | launches | total ({unit}) | mean ({unit}) | share |", "|---|---|---|---|---|"]
    for k in sorted(tot, key=lambda k: -tot[k]):
        lines.append(f"| {k} | {cnt[k]} | {tot[k]:.0f} | {tot[k] / cnt[k]:.1f} | {100 * tot[k] / s:.1f}% |")
    open(os.path.join(PROF, f"{tag}_launches.md"), "w").write("\n".join(lines) + "\n")
    return {k: {"launches": cnt[k], "total": tot[k], "share": tot[k] / s} for k in tot}


METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
           "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
           "sm__ops_path_tensor_src_bf16_dst_fp32.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_bytes.sum",
           "sm__throughput.avg.pct_of_peak_sustained_elapsed", "launch__registers_per_thread",
           "launch__grid_size", "smsp__cycles_active.avg"]


def to_bytes(v, unit):
    f = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9,
         "Tbyte": 1e12}.get(unit, 1)
    return float(v.replace(",", "")) * f


def full(path, tag, names):
    if path.endswith(".csv"):     # raw page exported on the GPU box (the .ncu-rep stays there)
        out = open(path).read()
        out = out[out.index('"ID"'):]
    else:
        out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    hdr, units, rows = r[0], r[1], r[2:]
    col = {h: i for i, h in enumerate(hdr)}
    res = []
    for j, row in enumerate(rows):
        d = {"kernel": short(row[col["Kernel Name"]]), "layer": names[j] if j < len(names) else str(j)}
        for m in METRICS:
            if m in col:
                v = row[col[m]]
                if m.startswith("dram__bytes") or m == "lts__t_bytes.sum":
                    d[m] = to_bytes(v, units[col[m]])
                else:
                    try:
                        d[m] = float(v.replace(",", ""))
                    except ValueError:
                        d[m] = v
                d[m + ".unit"] = units[col[m]]
        res.append(d)
    lines = [f"# ncu --set full: proxy conv kernels (e12s_umma_kernel = resize + E1 + E2, conv_umma_kernel = E3..D1) ({tag})", "",
             f"Source: `{os.path.basename(path)}` (one 4500-frame C2 batch, layers in capture order).", "",
             "| layer | time (us) | DRAM read (MB) | DRAM write (MB) | L2 bytes (MB) | tensor pipe % (mem_tensor) | "
             "tensor realtime % | DRAM % | regs |", "|---|---|---|---|---|---|---|---|---|"]
    def num(v):
        try:
            return float(str(v).replace(",", ""))
        except ValueError:
            return 0.0
    for d in res:
        for m in METRICS:
            if m in d:
                d[m] = num(d[m])
        t = d.get("gpu__time_duration.sum", 0)
        tu = d.get("gpu__time_duration.sum.unit", "")
        t_us = t / 1000 if tu in ("nsecond", "ns") else (t * 1000 if tu in ("msecond", "ms") else t)
        lines.append(f"| {d['layer']} | {t_us:.1f} | {d.get('dram__bytes_read.sum', 0) / 1e6:.1f} | "
                     f"{d.get('dram__bytes_write.sum', 0) / 1e6:.1f} | {d.get('lts__t_bytes.sum', 0) / 1e6:.1f} | "
                     f"{d.get('sm__mem_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed', 0):.1f} | "
                     f"{d.get('TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed', 0):.1f} | "
                     f"{d.get('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 0):.1f} | "
                     f"{d.get('launch__registers_per_thread', 0):.0f} |")
    open(os.path.join(PROF, f"{tag}_conv_full.md"), "w").write("\n".join(lines) + "\n")
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--launches")
    ap.add_argument("--full")
    ap.add_argument("--tag", required=True)
    ap.add_argument("--layers", default="E1+E2,E3,E4,E5,D1")
    ap.add_argument("--no-traffic", action="store_true", help="do not update conv_dram_bytes_per_batch")
    args = ap.parse_args()
    os.makedirs(PROF, exist_ok=True)
    summ_path = os.path.join(PROF, "ncu_summary.json")
    summ = json.load(open(summ_path)) if os.path.exists(summ_path) else {}
    summ["tag"] = args.tag
    if args.launches:
        summ["launch_shares"] = launches(args.launches, args.tag)
    if args.full:
        res = full(args.full, args.tag, args.layers.split(","))
        summ["conv_full" if not args.no_traffic else f"conv_full_{args.tag}"] = res
        if not args.no_traffic:
            summ["conv_dram_bytes_per_batch"] = sum(d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
                                                for d in res)
    json.dump(summ, open(summ_path, "w"), indent=1)
    print(json.dumps({k: v for k, v in summ.items() if k != "conv_full"}, indent=1)[:3000])


if __name__ == "__main__":
    main()
