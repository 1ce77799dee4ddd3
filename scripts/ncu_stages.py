#!/usr/bin/env python
"""Summarise the ncu --set full capture of resize / select / pack (scripts/prof_stages.sh)
into profiles/<tag>_stages.md: per launch the duration, DRAM bytes read + written, DRAM
throughput, and the algorithmic bytes of that launch (scripts/prof_stages.py) with the
traffic / algorithmic ratio (> 1 = re-reads).

    python scripts/ncu_stages.py --raw gpurun_out/r02e_stages_raw.csv --alg gpurun_out/r02e_stages.json --tag r02e
"""
import argparse
import csv
import io
import json
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
           "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
           "l1tex__throughput.avg.pct_of_peak_sustained_active", "lts__t_bytes.sum",
           "launch__registers_per_thread", "launch__grid_size", "sm__warps_active.avg.pct_of_peak_sustained_active"]
SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "nsecond": 1e-9, "usecond": 1e-6, "msecond": 1e-3,
         "ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1,
         "second": 1}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--raw", required=True)
    ap.add_argument("--alg", required=True)
    ap.add_argument("--tag", required=True)
    a = ap.parse_args()
    text = open(a.raw).read().splitlines()
    start = next(i for i, l in enumerate(text) if l.startswith('"ID"'))
    rows = list(csv.reader(io.StringIO("\n".join(text[start:]))))
    head, units, data = rows[0], rows[1], rows[2:]
    col = {h: i for i, h in enumerate(head)}
    alg = json.loads([l for l in open(a.alg).read().splitlines() if l.startswith("{")][-1])
    # launch order in prof_stages.py (select launches K5 once, or twice with a deferred pass)
    order = ["resize", "select_random", "pack_full", "select_trained_C2", "select_trained_C2s", "pack_multi_C2s"]
    out, recs = [], []
    seen = {"resize": 0, "select": 0, "pack": 0}
    rs_names = ["resize", "resize_C3"]
    sel_names = ["select_random", "select_trained_C2", "select_trained_C2s"]
    pack_names = ["pack_full", "pack_multi_C2s", "pack_full_C3"]
    for r in data:
        name = r[col["Kernel Name"]]

        def val(m):
            if m not in col or not r[col[m]]:
                return None
            v = float(r[col[m]].replace(",", ""))
            return v * SCALE.get(units[col[m]], 1)
        if "resize_even" in name:
            key = rs_names[min(seen["resize"], 1)]
            seen["resize"] += 1
        elif "select_kernel" in name:
            # each select call launches K5 twice (the small-slice pass and the deferred
            # full-slice pass, usually empty): pair them up, report the pass-0 launch
            key = sel_names[min(seen["select"] // 2, 2)] + ("" if seen["select"] % 2 == 0 else "_pass1")
            seen["select"] += 1
        elif "pack_kernel" in name:
            key = pack_names[min(seen["pack"], 2)]
            seen["pack"] += 1
        else:
            continue
        t = val("gpu__time_duration.sum")
        rd, wr = val("dram__bytes_read.sum") or 0, val("dram__bytes_write.sum") or 0
        ab = alg.get(key, {}).get("algorithmic_bytes")
        rec = {"kernel": key, "ncu_name": name.split("(")[0][:60], "time_ms": t * 1e3 if t else None,
               "dram_read_gb": rd / 1e9, "dram_write_gb": wr / 1e9, "dram_gbs": (rd + wr) / t / 1e9 if t else None,
               "dram_pct_peak": val("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
               "algorithmic_gb": ab / 1e9 if ab else None,
               "traffic_over_algorithmic": (rd + wr) / ab if ab else None,
               "registers": val("launch__registers_per_thread"), "grid": val("launch__grid_size")}
        recs.append(rec)
    md = [f"# ncu --set full: resize / select / pack ({a.tag})", "",
          "Captured with `TAG=%s bash scripts/prof_stages.sh` (one isolated launch each, cold L2, clocks not locked)." % a.tag,
          "Algorithmic bytes from `scripts/prof_stages.py` (resize: 2 of 4 source rows + output; select: scores + windows;",
          "pack: 2 x window bytes).  traffic / algorithmic > 1 means re-reads.", "",
          "| launch | ms | DRAM read GB | DRAM write GB | DRAM GB/s | DRAM % peak | algorithmic GB | traffic / alg |",
          "|---|---|---|---|---|---|---|---|"]
    for x in recs:
        f = lambda v, d=3: "-" if v is None else f"{v:.{d}f}"
        md.append(f"| {x['kernel']} | {f(x['time_ms'])} | {f(x['dram_read_gb'])} | {f(x['dram_write_gb'])} | "
                  f"{f(x['dram_gbs'], 0)} | {f(x['dram_pct_peak'], 1)} | {f(x['algorithmic_gb'])} | "
                  f"{f(x['traffic_over_algorithmic'], 2)} |")
    path = os.path.join(ROOT, "profiles", f"{a.tag}_stages.md")
    open(path, "w").write("\n".join(md) + "\n")
    json.dump(recs, open(os.path.join(ROOT, "profiles", f"{a.tag}_stages.json"), "w"), indent=1)
    print("\n".join(md))


if __name__ == "__main__":
    main()
