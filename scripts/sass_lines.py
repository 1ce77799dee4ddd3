"""Join an ncu SASS source page (CSV, --print-source sass) with line info from nvdisasm -gi
of the same build: per CUDA source line (innermost non-header site and its caller in
proxy.cu), warp-stall samples and executed instructions.

usage: python scripts/sass_lines.py <ncu_source.csv> <cubin> <mangled kernel> [top]"""
import collections, csv, re, subprocess, sys

src_csv, cubin, kern = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
dis = subprocess.run(["nvdisasm", "-gi", cubin], capture_output=True, text=True).stdout
# function blocks: ".text.<name>:" headers
blocks = re.split(r"\n\s*\.section\s+\.text\.", dis)
body = next(b for b in blocks if b.startswith(kern))
addr_line = {}
cur = None
for ln in body.split("\n"):
    m = re.search(r"//## File \"([^\"]+)\", line (\d+)(.*)", ln)
    if m:
        f = m.group(1).split("/")[-1]
        cur = (f, int(m.group(2)), m.group(3).strip())
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m and cur:
        addr_line[int(m.group(1), 16)] = cur
rows = list(csv.reader(open(src_csv)))
hi = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
hdr = rows[hi]
ia, isamp, iins = hdr.index("Address"), hdr.index("Warp Stall Sampling (All Samples)"), hdr.index("Instructions Executed")
stall_cols = [(i, h) for i, h in enumerate(hdr) if h.startswith("stall_") and "Not Issued" not in h]
agg = collections.defaultdict(lambda: [0, 0, collections.Counter()])
tot = 0
base = None
for r in rows[hi + 1:]:
    if len(r) <= iins or not r[ia].startswith("0x"):
        continue
    a = int(r[ia], 16)
    base = a if base is None else base      # ncu prints absolute addresses: offset from the entry
    a -= base
    key = addr_line.get(a, ("?", 0, ""))
    s = float(r[isamp] or 0)
    agg[key][0] += s
    agg[key][1] += float(r[iins] or 0)
    for i, h in stall_cols:
        agg[key][2][h[6:]] += float(r[i] or 0)
    tot += s
print(f"total samples {tot:.0f}")
for key, (s, ins, st) in sorted(agg.items(), key=lambda kv: -kv[1][0])[:top]:
    dom = ", ".join(f"{k} {v / max(s, 1):.0%}" for k, v in st.most_common(2))
    print(f"{s / tot:6.1%} {ins:12.0f}  {key[0]}:{key[1]} {key[2][:60]}  [{dom}]")
