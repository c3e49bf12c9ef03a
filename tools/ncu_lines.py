#!/usr/bin/env python
"""Aggregate an ncu source-page (SASS) profile to CUDA source lines via nvdisasm -g.
usage: tools_ncu_lines.py report.ncu-rep kernel_regex mangled_name [topN]"""
import collections, csv, io, os, re, subprocess, sys, tempfile

rep, kre, mangled = sys.argv[1], sys.argv[2], sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 25
lib = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "paper_conf_ipps_tayebbfg24_b200", "libmp.so")
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", lib], cwd=tmp, capture_output=True)
cub = [f for f in os.listdir(tmp) if f.endswith(".cubin")][0]
sass = subprocess.run(["nvdisasm", "-g", "-c", os.path.join(tmp, cub)], capture_output=True, text=True).stdout.split("\n")
start = next(i for i, l in enumerate(sass) if f".text.{mangled}:" in l)
cur, fmap, fname = None, {}, {}
for l in sass[start + 1:]:
    if l.startswith("\t.section") or l.startswith(".section"):
        break
    m = re.search(r'//## File "([^"]+)", line (\d+)', l)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    mo = re.match(r"\s*/\*([0-9a-f]{4,})\*/", l)
    if mo and cur:
        fmap[int(mo.group(1), 16)] = cur
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{kre}"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]
I = {k: i for i, k in enumerate(h)}
data, seen = [], set()
for r in rows[2:]:
    if len(r) == len(h) and r[0].startswith("0x") and r[0] not in seen:
        seen.add(r[0]); data.append(r)
base = int(data[0][0], 16)
col = os.environ.get("NCU_COL", "Warp Stall Sampling (All Samples)")
agg = collections.Counter()
reasons = collections.defaultdict(collections.Counter)
rcols = [k for k in h if k.startswith("stall_") and "Not Issued" not in k]
for r in data:
    key = fmap.get(int(r[0], 16) - base)
    agg[key] += int(r[I[col]] or 0)
    for k in rcols:
        reasons[key][k[6:]] += int(r[I[k]] or 0)
tot = sum(agg.values()) or 1
srcs = {}
for (k, c) in agg.most_common(top):
    if k is None:
        print(f"{100*c/tot:5.1f}%  ?"); continue
    f, ln = k
    k = (f, ln)
    if f not in srcs:
        p = os.path.join(os.path.dirname(lib), "csrc", f)
        srcs[f] = open(p).read().split("\n") if os.path.exists(p) else []
    txt = srcs[f][ln - 1].strip() if ln - 1 < len(srcs[f]) else ""
    rs = " ".join(f"{k}:{v}" for k, v in reasons[k].most_common(3) if v) if os.environ.get("REASONS") else ""
    print(f"{100*c/tot:5.1f}%  {f}:{ln}  {txt[:90]}  {rs}")
