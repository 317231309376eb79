"""Per-source-line instructions and stall samples of one kernel from an ncu
source page (csv, --print-source sass) joined with `nvdisasm -g` line info.
usage: python tools/src_stalls.py <sass.csv> <disasm.txt> <kernel-mangled-name> [top]"""
import collections
import csv
import re
import sys

csv_path, dis_path, kname = sys.argv[1], sys.argv[2], sys.argv[3]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
addr2line, cur, inside = {}, None, False
for ln in open(dis_path):
    if ln.startswith("//----"):
        inside = kname in ln
        continue
    if not inside:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        cur = (m.group(1).split('/')[-1], int(m.group(2)))
        continue
    m = re.match(r'\s*/\*([0-9a-f]{4,})\*/', ln)
    if m and cur:
        addr2line[int(m.group(1), 16)] = cur
rows = list(csv.reader(open(csv_path)))
hdr = rows[1]
col = {h: i for i, h in enumerate(hdr)}
stall_cols = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
base = None
ins, samp = collections.Counter(), collections.Counter()
stalls = collections.defaultdict(collections.Counter)
ops = collections.defaultdict(collections.Counter)
tot_s = tot_i = 0
for r in rows[2:]:
    try:
        a = int(r[col["Address"]], 16)
    except Exception:
        continue
    if base is None:
        base = a
    key = addr2line.get(a - base, ('?', 0))
    e = float(r[col["Instructions Executed"]] or 0)
    s = float(r[col["Warp Stall Sampling (All Samples)"]] or 0)
    ins[key] += e
    samp[key] += s
    tot_s += s
    tot_i += e
    for h in stall_cols:
        v = float(r[col[h]] or 0)
        if v:
            stalls[key][h[6:]] += v
    op = re.match(r'\s*(@!?U?P\w+\s+)?([A-Z0-9_]+)', r[col["Source"]])
    ops[key][op.group(2) if op else '?'] += e
print(f"total samples {tot_s:.0f}, warp instructions {tot_i:.0f}")
for k, v in samp.most_common(top):
    st = ", ".join(f"{n}:{c / v:.0%}" for n, c in stalls[k].most_common(3))
    print(f"{k[0]:22s}:{k[1]:4d} samp {v / tot_s:6.2%} ins {ins[k] / tot_i:6.2%}  [{st}]  {dict(ops[k].most_common(4))}")
by_file = collections.Counter()
for k, v in samp.items():
    by_file[k[0]] += v
print({f: f"{v / tot_s:.1%}" for f, v in by_file.most_common()})
