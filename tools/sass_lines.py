"""Join an ncu SASS source page (csv) with nvdisasm line info: instructions per source line.
usage: python tools/sass_lines.py <sass.csv> <disasm.txt> <work_units> [top]"""
import collections
import csv
import re
import sys

csv_path, dis_path, units = sys.argv[1], sys.argv[2], float(sys.argv[3])
top = int(sys.argv[4]) if len(sys.argv) > 4 else 45
cur = None
addr2line = {}
stack = []
for ln in open(dis_path):
    m = re.search(r'//## File "([^"]+)", line (\d+)(.*)', ln)
    if m:
        cur = (m.group(1).split('/')[-1], int(m.group(2)))
        continue
    m = re.match(r'\s*/\*([0-9a-f]{4,})\*/', ln)
    if m and cur:
        addr2line[int(m.group(1), 16)] = cur
rows = list(csv.reader(open(csv_path)))
hdr = rows[1]
data = rows[2:]
iA, iE, iS = hdr.index("Address"), hdr.index("Instructions Executed"), hdr.index("Source")
base = None
agg = collections.Counter()
aggop = collections.defaultdict(collections.Counter)
for r in data:
    try:
        a = int(r[iA], 16)
        e = float(r[iE] or 0)
    except Exception:
        continue
    if base is None:
        base = a
    key = addr2line.get(a - base, ('?', 0))
    agg[key] += e
    op = re.match(r'\s*(@!?U?P\w+\s+)?([A-Z0-9_]+)', r[iS])
    aggop[key][op.group(2) if op else '?'] += e
for k, v in agg.most_common(top):
    print(f"{k[0]:22s}:{k[1]:4d} {v * 32 / units:8.1f}/unit  {dict(aggop[k].most_common(4))}")
