"""Aggregate an ncu source page of k_simulate by function region (line ranges
of capgpu_device.cuh / capgpu_kernels.cuh / capgpu_gen.h): stall share and
warp instructions per warp-unit.
usage: python tools/prof_regions.py rep.ncu-rep obj.o kernel_regex units"""
import bisect
import collections
import csv
import glob
import io
import os
import re
import subprocess
import sys
import tempfile

rep, obj, kre, units = sys.argv[1], sys.argv[2], sys.argv[3], float(sys.argv[4])
SRC = {"capgpu_device.cuh": "paper_conf_icpp_masw25_b200/csrc/capgpu_device.cuh",
       "capgpu_kernels.cuh": "paper_conf_icpp_masw25_b200/csrc/capgpu_kernels.cuh",
       "capgpu_gen.h": "gen/capgpu_gen.h"}
starts = {}
for f, p in SRC.items():
    st = []
    for i, ln in enumerate(open(p), 1):
        m = re.match(r"^(?:__device__|__global__|GEN_HD)[^(]*?\b(\w+)\s*\(", ln) or \
            re.match(r"^\s+(k_\w+)\(DevParams", ln)
        if m:
            st.append((i, m.group(1)))
    starts[f] = st
sass = (open(rep).read() if rep.endswith(".csv") else
        subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                       capture_output=True, text=True).stdout)
srows = list(csv.reader(io.StringIO(sass)))
sh, sd = srows[1], srows[2:]
tmp = tempfile.mkdtemp()
subprocess.run(["cuobjdump", "-xelf", "all", os.path.abspath(obj)], cwd=tmp, capture_output=True)
cub = glob.glob(os.path.join(tmp, "*.cubin"))[0]
dis = subprocess.run(["nvdisasm", "--print-line-info", "-c", cub], capture_output=True, text=True).stdout
a2l, cur, on = {}, None, False
for ln in dis.splitlines():
    if re.match(r"^//-+ \.text\.", ln):
        if on:
            break
        on = re.search(kre, ln) is not None
        continue
    if not on:
        continue
    m = re.search(r'//## File "([^"]+)", line (\d+)', ln)
    if m:
        cur = (os.path.basename(m.group(1)), int(m.group(2)))
        continue
    m = re.match(r"\s*/\*([0-9a-f]{4,})\*/", ln)
    if m and cur:
        a2l[int(m.group(1), 16)] = cur
iA, iE = sh.index("Address"), sh.index("Instructions Executed")
iSt = sh.index("Warp Stall Sampling (All Samples)")
base = None
st, ins = collections.Counter(), collections.Counter()
for r in sd:
    try:
        a, e, s = int(r[iA], 16), float(r[iE] or 0), float(r[iSt] or 0)
    except (ValueError, IndexError):
        continue
    base = a if base is None else base
    f, line = a2l.get(a - base, ("?", 0))
    name = f
    if f in starts:
        ls = starts[f]
        k = bisect.bisect_right([x[0] for x in ls], line) - 1
        name = f"{f}:{ls[k][1]}" if k >= 0 else f
    st[name] += s
    ins[name] += e
W = units / 32
tot = sum(st.values()) or 1
print(f"{'region':45s} {'stall%':>7s} {'winst/wunit':>12s}")
for k, v in st.most_common():
    print(f"{k:45s} {v / tot * 100:7.1f} {ins[k] / W:12.1f}")
