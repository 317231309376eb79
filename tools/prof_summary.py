"""Summarise an ncu report of k_simulate: headline metrics, opcode mix and
per-source-line cost (warp instructions per warp-step) joined with nvdisasm
line info.  usage: python tools/prof_summary.py rep.ncu-rep obj.o kernel_regex units [top]"""
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
top = int(sys.argv[5]) if len(sys.argv) > 5 else 30
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, un, val = rows[0], rows[1], rows[2]
want = ["gpu__time_duration.sum", "launch__registers_per_thread", "launch__block_size", "launch__grid_size",
        "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct",
        "sm__warps_active.avg.per_cycle_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "sass__inst_executed_local_loads",
        "launch__occupancy_limit_shared_mem", "launch__occupancy_limit_registers"]
for i, h in enumerate(hdr):
    if h in want or (h.startswith("smsp__average_warps_issue_stalled") and h.endswith("per_issue_active.ratio")):
        try:
            if h.startswith("smsp__average_warps_issue_stalled") and float(val[i]) < 0.1:
                continue
        except ValueError:
            pass
        print(f"  {h} = {val[i]} {un[i]}")
sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                      capture_output=True, text=True).stdout
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
iA, iS, iE = sh.index("Address"), sh.index("Source"), sh.index("Instructions Executed")
iT, iSt = sh.index("Thread Instructions Executed"), sh.index("Warp Stall Sampling (All Samples)")
base = None
st, ins, thr, opc = (collections.Counter() for _ in range(4))
for r in sd:
    try:
        a, e, s, t = int(r[iA], 16), float(r[iE] or 0), float(r[iSt] or 0), float(r[iT] or 0)
    except (ValueError, IndexError):
        continue
    base = a if base is None else base
    k = a2l.get(a - base, ("?", 0))
    st[k] += s
    ins[k] += e
    thr[k] += t
    m = re.match(r"\s*(@!?U?P\w+\s+)?([A-Z0-9_]+)", r[iS])
    opc[m.group(2) if m else "?"] += e
W = units / 32
print(f"  static instructions mapped: {len(a2l)}; warp-instr per warp-unit: {sum(ins.values()) / W:.1f}")
print("  ops:", ", ".join(f"{k} {v / W:.0f}" for k, v in opc.most_common(16)))
tot = sum(st.values()) or 1
for k, v in st.most_common(top):
    print(f"  {k[0]:20s}:{k[1]:4d} stall {v / tot * 100:5.1f}%  winst/wunit {ins[k] / W:7.1f}  thr/inst {thr[k] / max(ins[k], 1):5.1f}")
