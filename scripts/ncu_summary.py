"""Summarise an .ncu-rep: key throughput metrics, stall breakdown, top stalled SASS lines."""
import csv, io, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25

def ncu(*a):
    return subprocess.run(["ncu", "-i", rep, *a], capture_output=True, text=True).stdout

det = list(csv.reader(io.StringIO(ncu("--page", "details", "--csv"))))
h = det[0]
si, mi, ui, vi = h.index("Section Name"), h.index("Metric Name"), h.index("Metric Unit"), h.index("Metric Value")
want = ["Duration", "DRAM Throughput", "Memory Throughput", "L2 Cache Throughput", "L1/TEX Cache Throughput",
        "Compute (SM) Throughput", "L2 Hit Rate", "L1/TEX Hit Rate", "Issue Slots Busy", "Executed Ipc Active",
        "Achieved Occupancy", "Registers Per Thread", "Executed Instructions", "Warp Cycles Per Issued Instruction",
        "Eligible Warps Per Scheduler", "No Eligible"]
for r in det[1:]:
    if r[mi] in want:
        print(f"{r[mi]:40s} {r[vi]:>16s} {r[ui]}")
raw = list(csv.reader(io.StringIO(ncu("--page", "raw", "--csv"))))
hdr = raw[0]
for name in ("dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "sm__warps_active.avg.pct_of_peak_sustained_active"):
    if name in hdr:
        i = hdr.index(name)
        print(f"{name:40s} {raw[2][i]:>16s} {raw[1][i]}")
ws = list(csv.reader(io.StringIO(ncu("--page", "details", "--csv", "--section", "WarpStateStats", "--details-all"))))
print("-- warp state (cycles per issued instruction)")
for r in ws[1:]:
    if len(r) > vi and r[mi].startswith("Stall") or (len(r) > vi and r[mi] == "Selected"):
        try:
            if float(r[vi]) >= 0.2: print(f"   {r[mi]:32s} {r[vi]}")
        except ValueError:
            pass
src = list(csv.reader(io.StringIO(ncu("--page", "source", "--csv", "--print-source", "sass"))))
h = src[1]
ai, ssi, wi, ei = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
rows = []
for r in src[2:]:
    try:
        rows.append((float(r[wi] or 0), float(r[ei] or 0), r[ssi]))
    except (ValueError, IndexError):
        pass
tot = sum(x[0] for x in rows) or 1
print(f"-- top stalled SASS (of {int(tot)} samples)")
for w, e, s in sorted(rows, reverse=True)[:top]:
    print(f"  {100*w/tot:5.1f}% {e/1e6:8.2f}M  {s.strip()[:90]}")
