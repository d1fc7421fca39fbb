"""Summarise an ncu --set full report: key metrics per kernel + top SASS stalls."""
import csv, subprocess, sys, io
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
h = r[0]
ki, mi, vi, ui, ii = (h.index(x) for x in ("Kernel Name", "Metric Name", "Metric Value", "Metric Unit", "ID"))
want = ["Duration", "DRAM Throughput", "Memory Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Compute (SM) Throughput",
        "Executed Ipc Active", "Issue Slots Busy", "Achieved Occupancy", "Theoretical Occupancy", "Registers Per Thread",
        "Grid Size", "Block Size", "Dynamic Shared Memory Per Block"]
cur = None
for x in r[1:]:
    if x[mi] in want:
        if x[ii] != cur:
            cur = x[ii]
            print(f"--- [{cur}] {x[ki][:90]}")
        print(f"    {x[mi]:32s} {x[vi]} {x[ui]}")
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rr = list(csv.reader(io.StringIO(raw)))
hh = rr[0]
cols = [i for i, n in enumerate(hh) if n in ("dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum",
                                             "lts__t_bytes.sum", "l1tex__t_bytes.sum")]
units = rr[1]
for row in rr[2:]:
    print("raw:", row[hh.index("Kernel Name")][:50], {hh[i] + f"[{units[i]}]": row[i] for i in cols})
