"""Print selected ncu --page details sections for kernels matching a substring."""
import csv, subprocess, sys
rep, pat = sys.argv[1], sys.argv[2]
secs = sys.argv[3].split(",") if len(sys.argv) > 3 else ["GPU Speed Of Light Throughput", "Memory Workload Analysis",
                                                          "Occupancy", "Warp State Statistics", "Scheduler Statistics",
                                                          "Compute Workload Analysis", "Launch Statistics"]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(out.splitlines()))
h = r[0]
ki, si, mi, vi, ui = (h.index(x) for x in ("Kernel Name", "Section Name", "Metric Name", "Metric Value", "Metric Unit"))
for row in r[1:]:
    if pat in row[ki] and row[si] in secs:
        print(f"{row[si][:18]:18s} | {row[mi]:45s} | {row[vi]} {row[ui]}")
