import csv, sys, subprocess
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(out.splitlines()))
h = r[0]
want = ["Duration", "Elapsed Cycles", "SM Active Cycles", "Compute (SM) Throughput", "Memory Throughput",
        "DRAM Throughput", "L1/TEX Cache Throughput", "L2 Cache Throughput", "Executed Ipc Active",
        "Issue Slots Busy", "Registers Per Thread", "Achieved Active Warps Per SM", "L1/TEX Hit Rate",
        "L2 Hit Rate", "Executed Instructions", "Grid Size", "Block Size", "No Eligible",
        "Warp Cycles Per Issued Instruction", "Dynamic Shared Memory Per Block", "Theoretical Occupancy"]
for row in r[1:]:
    d = dict(zip(h, row))
    if d.get("Metric Name") in want:
        print(d["Kernel Name"][:40].ljust(40), d["Metric Name"].ljust(36), d["Metric Value"], d["Metric Unit"])
