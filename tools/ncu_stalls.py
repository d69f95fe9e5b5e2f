"""Kernel-wide warp-stall breakdown (sum over SASS lines) + key details metrics.  Usage: ncu_stalls.py rep"""
import csv, subprocess, sys, collections
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines())); hdr = rows[1]; data = [r for r in rows[2:] if len(r) == len(hdr)]
agg = collections.Counter()
for r in data:
    for i, h in enumerate(hdr):
        if h.startswith("stall_") and "Not Issued" not in h and r[i] not in ("", "-"):
            agg[h[6:]] += float(r[i])
tot = sum(agg.values())
print("stalls:", ", ".join(f"{k}={v/tot:.1%}" for k, v in agg.most_common(10)))
det = subprocess.run(["ncu", "-i", rep, "--page", "details", "--csv"], capture_output=True, text=True).stdout
want = ("Duration", "Issue Slots Busy", "Issued Ipc Active", "Achieved Occupancy", "Registers Per Thread", "Memory Throughput",
        "DRAM Throughput", "L1/TEX Hit Rate", "L2 Hit Rate", "Compute (SM) Throughput", "Block Limit", "Waves Per SM")
for r in csv.reader(det.splitlines()):
    if len(r) > 14 and any(r[-4] == w or r[-4].startswith(w) for w in want):
        print(f"  {r[-4]:40s} {r[-1]:>14s} {r[-2]}")
