"""Top SASS instructions by warp-stall samples from `ncu --page source --csv --print-source sass`,
with the stall-reason columns that dominate each.  Usage: ncu_hot.py report.ncu-rep [N]"""
import csv, subprocess, sys
rep = sys.argv[1]; N = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines()))
hdr = rows[1]; data = [r for r in rows[2:] if len(r) == len(hdr)]
si = hdr.index("Warp Stall Sampling (All Samples)")
stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") or "Stall" in h and i != si and "Not-issued" not in h]
tot = sum(float(r[si] or 0) for r in data)
print("total samples", tot, "instructions", len(data))
idx = sorted(range(len(data)), key=lambda i: -float(data[i][si] or 0))[:N]
for i in sorted(idx):
    r = data[i]
    reasons = sorted(((float(r[c] or 0), hdr[c]) for c in stall_cols if r[c] not in ("", "0")), reverse=True)[:3]
    print(f"{i:5d} {float(r[si])/tot:6.1%} {r[1].strip()[:60]:60s} " + " ".join(f"{h.replace('stall_','')}={v:.0f}" for v, h in reasons))
