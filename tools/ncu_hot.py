"""Top SASS instructions by warp-stall samples from an ncu report (source page, sass view)."""
import csv, subprocess, sys
rep = sys.argv[1]; top = int(sys.argv[2]) if len(sys.argv) > 2 else 30
kern = sys.argv[3] if len(sys.argv) > 3 else None
cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"]
if kern: cmd += ["-k", kern]
out = subprocess.run(cmd, capture_output=True, text=True).stdout.splitlines()
rows = list(csv.reader(out))
hdr = None; data = []
for r in rows:
    if len(r) > 3 and r[0] == "Address": hdr = r; continue
    if hdr and len(r) == len(hdr): data.append(r)
si = hdr.index("Warp Stall Sampling (All Samples)")
tot = sum(float(r[si] or 0) for r in data)
print("total samples", tot, "instructions", len(data))
idx = sorted(range(len(data)), key=lambda i: -float(data[i][si] or 0))
for i in idx[:top]:
    r = data[i]
    print(f"{100*float(r[si] or 0)/tot:5.1f}%  {i:5d} {r[0][-5:]} {r[1].strip()[:90]}")
