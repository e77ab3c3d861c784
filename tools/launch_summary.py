"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list: total time per kernel name."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = None
tot = collections.defaultdict(float); cnt = collections.Counter()
for r in rows:
    if r and r[0] == "ID": hdr = r; continue
    if hdr is None or len(r) != len(hdr): continue
    d = dict(zip(hdr, r))
    if d.get("Metric Name") != "gpu__time_duration.sum": continue
    name = d["Kernel Name"].split("(")[0]
    v = float(d["Metric Value"].replace(",", ""))
    unit = d.get("Metric Unit", "nsecond")
    v = v / 1e3 if unit in ("ns", "nsecond") else (v if unit in ("us", "usecond") else v * 1e3)
    tot[name] += v; cnt[name] += 1
T = sum(tot.values())
print(f"total {T/1e3:.2f} ms over {sum(cnt.values())} launches")
for k, v in sorted(tot.items(), key=lambda x: -x[1]):
    print(f"{v/1e3:9.2f} ms {100*v/T:5.1f}%  n={cnt[k]:6d}  avg {v/cnt[k]:8.1f} us  {k}")
