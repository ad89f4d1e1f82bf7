"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel."""
import csv, sys, collections
rows = list(csv.reader(open(sys.argv[1])))
hdr = None
agg = collections.OrderedDict()
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if not hdr or len(r) != len(hdr):
        continue
    d = dict(zip(hdr, r))
    if d.get("Metric Name") != "gpu__time_duration.sum":
        continue
    name = d["Kernel Name"].split("(")[0]
    v = float(d["Metric Value"].replace(",", ""))
    unit = d.get("Metric Unit", "")
    us = v / 1000.0 if unit in ("nsecond", "ns") else v if unit in ("usecond", "us") else v * 1000 if unit == "msecond" else v
    a = agg.setdefault(name, [0, 0.0])
    a[0] += 1
    a[1] += us
tot = sum(x[1] for x in agg.values())
print(f"{'kernel':60s} {'launches':>8s} {'total_us':>10s} {'share':>6s}")
for k, (n, us) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
    print(f"{k[:60]:60s} {n:8d} {us:10.1f} {100*us/tot:5.1f}%")
print(f"{'TOTAL':60s} {sum(x[0] for x in agg.values()):8d} {tot:10.1f}")
