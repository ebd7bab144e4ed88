"""Summarise an ncu --metrics gpu__time_duration.sum CSV launch list per kernel."""
import csv, collections, sys
for path in sys.argv[1:]:
    hdr = None; data = []
    for r in csv.reader(open(path)):
        if r and r[0] == "ID": hdr = r; continue
        if hdr and len(r) == len(hdr): data.append(dict(zip(hdr, r)))
    agg = collections.defaultdict(list)
    for d in data:
        agg[(d["Kernel Name"][:48], d["Grid Size"])].append(float(d["Metric Value"]))
    print(path)
    for (k, g), v in agg.items():
        print(f"  {k:48s} grid={g:14s} n={len(v):4d} mean={sum(v)/len(v)/1e3:9.2f}us min={min(v)/1e3:8.2f}us")
