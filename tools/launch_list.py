"""Format an `ncu --metrics gpu__time_duration.sum --csv` launch list: one line per launch and
each sshopm kernel's share of the sshopm kernel time.  Usage: launch_list.py launches.csv [header]"""
import csv
import sys
from collections import OrderedDict

rows = list(csv.reader(open(sys.argv[1])))
hdr = None
launches = []
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get("Metric Name") == "gpu__time_duration.sum":
            ns = float(d["Metric Value"].replace(",", ""))
            if d.get("Metric Unit") == "usecond":
                ns *= 1e3
            elif d.get("Metric Unit") == "msecond":
                ns *= 1e6
            launches.append((d["Kernel Name"], ns))
if len(sys.argv) > 2:
    print(sys.argv[2])
print("# per-launch device time (cold-cache, serialised); compare shares, not absolutes")
for name, ns in launches:
    print(f"{ns:12.0f} ns  {name}")
share = OrderedDict()
for name, ns in launches:
    if "sshopm" in name:
        key = name.split("(")[0]
        share[key] = share.get(key, 0.0) + ns
tot = sum(share.values()) or 1.0
print("# shares of sshopm kernel time:")
for k, v in share.items():
    print(f"#   {k:60s} {100 * v / tot:5.1f}%")
