"""Per-stall-reason totals and the top stalled SASS lines of one kernel from an ncu report's source page:
    ncu -i rep.ncu-rep --page source --csv --print-source sass > src.csv; python tools/ncu_stalls.py src.csv"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr = rows[1]
reasons = [h for h in hdr if h.startswith("stall_") and "Not Issued" not in h]
ix = {h: i for i, h in enumerate(hdr)}
tot = {r: 0 for r in reasons}
lines = []
for r in rows[2:]:
    if len(r) < len(hdr):
        continue
    vals = {k: int(float(r[ix[k]] or 0)) for k in reasons}
    for k in reasons:
        tot[k] += vals[k]
    lines.append((sum(vals.values()), r[ix["Source"]].strip(), vals, r[ix["Instructions Executed"]]))
allv = sum(tot.values()) or 1
print("stall share:", ", ".join(f"{k[6:]} {100 * v / allv:.1f}%" for k, v in sorted(tot.items(), key=lambda t: -t[1]) if v))
for s, src, vals, ex in sorted(lines, key=lambda t: -t[0])[:int(sys.argv[2]) if len(sys.argv) > 2 else 20]:
    top = sorted(vals.items(), key=lambda t: -t[1])[:3]
    print(f"{s:7d} {src[:64]:<64} exec={ex} " + " ".join(f"{k[6:]}={v}" for k, v in top if v))
