"""Summarise the parity reports the -m gpu tests wrote to gpurun_out/parity/*.json into one table:
    python tools/parity_summary.py [gpurun_out/parity] > profiles/r2/parity_summary.md"""
import glob
import json
import os
import sys

d = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/parity"
rows = []
for f in sorted(glob.glob(os.path.join(d, "*.json"))):
    r = json.load(open(f))
    rows.append((os.path.basename(f)[:-5], r))
cols = ["lanes", "flag_mismatch", "flag_boundary", "flag_sensitive", "flag_unexplained", "lam_violations",
        "lam_boundary", "lam_unexplained", "lam_max_rel", "angle_violations", "angle_unexplained", "angle_max_aligned",
        "sensitive_lanes", "sensitive_frac", "max_sensitive", "max_rel", "outliers", "unexplained", "angle_max",
        "representatives"]
used = [c for c in cols if any(c in r for _, r in rows)]
print("# Parity reports of the -m gpu tests (tests/parity.py; DESIGN.md 5)\n")
print(f"{len(rows)} reports from `{d}`.  Explained lanes are counted per rule; every `*unexplained` column must be 0.\n")
print("| test | " + " | ".join(used) + " |")
print("|---|" + "---|" * len(used))


def fmt(v):
    if isinstance(v, float):
        return f"{v:.3g}"
    return "" if v is None else str(v)


for name, r in rows:
    print(f"| {name} | " + " | ".join(fmt(r.get(c)) for c in used) + " |")
tot = {c: sum(r.get(c, 0) or 0 for _, r in rows) for c in ("lanes", "flag_unexplained", "lam_unexplained",
                                                            "angle_unexplained", "unexplained", "sensitive_lanes")}
print(f"\nTotals: {tot}")
