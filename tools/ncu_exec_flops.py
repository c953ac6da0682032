"""Executed FP32 flops of the kernel in an ncu --set full report, from the source page's predicated-on
thread instruction counts (FFMA2 x4, FMUL2/FADD2/FFMA x2, FMUL/FADD x1), and its DRAM bytes.
    python tools/ncu_exec_flops.py report.ncu-rep  ->  one JSON line"""
import csv
import io
import json
import re
import subprocess
import sys

rep = sys.argv[1]


def page(*a):
    return subprocess.run(["ncu", "-i", rep] + list(a), capture_output=True, text=True).stdout


src = list(csv.reader(io.StringIO(page("--page", "source", "--csv", "--print-source", "sass"))))
hdr = src[1]
ix = {h: i for i, h in enumerate(hdr)}
w = {"FFMA2": 4, "FMUL2": 2, "FADD2": 2, "FFMA": 2, "FMUL": 1, "FADD": 1}
tot = 0
for r in src[2:]:
    if len(r) != len(hdr):
        continue
    op = re.sub(r"^@!?U?P\d+\s+", "", r[ix["Source"]].strip()).split(" ")[0].split(".")[0]
    if op in w:
        tot += int(r[ix["Predicated-On Thread Instructions Executed"]] or 0) * w[op]
raw = list(csv.reader(io.StringIO(page("--page", "raw", "--csv", "--print-units", "base"))))
d = dict(zip(raw[0], raw[2]))
t = float(d["gpu__time_duration.sum"]) * 1e-9
out = {"kernel": d.get("Kernel Name", "")[:80], "time_ms": t * 1e3, "executed_fp32_gflop": tot / 1e9,
       "executed_tflops": tot / t / 1e12,
       "fma_pipe_active_pct": float(d["sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active"]),
       "dram_bytes": int(float(d["dram__bytes_read.sum"]) + float(d["dram__bytes_write.sum"]))}
print(json.dumps(out))
