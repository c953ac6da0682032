"""Model every loop (backward branch) of every kernel in a cubin: python loops.py file.cubin [-v] [-k substr]"""
import os
import re
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
import rfmodel  # noqa: E402


def main(cubin, verbose=False, ksub=None):
    txt = subprocess.run(["cuobjdump", "-sass", cubin], capture_output=True, text=True).stdout
    for block in txt.split("Function : ")[1:]:
        name = block.split("\n", 1)[0].strip()
        if ksub and ksub not in name:
            continue
        path = "/tmp/_rf_block.sass"
        with open(path, "w") as f:
            f.write(block)
        ins = rfmodel.parse(path)
        for addr, op, args in ins:
            if not op.startswith("BRA"):
                continue
            tgt = None
            for a in args:
                mm = re.search(r"0x([0-9a-f]+)", a)
                if mm:
                    tgt = int(mm.group(1), 16)
            if tgt is not None and tgt < addr and addr - tgt > 0x100:
                region = [i for i in ins if tgt <= i[0] <= addr]
                d, f, a_, rows = rfmodel.model(region)
                b, e = rfmodel.split(rows)
                print(f"{name[:80]:<80} loop {tgt:05x}-{addr:05x}: n={len(region)} base={b} excess={e} "
                      f"est={rfmodel.fitted(b, e):.1f} fma={f} alu={a_}")
                if verbose:
                    for r in rows:
                        print(f"   {r[0]:05x} {r[1]:<26} rt={r[2]} e={r[3]} o={r[4]}")


if __name__ == "__main__":
    k = sys.argv[sys.argv.index("-k") + 1] if "-k" in sys.argv else None
    main(sys.argv[1], "-v" in sys.argv, k)
