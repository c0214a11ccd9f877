"""Per-opcode attribution of an ncu source page (--page source --csv --print-source
sass): instructions executed, L1 tag requests (global) and L2 theoretical sectors
per load/store/shuffle class.  python scripts/sass_attrib.py <file.csv> ..."""
import csv
import sys


def attrib(path):
    rows = list(csv.reader(open(path)))
    start = 1 if rows[0][0] == "Kernel Name" else 0
    h, data = rows[start], rows[start + 1:]
    iS, iE = h.index("Source"), h.index("Instructions Executed")
    iT, iL2 = h.index("L1 Tag Requests Global"), h.index("L2 Theoretical Sectors Global")
    iTh = h.index("Thread Instructions Executed")
    tot = {}
    for r in data:
        if len(r) <= iL2:
            continue
        s = r[iS].strip()
        op = s.split()[1] if s.startswith("@") else s.split()[0]
        key = None
        if op.startswith("LDG"):
            key = ("LDG.256" if ".256" in op else "LDG.128" if ".128" in op else "LDG.64" if ".64" in op
                   else "LDG.32")
        elif op.startswith("SHFL"):
            key = "SHFL"
        elif op.startswith("STG"):
            key = "STG"
        elif op.startswith(("LDS", "STS", "LD.", "ST.")):
            key = op.split(".")[0]
        if key:
            t = tot.setdefault(key, [0, 0, 0.0, 0.0])
            t[0] += int(r[iE] or 0)
            t[1] += int(r[iTh] or 0)
            t[2] += float(r[iT] or 0)
            t[3] += float(r[iL2] or 0)
    return tot


for p in sys.argv[1:]:
    print("==", p)
    print(f"   {'class':8s} {'warp inst':>12s} {'thread inst':>13s} {'L1 tag req':>12s} {'L2 sectors':>12s}")
    for k, v in sorted(attrib(p).items()):
        print(f"   {k:8s} {v[0]:>12d} {v[1]:>13d} {v[2]:>12.0f} {v[3]:>12.0f}")
