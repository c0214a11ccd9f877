"""Average each metric per kernel over the launches of an `ncu --csv` metrics log
(developer tool): python scripts/ncu_csv_avg.py gpurun_out/x.csv"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
start = next(i for i, r in enumerate(rows) if r and r[0] == "ID")
hdr = rows[start]
ki, mi, vi = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
d = collections.OrderedDict()
for r in rows[start + 1:]:
    if len(r) < len(hdr):
        continue
    d.setdefault(r[ki], collections.OrderedDict()).setdefault(r[mi], []).append(float(r[vi].replace(",", "")))
for k, m in d.items():
    print(k.split("(")[0][:70])
    print("    " + "  ".join(f"{mm.split('.')[0].replace('__', ':')}={sum(v) / len(v):.4g}" for mm, v in m.items()))
