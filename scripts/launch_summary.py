"""Summarise an ncu launch list (--metrics gpu__time_duration.sum --csv) per kernel name:
launches, total time, share, average.  python scripts/launch_summary.py launches.csv"""
import collections
import csv
import sys

rows = [r for r in csv.reader(open(sys.argv[1])) if len(r) > 10]
h, rows = rows[0], rows[1:]
ik, iv, iu = h.index("Kernel Name"), h.index("Metric Value"), h.index("Metric Unit")
tot = collections.defaultdict(float)
cnt = collections.Counter()
for r in rows:
    v = float(r[iv].replace(",", ""))
    v = v / 1e3 if r[iu] == "ns" else v * 1e3 if r[iu] == "ms" else v   # -> us
    tot[r[ik]] += v
    cnt[r[ik]] += 1
allt = sum(tot.values())
print(f"launches {sum(cnt.values())}, total {allt:.1f} us (cold-cache, serialised under ncu)")
for k, v in sorted(tot.items(), key=lambda t: -t[1]):
    print(f"{cnt[k]:5d} {v:12.1f} us {100 * v / allt:5.1f}%  avg {v / cnt[k]:8.2f} us  {k[:120]}")
