"""Markdown table from scripts/mode_study.sh's ncu CSV (every second launch is the profiled one)."""
import collections
import csv
import re
import sys

lines = open(sys.argv[1]).read().splitlines()
runs = [l.split("RUN ", 1)[1] for l in lines if l.startswith("RUN ")]
rows = [r for r in csv.reader([l for l in lines if l.startswith('"')]) if len(r) > 10]
h, rows = rows[0], rows[1:]
iid, im, iv, iu = h.index("ID"), h.index("Metric Name"), h.index("Metric Value"), h.index("Metric Unit")
SCALE = {"ns": 1, "nsecond": 1, "us": 1e3, "usecond": 1e3, "ms": 1e6, "msecond": 1e6,
         "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
d = collections.OrderedDict()
for r in rows:   # durations -> ns, sizes -> bytes; per-opcode instances -> {opcode: count}
    v = r[iv]
    if "(" in v:
        ops = dict((k.strip(), float(c)) for k, c in (e.split(":") for e in v[v.index("(") + 1:-1].split(";")))
        d.setdefault(int(r[iid]), {})[r[im] + ":ops"] = ops
        v = v[:v.index("(")]
    d.setdefault(int(r[iid]), {})[r[im]] = float(v.replace(",", "")) * SCALE.get(r[iu], 1)
ids = sorted(d)[1::2]   # warm launch, then the profiled launch
print("| run | time us | DRAM GB | inst (M) | SHFL (M) | BAR/WARPSYNC (M) | warp exec eff | divergent branch % | LDS (M) | STS (M) | issue % | long-sb stall/issue |")
print("|---|---:|---:|---:|---:|---:|---:|---:|---:|---:|---:|---:|")
for name, i in zip(runs, ids):
    m = d[i]
    div = 100 * m["smsp__sass_branch_targets_threads_divergent.sum"] / max(1, m["smsp__sass_branch_targets.sum"])
    print(f"| {name} | {m['gpu__time_duration.sum'] / 1e3:.1f} | "
          f"{(m['dram__bytes_read.sum'] + m['dram__bytes_write.sum']) / 1e9:.3f} | "
          f"{m['smsp__inst_executed.sum'] / 1e6:.1f} | "
          f"{m.get('sass__inst_executed_per_opcode:ops', {}).get('SHFL', 0) / 1e6:.2f} | "
          f"{sum(c for k, c in m.get('sass__inst_executed_per_opcode:ops', {}).items() if k in ('WARPSYNC', 'BAR', 'NANOSLEEP')) / 1e6:.2f} | "
          f"{m['smsp__thread_inst_executed_per_inst_executed.ratio'] / 32:.2f} | {div:.1f} | "
          f"{m['sm__sass_inst_executed_op_shared_ld.sum'] / 1e6:.2f} | {m['sm__sass_inst_executed_op_shared_st.sum'] / 1e6:.2f} | "
          f"{m['smsp__issue_active.avg.pct_of_peak_sustained_active']:.1f} | "
          f"{m['smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio']:.1f} |")
