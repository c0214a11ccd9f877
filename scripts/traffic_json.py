"""profiles/traffic.json from the round's ncu --set full raw exports
(scripts/prof_round.sh): dram__bytes_read.sum + dram__bytes_write.sum per launch,
keyed like bench.cfg_key(spec, candidate)."""
import csv
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
TAGS = {  # capture tag -> (spec name, bench candidate tuple)
    "cfg2_S2bq": ("cfg2", [2, "spmd", 1, 1024, 0, "bq"]),
    "cfg2_S2bv": ("cfg2", [2, "spmd", 1, 1024, 0, "bv"]),
    "cfg2_S1bv": ("cfg2", [1, "spmd", 1, 1024, 0, "bv"]),
    "g100_S2bq": ("g100", [2, "spmd", 1, 1024, 0, "bq"]),
    "g100_S2bv": ("g100", [2, "spmd", 1, 1024, 0, "bv"]),
    "g100_S1bv": ("g100", [1, "spmd", 1, 1024, 0, "bv"]),
    "cfg5_S8bv": ("cfg5", [8, "spmd", 1, 1024, 0, "bv"]),
    "cfg5_S1bv": ("cfg5", [1, "spmd", 1, 1024, 0, "bv"]),
    "cfg2_S2bqp": ("cfg2", [2, "spmd", 1, 1024, 0, "bqp"]),
    "cfg2_S1bqp": ("cfg2", [1, "spmd", 1, 1024, 0, "bqp"]),
    "g100_S2bqp": ("g100", [2, "spmd", 1, 1024, 0, "bqp"]),
    "g100_S1bqp": ("g100", [1, "spmd", 1, 1024, 0, "bqp"]),
}


def dram_bytes(path):
    rows = list(csv.reader(open(path)))
    h, u, v = rows[0], rows[1], rows[2]
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    tot = 0.0
    for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
        i = h.index(m)
        tot += float(v[i].replace(",", "")) * scale[u[i]]
    return tot


def main(src):
    path = os.path.join(ROOT, "profiles", "traffic.json")
    out = json.load(open(path)) if os.path.exists(path) else {}   # keys not re-captured are kept
    out["_note"] = ("dram__bytes_read.sum + dram__bytes_write.sum per launch, one ncu --set full capture "
                    "(--clock-control none, cold L2) per key; key = '<spec>:<bench candidate tuple>'; "
                    f"latest source {src}")
    for tag, (spec, c) in TAGS.items():
        p = os.path.join(src, f"{tag}_raw.csv")
        if os.path.exists(p):
            out[f"{spec}:{json.dumps(c)}"] = dram_bytes(p)
    with open(path, "w") as f:
        json.dump(out, f, indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/prof")
