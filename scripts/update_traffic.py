"""profiles/ncu_traffic.json <- dram__bytes_read.sum + dram__bytes_write.sum of the
ncu --set full summaries (scripts/ncu_summary.py output), per workload.

    python scripts/update_traffic.py tdes=profiles/r1_ncu_tdes_full.txt mm=profiles/r1_ncu_mm_full.txt
"""
import json
import os
import sys

UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def parse(path):
    vals = {}
    for line in open(path):
        parts = line.split()
        if len(parts) >= 2:
            try:
                vals[parts[0]] = (float(parts[1].replace(",", "")), parts[2] if len(parts) > 2 else "")
            except ValueError:   # opmix lines
                pass
    b = sum(v * UNIT.get(u, 1) for k, (v, u) in vals.items() if k in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    return b, vals.get("gpu__time_duration.sum")


def main():
    out_path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_traffic.json")
    out = json.load(open(out_path)) if os.path.exists(out_path) else {}
    for arg in sys.argv[1:]:
        name, path = arg.split("=", 1)
        b, dur = parse(path)
        out[name] = {"dram_bytes_per_launch": b, "ncu_duration": dur,
                     "source": f"{path} (ncu --set full, one self-draining launch)"}
    json.dump(out, open(out_path, "w"), indent=1)


if __name__ == "__main__":
    main()
