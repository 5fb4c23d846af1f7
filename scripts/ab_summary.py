"""Summarise scripts/var_ab.sh outputs: tasks/s per (workload, variant) and the probe ceilings."""
import glob
import json
import os
import re
import sys

d = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out"
rows = {}
for f in sorted(glob.glob(os.path.join(d, "*_*_*.json"))):
    m = re.match(r"(?:ab_)?(\w+?)_(\w+)_(\d+)\.json", os.path.basename(f))
    if not m:
        continue
    try:
        v = json.loads(open(f).read().strip().splitlines()[-1])["value"]
    except Exception:
        v = None
    rows.setdefault(m.group(1), {}).setdefault(m.group(2), []).append(v)
for w, vs in rows.items():
    print(w, {k: [round(x / 1e6, 2) if x else x for x in xs] for k, xs in vs.items()})
for f in sorted(glob.glob(os.path.join(d, "*t*.txt"))):
    print(os.path.basename(f), open(f).read().strip())
for f in sorted(glob.glob(os.path.join(d, "ab_probe_*.json"))):
    try:
        j = json.loads(open(f).read().strip().splitlines()[-1])
        print(os.path.basename(f), {k: {kk: round(vv / 1e6, 1) for kk, vv in x.items() if kk.endswith("per_s")}
                                    for k, x in j.items() if isinstance(x, dict)})
    except Exception as e:
        print(f, "unparsed", e)
