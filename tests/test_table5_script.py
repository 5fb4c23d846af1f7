"""scripts/table5.py: Table 5's layout from bench lines — speedups of the
with / without shared-memory runs over the naive baseline of the shared-memory version."""
import json
import subprocess
import sys


def _line(value, naive, shmem):
    return {"value": value, "naive": {"tasks_per_s": naive}, "config": {"task_shmem_bytes": shmem}}


def test_table5_speedups(tmp_path):
    lines = {"dct": _line(27.0, 0.3, 8192), "dct_noshm": _line(18.0, 0.25, 0),
             "mm": _line(45.0, 0.5, 8192), "mm_noshm": _line(50.0, 0.4, 0)}
    for k, v in lines.items():
        (tmp_path / f"bench_{k}.json").write_text(json.dumps(v) + "\n")
    out = subprocess.run([sys.executable, "scripts/table5.py", str(tmp_path)], capture_output=True, text=True,
                         check=True).stdout.strip().splitlines()
    dct, mm = (json.loads(x) for x in out)
    assert dct["body"] == "DCT" and abs(dct["speedup_with"] - 90.0) < 1e-9
    assert abs(dct["speedup_without"] - 60.0) < 1e-9          # over the shmem version's naive run
    assert abs(dct["with_over_without"] - 1.5) < 1e-9
    assert mm["body"] == "MM" and abs(mm["with_over_without"] - 0.9) < 1e-9
    assert dct["task_shmem_bytes"] == [8192, 0]
