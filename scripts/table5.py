"""Table 5 on B200 from bench lines: Pagoda with and without shared
memory, each as a speedup over the naive one-launch-per-task baseline (the CUDA-HyperQ
stand-in) of the version that uses shared memory, as the paper compares.

    python scripts/table5.py DIR   # DIR holds bench_{dct,dct_noshm,mm,mm_noshm}.json
"""
import json
import os
import sys


def line(d, w):
    with open(os.path.join(d, f"bench_{w}.json")) as f:
        return json.loads(f.read().strip().splitlines()[-1])


def main():
    d = sys.argv[1] if len(sys.argv) > 1 else "gpurun_out/final"
    rows = []
    for body, shm, noshm in (("DCT", "dct", "dct_noshm"), ("MM", "mm", "mm_noshm")):
        a, b = line(d, shm), line(d, noshm)
        ref = a["naive"]["tasks_per_s"]
        rows.append({"body": body, "with_shmem_tasks_per_s": a["value"], "without_shmem_tasks_per_s": b["value"],
                     "naive_with_shmem_tasks_per_s": ref, "speedup_with": a["value"] / ref,
                     "speedup_without": b["value"] / ref, "with_over_without": a["value"] / b["value"],
                     "task_shmem_bytes": [a["config"]["task_shmem_bytes"], b["config"]["task_shmem_bytes"]],
                     "paper": {"DCT": "1.35x with (25% occupancy), 1.25x without (97%)",
                               "MM": "1.51x with (97%), 1.20x without (97%)"}[body]})
    for r in rows:
        print(json.dumps(r))


if __name__ == "__main__":
    main()
