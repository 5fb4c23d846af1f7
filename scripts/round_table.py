#!/usr/bin/env python
"""Markdown results table from a default bench line (`python bench.py` JSON):
the headline (config 2) and the configs under "configs".

    python scripts/round_table.py profiles/r2_bench_default.json
"""
import json
import sys


def row(name, r):
    rf = r["roofline"]
    tr = rf.get("traffic") or {}
    dram = ""
    if tr.get("dram_bytes_per_launch") and tr.get("algorithmic_hbm_bytes"):
        dram = f" (DRAM {tr['dram_bytes_per_launch'] / tr['algorithmic_hbm_bytes']:.2f}x algorithmic)"
    fus = r.get("static_fusion", {}).get("tasks_per_s")
    nai = r.get("naive", {}).get("tasks_per_s")
    host = r.get("host_tasks_per_s")
    e2e = r.get("e2e", {}).get("value")
    return (f"| {name} | **{r['value'] / 1e6:.2f} M** | {r['ms_per_step']:.3f} | {rf['resource']}, {rf['frac']:.3f}{dram} | "
            f"{host / 1e6:.2f} M | {host / nai:.0f}x | {host / fus:.2f}x | "
            f"{r.get('p50_spawn_to_done_us', float('nan')):.1f} | {e2e / 1e6:.2f} M |" if e2e else
            f"| {name} | **{r['value'] / 1e6:.2f} M** | {r['ms_per_step']:.3f} | {rf['resource']}, {rf['frac']:.3f}{dram} | "
            f"{host / 1e6:.2f} M | {host / nai:.0f}x | {host / fus:.2f}x | "
            f"{r.get('p50_spawn_to_done_us', float('nan')):.1f} | — |")


def main(path):
    d = json.loads(open(path).read().strip().splitlines()[-1])
    print("| Config | tasks/s (device) | ms/step | roofline (resource, frac) | tasks/s (host clock) | vs naive | "
          "vs static fusion | p50 loaded µs | e2e (H2D + D2H in the step) |")
    print("|---|---|---|---|---|---|---|---|---|")
    print(row("C2 3DES 32768×128 (headline)", d))
    names = {"C1": "C1 MB 1024×128", "C3": "C3 MM 65536×256", "C4": "C4 FB/BF/CONV/DCT mix 32768",
             "C5": "C5 1M mixed (1 GPU)"}
    for k, r in d.get("configs", {}).items():
        print(row(names.get(k, k), r))
    lat = d.get("latency", {})
    if lat:
        print(f"\nIsolated NOP spawn→done p50 {lat['isolated_nop128_us']['p50']:.1f} µs against the PCIe ping-pong floor "
              f"{lat['pingpong_floor_us']['p50']:.2f} µs ({lat['isolated_nop128_over_floor']:.2f}×); "
              f"SM clock {d['clocks']['sm_mhz']:.0f} MHz, throttle reasons {d['clocks']['reasons'] or 'none'}; "
              f"CPU oracle {d['cpu_baseline']['value']:.0f} tasks/s on {d['cpu_baseline']['cores']} threads "
              f"({d['cpu_baseline']['single_thread']['value']:.0f} on one).")


if __name__ == "__main__":
    main(sys.argv[1])
