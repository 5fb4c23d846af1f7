"""Per-workload MasterKernel context presets: the launch configuration bench.py
times for each BASELINE.json workload, shared with the
full-size parity tests so that they run in exactly that configuration."""

# mtbs_per_sm / arena_bytes: pagoda_config; resident: PAGODA_RESIDENT_TDES (+ registered round
# keys in bench.py); spread: PAGODA_SPREAD; producers: host spawner threads per step
PRESETS = {
    # 3DES tasks hold 512 B: an 8 KiB arena (not 40) lets the L1 carveout keep the executors' register spills
    # (34.4 vs 33.7 M tasks/s)
    "tdes": {"mtbs_per_sm": 2, "arena_bytes": 8 * 1024, "resident": True},
    # MB: 1 MTB/SM (64 registers), at most 2 tasks held per MTB: the rest wait in the ring for whichever MTB
    # frees first, so the saturated tiles spread by completion (4.75 M vs 4.27 M with spread-first claims)
    "mb": {"mtbs_per_sm": 1, "arena_bytes": 96 * 1024, "resident": False, "max_tasks": 2},
    # MM: 512-thread MTBs (2x schedulers), the copy-engine ingest (no staging shared memory in MTB 0) and a 24 KiB
    # arena (2 tasks x 8 KiB): shared memory per SM drops from 227 to ~130 KiB and L1 serves the 32-register
    # spills (47 % -> most hits); 3 host producers.  48.3 -> 53-54 M tasks/s (62 M self-draining)
    "mm": {"mtbs_per_sm": 4, "arena_bytes": 24 * 1024, "resident": False, "ce": True, "producers": 3},
    "mix": {"mtbs_per_sm": 1, "arena_bytes": 200 * 1024, "resident": False, "producers": 2},
    "nop": {"mtbs_per_sm": 2, "arena_bytes": 16 * 1024, "resident": False, "producers": 2, "ce": True},   # 68 -> 92 M
    # C5: 1M mixed shapes; 8 producer threads validate and spawn in parallel (16.0 -> 17.0 M tasks/s vs 1)
    "c5": {"mtbs_per_sm": 1, "arena_bytes": 144 * 1024, "resident": True, "producers": 8},
    "mpe": {"mtbs_per_sm": 2, "arena_bytes": 40 * 1024, "resident": True},
    "tdes_var": {"mtbs_per_sm": 2, "arena_bytes": 40 * 1024, "resident": True},
    "mm_tc": {"mtbs_per_sm": 4, "arena_bytes": 24 * 1024, "resident": False, "ce": True, "producers": 2},   # 45 -> 52 M
    "mm64": {"mtbs_per_sm": 2, "arena_bytes": 96 * 1024, "resident": False},        # 3 tasks x 32 KiB per MTB
    "mm_noshm": {"mtbs_per_sm": 4, "arena_bytes": 8 * 1024, "resident": False, "ce": True,   # Table 5 ablation:
                 "producers": 3},                                                          # MM's runtime settings
    "dct": {"mtbs_per_sm": 2, "arena_bytes": 96 * 1024, "resident": False},         # 8 KiB grants (sweep: 4/8/16/32 KiB)
    "dct_noshm": {"mtbs_per_sm": 2, "arena_bytes": 96 * 1024, "resident": False},
}

RESIDENT_TDES = 0x4   # include/pagoda.h
SPREAD = 0x10
CE_INGEST = 0x40


def ctx_kwargs(workload: str, flags: int = 0) -> dict:
    """pagoda_config keyword arguments (Pagoda(**...)) of the workload's preset."""
    pr = PRESETS[workload]
    f = flags | (RESIDENT_TDES if pr["resident"] else 0) | (SPREAD if pr.get("spread") else 0) | \
        (CE_INGEST if pr.get("ce") else 0)
    kw = {"flags": f, "mtbs_per_sm": pr["mtbs_per_sm"], "arena_bytes": pr["arena_bytes"]}
    if pr.get("exec_warps"):
        kw["exec_warps"] = pr["exec_warps"]
    if pr.get("sched_groups"):
        kw["sched_groups"] = pr["sched_groups"]
    if pr.get("max_tasks"):
        kw["max_tasks"] = pr["max_tasks"]
    return kw
