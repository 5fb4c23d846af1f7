"""The full-size parity tests and bench.py share one set of context presets
(paper_conf_ppopp_yehsser17_b200/presets.py): the launch configuration the
bench times is the one the parity tests check."""
import bench
from paper_conf_ppopp_yehsser17_b200 import pagoda as PG
from paper_conf_ppopp_yehsser17_b200 import presets


def test_bench_uses_package_presets():
    assert bench.PRESETS is presets.PRESETS
    assert set(presets.PRESETS) == set(bench.WORKLOADS)


def test_ctx_kwargs_match_bench_context():
    assert presets.RESIDENT_TDES == PG.RESIDENT_TDES and presets.SPREAD == PG.SPREAD
    assert presets.CE_INGEST == PG.CE_INGEST
    for w in bench.WORKLOADS:
        class A:
            workload = w
            no_resident = False
            mtbs = 0
            arena_kb = 0
            exec_warps = 0
            spread = -1
            groups = 0
        cfg = bench.ctx_config(A, PG, w)
        kw = presets.ctx_kwargs(w, PG.NO_START)
        assert cfg == kw, w


def test_every_workload_has_its_bench_tables():
    """Each bench workload names its dtype, config, oracle sample sizes, and the
    arena of its preset holds at least one task of its largest shmem request."""
    for w in bench.WORKLOADS:
        assert w in bench.DTYPE and w in bench.REF_SAMPLE and w in bench.CPU_SAMPLE, w
        cfg = bench.workload_config(w)
        assert cfg["workload"] and cfg["n_tasks"] > 0, w
        if "shmem_bytes" in cfg:
            assert presets.PRESETS[w]["arena_bytes"] >= cfg["shmem_bytes"], w


def test_oracle_sample_for_new_workloads():
    """The cpu_baseline leg builds oracle calls for the Table 4/5 workloads (a few run here)."""
    for w in ("dct", "dct_noshm", "mm_noshm", "mm64"):
        calls, what = bench.oracle_tasks(w, 2)
        assert len(calls) == 2 and what
        outs = [c() for c in calls]
        assert outs[0].shape == ((64, 64) if w == "mm64" else (128, 128) if w.startswith("dct") else (32, 32))
