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
    for w in bench.WORKLOADS:
        class A:
            workload = w
            no_resident = False
            mtbs = 0
            arena_kb = 0
        cfg = bench.ctx_config(A, PG)
        kw = presets.ctx_kwargs(w, PG.NO_START)
        assert cfg == kw, w
