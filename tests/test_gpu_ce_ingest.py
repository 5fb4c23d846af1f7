"""The copy-engine ingest (PAGODA_CE_INGEST): the context's host thread copies published
TaskTable entries into the device ring and publishes the ring's tail with a stream memory
operation; MTB 0's scanner warp reports the cells the schedulers handed back.  Semantics must
be those of the doorbell ingest: exactly-once completion, ring reuse only after hand-back,
sessions (start / stop / drain), one-MTB contexts, and bit-exact bodies."""
import numpy as np
import pytest

import oracle
from gpu_util import Dev, ptr
from paper_conf_ppopp_yehsser17_b200 import tasks as T
from paper_conf_ppopp_yehsser17_b200 import workloads as W
from paper_conf_ppopp_yehsser17_b200.pagoda import CE_INGEST, NO_START, Pagoda

pytestmark = pytest.mark.gpu


def test_ce_mark_exactly_once_and_tid():
    dev = Dev()
    n = 300
    cnt = dev.zeros(4)
    out = dev.zeros(n * 256 * 4)
    with Pagoda(flags=CE_INGEST) as p:
        for k in range(n):
            a = T.records(T.MARK, 1)
            a["out"], a["cnt"], a["base"], a["tag"] = ptr(out), ptr(cnt), k * 256, k + 1
            assert p.taskSpawn(200, 1, 0, True, T.MARK, a) == k
        assert p.waitAll() == 0
    o = Dev.get(out, np.uint32).reshape(n, 256)
    assert (o[:, :200] == np.arange(1, n + 1, dtype=np.uint32)[:, None]).all()
    assert Dev.get(cnt, np.uint32)[0] == n * 200


@pytest.mark.parametrize("mtbs,sms", [(2, 0), (4, 0), (1, 1)])
def test_ce_ring_reuse_after_hand_back(mtbs, sms):
    """Many more tasks than ring entries: the copy stream may overwrite a cell only after the
    scanner saw it handed back (tiny ring, one-MTB context too)."""
    kw = {"mtbs_per_sm": mtbs, "ring_entries": 256, "comp_entries": 1024, "flags": CE_INGEST}
    if sms:
        kw.update(num_sms=sms, arena_bytes=64 * 1024)
    elif mtbs == 4:
        kw["arena_bytes"] = 48 * 1024
    with Pagoda(**kw) as p:
        ids = p.spawn_many(30000, 64, 1, 0, False, T.NOP, None, ids=True)
        assert p.waitAll() == 0
        assert ids[-1] == 29999 and all(p.check(int(i)) == 1 for i in ids[::997])


def test_ce_sessions_stop_start_drain():
    with Pagoda(flags=CE_INGEST | NO_START, ring_entries=1024) as p:
        p.spawn_many(1000, 128, 1, 0, False, T.NOP, None)    # spawned while stopped (fits the ring)
        assert p.start_drain() == 0 and p.stop() == 0
        assert p.info().completed_low == 1000
        for s in range(3):
            assert p.start() == 0
            p.spawn_many(5000, 96, 2, 1024, True, T.NOP, None)
            assert p.stop() == 0
        assert p.info().completed_low == 16000


def test_ce_mm_parity_full_size():
    w = W.matmul(65536)
    with Pagoda(mtbs_per_sm=4, arena_bytes=48 * 1024, flags=CE_INGEST) as p:
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0
    C = w.outputs()["C"]
    A, B = w.host["A"], w.host["B"]
    for k in list(range(0, 65536, 509)) + [65535]:
        ref = oracle.mm32(A[k], B[k])
        assert np.array_equal(C[k], ref), k
