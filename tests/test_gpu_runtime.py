"""Runtime semantics on the GPU through the C-ABI (Table 1):
spawn/wait/check/waitAll contract, exactly-once completion, getTid, syncBlock,
getSMPtr, liveness, validation, multiple producers, and the scheduler ledger
replayed by the oracle-side checker."""
import errno
import threading
import time

import numpy as np
import pytest

from gpu_util import Dev, ptr
from paper_conf_ppopp_yehsser17_b200 import tasks as T
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, Pagoda, TRACE

pytestmark = pytest.mark.gpu


def test_init_info_shutdown():
    with Pagoda() as p:
        i = p.info()
        assert i.sm_count == 148 and i.n_mtb == 296 and i.running == 1
        assert i.regs_per_thread <= 32
        assert p.waitAll() == 0
    # 1 MTB per SM variant (64 registers per thread)
    with Pagoda(mtbs_per_sm=1, arena_bytes=200 * 1024) as p:
        assert p.info().n_mtb == 148
        ids = p.spawn_many(1000, 128, 1, 0, False, T.NOP, None, ids=True)
        assert p.waitAll() == 0 and all(p.check(int(i)) == 1 for i in ids[::97])


def test_nop_many_shapes_exactly_once():
    shapes = [(32, 1, 0, 0), (128, 1, 0, 0), (256, 1, 8192, 1), (100, 3, 600, 1), (992, 1, 0, 1), (64, 15, 0, 1),
              (32, 31, 512, 1), (1024, 1, 0, 1), (32, 32, 0, 0)]
    with Pagoda() as p:
        ids = []
        for k in range(3000):
            th, nb, sh, sy = shapes[k % len(shapes)]
            ids.append(p.taskSpawn(th, nb, sh, sy, T.NOP))
        assert ids == list(range(3000))
        assert p.waitAll() == 0
        assert all(p.check(i) == 1 for i in ids)
        assert p.wait(1234) == 0
        assert p.info().completed_low == 3000


def test_lone_task_liveness():
    """A single task with nothing spawned after it must still run (the paper
    needs a last-task flush for this)."""
    with Pagoda() as p:
        time.sleep(0.05)
        t0 = time.perf_counter()
        tid = p.taskSpawn(128, 1, 0, False, T.NOP)
        assert p.wait(tid) == 0
        assert time.perf_counter() - t0 < 0.5


def test_mark_counts_and_tid_bijection():
    n = 400
    shapes = [(32, 1), (96, 2), (128, 1), (100, 3), (256, 1), (40, 7), (512, 1), (992, 1)]
    dev = Dev()
    cap = 992 * n
    out = dev.zeros(cap * 4)
    cnt = dev.zeros(n * 4)
    tids = dev.zeros(cap * 4)
    base = np.zeros(n, np.int64)
    b = 0
    for k in range(n):
        th, nb = shapes[k % len(shapes)]
        base[k] = b
        b += ((th + 31) // 32) * 32 * nb
    assert b <= cap
    with Pagoda() as p:
        for k in range(n):
            th, nb = shapes[k % len(shapes)]
            a = T.records(T.MARK, 1)
            a["out"], a["cnt"], a["base"], a["tag"] = ptr(out), ptr(cnt) + 4 * k, base[k], k + 1
            assert p.taskSpawn(th, nb, 0, False, T.MARK, a) == 2 * k
            t = T.records(T.TID, 1)
            t["out"], t["base"] = ptr(tids), base[k]
            assert p.taskSpawn(th, nb, 0, False, T.TID, t) == 2 * k + 1
        assert p.waitAll() == 0
    o = Dev.get(out, np.uint32)
    c = Dev.get(cnt, np.uint32)
    tv = Dev.get(tids, np.uint32)
    for k in range(n):
        th, nb = shapes[k % len(shapes)]
        w = (th + 31) // 32
        assert c[k] == th * nb                     # every live thread ran exactly once
        seg = o[base[k]: base[k] + 32 * w * nb].reshape(nb, 32 * w)
        assert (seg[:, :th] == k + 1).all() and (seg[:, th:] == 0).all()
        ts = tv[base[k]: base[k] + 32 * w * nb].reshape(nb, 32 * w)
        for j in range(nb):                        # getTid = (j*w + warp)*32 + lane
            assert (ts[j, :th] == (j << 16) + np.arange(th)).all()


def test_barrier_and_smem_isolation_under_sharing():
    """BAR tasks (multi-phase syncBlock across warps) and SMEM tasks (fill,
    hold, verify) share MTBs with each other and with NOP traffic: zero
    errors means barrier IDs scope only their TB and granules never overlap."""
    dev = Dev()
    err = dev.zeros(8)
    scratch = dev.zeros(4 * 992 * 15)
    with Pagoda() as p:
        for k in range(3000):
            kind = k % 3
            if kind == 0:
                a = T.records(T.BAR, 1)
                a["err"], a["scratch"], a["phases"] = ptr(err), ptr(scratch) + 0, 8
                th = [64, 128, 256, 512][k % 4]
                # shared-memory scratch (granted) so tasks do not share the global scratch
                assert p.taskSpawn(th, 1, th * 4, True, T.BAR, a) >= 0
            elif kind == 1:
                a = T.records(T.SMEM, 1)
                a["err"], a["bytes"], a["spin_ns"], a["seed"] = ptr(err) + 4, [512, 3000, 8192, 20000][k % 4], 2000, k
                assert p.taskSpawn([32, 64, 128][k % 3], 1, int(a["bytes"][0]), True, T.SMEM, a) >= 0
            else:
                assert p.taskSpawn(32 * (1 + k % 8), 1, 0, False, T.NOP) >= 0
        assert p.waitAll() == 0
    e = Dev.get(err, np.uint32)
    assert e[0] == 0, "barrier errors"
    assert e[1] == 0, "shared-memory corruption / misalignment"


def test_check_gate_semantics():
    import torch
    flag = torch.zeros(16, dtype=torch.int32).pin_memory()
    with Pagoda() as p:
        a = T.records(T.GATE, 1)
        a["flag"] = flag.data_ptr()
        tid = p.taskSpawn(32, 1, 0, False, T.GATE, a)
        after = p.taskSpawn(64, 1, 0, False, T.NOP)
        time.sleep(0.05)
        assert p.check(tid) == 0                  # still gated
        assert p.wait(after) == 0                 # others flow past a blocked task
        flag[0] = 1
        assert p.wait(tid) == 0 and p.check(tid) == 1
        assert p.check(tid + 100) == -errno.EINVAL
        assert p.wait(-1) == -errno.EINVAL


def test_validation_and_shutdown_errors():
    p = Pagoda()
    E = -errno.EINVAL
    assert p.taskSpawn(0, 1, 0, 0, T.NOP) == E
    assert p.taskSpawn(1025, 1, 0, 0, T.NOP) == E          # > 1024 threads
    assert p.taskSpawn(32, 1, 96 * 1024 + 1, 0, T.NOP) == E   # one TB larger than an MTB's arena
    assert p.taskSpawn(32, 65536, 0, 0, T.NOP) == E         # > 65535 TBs
    assert p.taskSpawn(128, 1, 0, 0, 99) == E
    assert p.taskSpawn(128, 1, 0, 0, T.NOP, b"\0" * 41) == E
    assert p.taskSpawn(1024, 1, 96 * 1024, 1, T.NOP) >= 0  # a whole MTB: all 32 warps (self-scheduling)
    assert p.taskSpawn(128, 8, 0, 1, T.NOP) >= 0
    assert p.taskSpawn(32, 32, 0, 1, T.NOP) >= 0
    assert p.shutdown() == 0


def test_multi_producer_ids_unique():
    n_thr, per = 4, 4000
    got = [[] for _ in range(n_thr)]
    with Pagoda() as p:
        def prod(i):
            for _ in range(per):
                got[i].append(p.taskSpawn(64, 1, 0, False, T.NOP))
        th = [threading.Thread(target=prod, args=(i,)) for i in range(n_thr)]
        [t.start() for t in th]
        [t.join() for t in th]
        assert p.waitAll() == 0
        for g in got:
            assert all(b > a for a, b in zip(g, g[1:]))          # increasing per producer
        allids = sorted(sum(got, []))
        assert allids == list(range(n_thr * per))              # unique across producers


@pytest.mark.parametrize("producers", [2, 3, 8])
def test_spawn_shapes_multi_producer_exactly_once(producers):
    """pagoda_taskSpawnShapesMT: several host threads spawn one workload (blocks of 256
    tasks, block b by producer b mod P) across a ring wrap: every task runs exactly once
    with its own args, the ids are a permutation of the range, and a bad shape anywhere
    rejects the whole call before anything is spawned."""
    n = 70000 + 123                                   # > ring entries (2^16): producers wait for slots
    dev = Dev()
    cnt = dev.zeros(n * 4)
    shapes = np.zeros((n, 5), np.int32)
    shapes[:, 0] = np.where(np.arange(n) % 3 == 0, 64, 32)
    shapes[:, 1] = 1
    shapes[:, 4] = T.MARK
    a = T.records(T.MARK, n)
    out = dev.zeros(64 * 4)
    a["out"], a["base"], a["tag"] = ptr(out), 0, 1
    a["cnt"] = ptr(cnt) + 4 * np.arange(n)
    with Pagoda() as p:
        bad = shapes.copy()
        bad[n - 1, 4] = 999
        with pytest.raises(OSError):
            p.spawn_shapes(bad, T.to_raw(a), producers=producers)
        assert p.info().completed_low == 0 and p.waitAll() == 0
        ids = p.spawn_shapes(shapes, T.to_raw(a), ids=True, producers=producers)
        assert p.waitAll() == 0
        assert np.array_equal(np.sort(ids), np.arange(n))
        assert all(p.check(int(i)) == 1 for i in ids[::1001])
    c = Dev.get(cnt, np.uint32)
    assert np.array_equal(c, shapes[:, 0].astype(np.uint32))   # each task's threads ran once


def test_lifecycle_stamps_ordered():
    """PAGODA_LIFECYCLE: every stage of every task is stamped once, in causal order
    (published -> loaded -> placed -> body start -> body end -> fenced -> queued ->
    forwarded; %globaltimer is one clock for all SMs, 1 us slack for its granularity)."""
    from paper_conf_ppopp_yehsser17_b200.pagoda import LIFECYCLE, NO_START
    n = 5000
    with Pagoda(flags=LIFECYCLE | NO_START) as p:
        assert p.start() == 0
        ids = p.spawn_many(n, 128, 1, 1024, True, T.NOP, None, ids=True)
        assert p.stop() == 0
        L = p.lifecycle(int(ids[0]), n).astype(np.int64)
    assert (L > 0).all()
    assert (np.diff(L, axis=1) >= -1000).all()


def test_single_mtb_context():
    """One MTB on one SM: MTB 0 runs tasks itself (single-warp ingest, completion records
    straight to the host window, no forwarders): spawn across a ring wrap and check."""
    with Pagoda(num_sms=1, mtbs_per_sm=1, arena_bytes=64 * 1024, ring_entries=1024) as p:
        assert p.info().n_mtb == 1
        ids = p.spawn_many(5000, 128, 1, 2048, True, T.NOP, None, ids=True)
        assert p.waitAll() == 0
        assert all(p.check(int(i)) == 1 for i in ids[::101])
        ids = [p.taskSpawn(992, 1, 0, True, T.NOP) for _ in range(50)]
        assert p.waitAll() == 0 and all(p.check(i) == 1 for i in ids)


def test_ring_wraparound_and_completion_window():
    """More tasks than ring entries and completion slots: slots are reused only
    after their previous occupant is consumed / done."""
    with Pagoda(ring_entries=256, comp_entries=512) as p:
        ids = p.spawn_many(20000, 64, 1, 0, False, T.NOP, None, ids=True)
        assert p.waitAll() == 0
        assert ids[-1] == 19999 and p.check(19999) == 1 and p.check(5) == 1


def test_chain_visibility():
    """Task k reads task k-1's output after a host wait (memory visibility
    across tasks)."""
    dev = Dev()
    # MM with B = I copies A exactly; chain A_k = C_{k-1}, each spawned after wait(k-1)
    eye = np.eye(32, dtype=np.float32)
    A0 = np.arange(1024, dtype=np.float32).reshape(32, 32) / 7
    Ibuf = dev.put(eye)
    mats = [dev.put(A0)] + [dev.zeros(4096) for _ in range(30)]
    with Pagoda() as p:
        for k in range(1, 31):
            a = T.records(T.MM, 1)
            a["A"], a["B"], a["C"] = ptr(mats[k - 1]), ptr(Ibuf), ptr(mats[k])
            tid = p.taskSpawn(256, 1, 8192, True, T.MM, a)
            assert p.wait(tid) == 0
    assert np.array_equal(Dev.get(mats[30], np.float32, (32, 32)), A0)


@pytest.mark.parametrize("max_tasks", [0, 2])
def test_ledger_invariants_debug_config(max_tasks):
    """Trace mode on a small grid with few executor warps and a small arena:
    the oracle-side checker replays every MTB's allocator events (no double
    assignment of warps / granules / barrier IDs, frees match allocs, every
    TB allocated once on one MTB, everything freed).  With a claim cap
    (pagoda_config.max_tasks) no MTB ever runs more than that many tasks at once."""
    import oracle
    rng = np.random.default_rng(5)
    alphabet = [(32, 1, 0, 0), (64, 1, 0, 1), (128, 1, 0, 1), (32, 1, 512, 0), (64, 1, 2048, 1), (128, 1, 4096, 1),
                (32, 3, 1024, 1), (96, 2, 0, 1)]
    dev = Dev()
    err = dev.zeros(8)
    n = 1500
    with Pagoda(num_sms=2, mtbs_per_sm=1, exec_warps=8, arena_bytes=16 * 1024 + 16384, flags=TRACE,
                trace_events=16384, max_tasks=max_tasks) as p:
        info = p.info()
        meta = []
        for k in range(n):
            th, nb, sh, sy = alphabet[rng.integers(len(alphabet))]
            a = T.records(T.SMEM, 1)
            a["err"], a["bytes"], a["spin_ns"], a["seed"] = ptr(err), sh, int(rng.integers(0, 3000)), k
            tid = p.taskSpawn(th, nb, sh, sy, T.SMEM if sh else T.NOP, a if sh else None)
            assert tid == k
            meta.append((tid, ((th + 31) // 32) * nb, nb))
        assert p.waitAll() == 0
        time.sleep(0.05)      # let schedulers fold the last frees into the ledger
        evs = np.concatenate([p.trace(m) for m in range(info.n_mtb)])
        ex = [p.exec_trace(m, w) for m in range(info.n_mtb) for w in range(32)]
    assert Dev.get(err, np.uint32)[0] == 0
    tasks = np.array(meta, oracle.TASK_DTYPE)
    granules = (16 * 1024 + 16384) // 512
    # MTB 0 lends 32 granules to the ingest warp: checking against the full arena is the weaker bound
    ok, msg = oracle.ledger_check(evs.view(oracle.LEDGER_DTYPE), info.n_mtb, 8, granules, 15, tasks)
    assert ok, msg
    # a warp never runs two tasks at once
    for e in ex:
        if len(e) > 1:
            s = np.sort(e, order="t_start")
            assert (s["t_start"][1:] >= s["t_end"][:-1]).all()
    assert sum(len(e) for e in ex) == sum(m[1] for m in meta)
    if max_tasks:   # tasks in a body at once, per MTB (a task: its first warp's start to its last warp's end)
        for m in range(info.n_mtb):
            recs = np.concatenate(ex[m * 32:(m + 1) * 32])
            if len(recs) == 0:
                continue
            ids = np.unique(recs["task_id"])
            st = np.array([recs["t_start"][recs["task_id"] == i].min() for i in ids], np.int64)
            en = np.array([recs["t_end"][recs["task_id"] == i].max() for i in ids], np.int64)
            evs = sorted([(int(x), 1) for x in st] + [(int(x), -1) for x in en], key=lambda e: (e[0], e[1]))
            cur = peak = 0
            for _, dv in evs:
                cur += dv
                peak = max(peak, cur)
            assert peak <= max_tasks, (m, peak)


def test_sessions_stop_start_and_drain():
    """pagoda_stop / pagoda_start keep ring positions and ids; a drain session
    runs everything spawned while stopped and exits by itself; every task still
    completes exactly once (MARK counters)."""
    from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START
    dev = Dev()
    n = 6000
    cnt = dev.zeros(4 * n)
    out = dev.zeros(4 * 64 * n)
    a = T.records(T.MARK, n)
    a["out"], a["cnt"] = ptr(out), ptr(cnt) + 4 * np.arange(n)
    a["base"], a["tag"] = 64 * np.arange(n), np.arange(n) + 1
    with Pagoda(flags=NO_START) as p:
        ids = p.spawn_many(2000, 64, 1, 0, False, T.MARK, a[:2000], ids=True)   # while stopped
        assert p.check(int(ids[-1])) == 0
        assert p.start_drain() == 0
        assert p.stop() == 0
        assert p.check(int(ids[-1])) == 1 and p.session_ms() > 0
        for s in range(2):
            assert p.start() == 0
            lo = 2000 + 2000 * s
            ids = p.spawn_many(2000, 64, 1, 0, False, T.MARK, a[lo:lo + 2000], ids=True)
            assert p.stop() == 0
            assert all(p.check(int(i)) == 1 for i in ids[::97])
        assert p.start() == 0
    c = Dev.get(cnt, np.uint32)
    assert (c == 64).all()
    o = Dev.get(out, np.uint32).reshape(n, 64)
    assert (o == (np.arange(n) + 1)[:, None]).all()


@pytest.mark.gpu
def test_session_starting_exactly_at_the_ring_wrap():
    """Each session spawns exactly R tasks, so every new session's first spawn
    needs ring slot 0 of the previous lap: the host must see the consumed count
    of the previous session (a reset of it would block the spawn forever)."""
    R = 4096
    from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START
    with Pagoda(ring_entries=R, flags=NO_START, watchdog_s=20.0) as p:
        for _ in range(4):
            assert p.start() == 0
            p.spawn_many(R, 128, 1, 0, False, T.NOP, None)
            assert p.stop() == 0


def test_pingpong_floor():
    """The PCIe round-trip floor: every echo returns, in
    microseconds, and an isolated NOP task costs at least one round trip."""
    from paper_conf_ppopp_yehsser17_b200.pagoda import pingpong
    rtt = pingpong(0, 500)
    assert (rtt > 0).all() and np.median(rtt) < 50_000
    with Pagoda() as p:
        lat = p.latency_loop(200, 128, 1, 0, False, T.NOP)
    assert np.median(lat) >= 0.9 * np.median(rtt)


# ---------------------------------------------------------------- tasks spread over several MTBs (NEXT-3)
def test_spread_tasks_ids_and_exactly_once():
    """Tasks larger than one MTB (Fig. 8's large tasks): MARK and
    TID over k MTB entries run every thread once, the task completes once, and
    it consumes k ids; the oracle-side rule gives the same ids."""
    import oracle as O
    dev = Dev()
    cases = [(128, 64, 0, 1), (32, 2048, 0, 0), (1024, 5, 0, 1), (100, 40, 600, 1), (64, 17, 48 * 1024, 1)]
    cap = sum(th * nb for th, nb, _, _ in cases)
    out = dev.zeros(4 * 4 * (32 * 2048 + 4096))
    cnt = dev.zeros(4 * len(cases))
    tid_out = dev.zeros(4 * 32 * 2048)
    orc = O.Ctx(exec_warps=32)
    with Pagoda() as p:
        ids, base = [], 0
        for i, (th, nb, sh, sy) in enumerate(cases):
            args = np.array([(ptr(out) + 4 * base, ptr(cnt) + 4 * i, 0, 1000 + i)], T.ARGS[T.MARK])
            ids.append(p.taskSpawn(th, nb, sh, sy, T.MARK, args))
            assert orc.spawn(th, nb, sh, sy, O.NOP, None) == ids[-1]   # same id rule
            base += ((th + 31) // 32) * 32 * nb
        targs = np.array([(ptr(tid_out), 0, 0)], T.ARGS[T.TID])
        tid_id = p.taskSpawn(32, 2048, 0, 0, T.TID, targs)
        nop = p.taskSpawn(32, 1, 0, 0, T.NOP)
        assert ids[0] == 0 and ids[1] == 8 and tid_id > ids[-1] and nop > tid_id
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert all(p.check(i) == 1 for i in ids + [tid_id, nop])
    c = Dev.get(cnt, np.uint32)
    o = Dev.get(out, np.uint32)
    base = 0
    for i, (th, nb, _, _) in enumerate(cases):
        assert c[i] == th * nb, (i, c[i])
        span = ((th + 31) // 32) * 32
        seg = o[base: base + span * nb].reshape(nb, span)
        assert (seg[:, :th] == 1000 + i).all() and (seg[:, th:] == 0).all(), i
        base += span * nb
    t = Dev.get(tid_out, np.uint32)
    assert np.array_equal(t >> 16, np.arange(32 * 2048) // 32)           # getBlockIdx: global TB index
    assert np.array_equal(t & 0xFFFF, np.arange(32 * 2048) % 32)         # getBlockTid


def test_spread_task_parity_and_sync():
    """Bodies over spread tasks: a Mandelbrot tile with 4096 threads (16 TBs of
    256 = 2 MTB entries), 3DES with 32 TBs, and BAR phases (syncBlock per TB)
    over 40 syncing TBs."""
    import oracle as O
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    mb = W.mandelbrot(8, threads=256)
    mb.shapes[:, 1] = 16
    td = W.tdes(6, shmem=2560)
    td.shapes[:, 1] = 32
    dev = Dev()
    err = dev.zeros(4)
    scratch = dev.zeros(4 * 1024 * 40)
    bargs = np.array([(ptr(err), ptr(scratch), 5, 0)], T.ARGS[T.BAR])
    with Pagoda() as p:
        p.spawn_shapes(mb.shapes, mb.args)
        p.spawn_shapes(td.shapes, td.args)
        p.taskSpawn(128, 40, 0, 1, T.BAR, bargs)
        assert p.waitAll() == 0 and p.info().device_error == 0
    out = mb.outputs()["out"]
    for k in range(8):
        assert np.array_equal(out[k], O.mandelbrot_tile(int(mb.host["tx"][k]), int(mb.host["ty"][k])))
    out = td.outputs()["out"]
    for k in range(6):
        assert np.array_equal(out[k], O.tdes_ecb(td.host["packets"][k], I.TDES_KEYS))
    assert Dev.get(err, np.uint32)[0] == 0


def test_four_mtbs_per_sm():
    """512-thread MTBs, 4 per SM (twice the schedulers): 592 MTBs, 16 worker
    warps each; a 1024-thread TB no longer fits one MTB (-EINVAL); 16-warp TBs
    and tasks spread over MTBs still run exactly once; MM parity."""
    import oracle
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    w = W.matmul(2000)
    with Pagoda(mtbs_per_sm=4, arena_bytes=48 * 1024) as p:
        i = p.info()
        assert i.n_mtb == 592 and i.exec_warps == 16
        assert p.taskSpawn(1024, 1, 0, 0, T.NOP) == -errno.EINVAL
        ids = p.spawn_many(3000, 512, 1, 0, True, T.NOP, None, ids=True)
        big = p.taskSpawn(128, 40, 0, 1, T.NOP)
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert all(p.check(int(x)) == 1 for x in ids[::101]) and p.check(big) == 1
    out = w.outputs()["C"]
    for k in range(0, 2000, 37):
        assert np.array_equal(out[k], oracle.mm32(w.host["A"][k], w.host["B"][k])), k


def _pool_members():
    """Pool members: every GPU present; on a one-GPU machine two half-GPU members (2 x 74 SMs:
    two co-resident MasterKernels, SURVEY §4 layer 6)."""
    import torch
    n = torch.cuda.device_count()
    return (list(range(n)), {}) if n > 1 else ([0, 0], {"num_sms": 74})


def test_pool_least_loaded_spawner():
    """The in-process multi-GPU pool: one spawner thread per member (NUMA-bound),
    runs of tasks claimed least-loaded-first.  Single spawns and batched spawns land on every
    member, complete, and compute what the oracle does (config 5 tasks)."""
    import oracle
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    from paper_conf_ppopp_yehsser17_b200.pagoda import Pool
    devs, cfg = _pool_members()
    n_dev = len(devs)
    ws = [W.c5(3000, pool_size=32, device=f"cuda:{d}", fill=0xAB) for d in devs]
    pool = Pool(devs, **cfg)
    assert pool.size() == n_dev
    assert pool.pick(4) in range(n_dev)
    tid, idx = pool.spawn(128, 1, 0, False, T.NOP, [b""] * n_dev)
    assert tid >= 0 and idx in range(n_dev)
    ids, dev = pool.spawn_shapes(ws[0].shapes, [w.args for w in ws], chunk=64)
    assert pool.waitAll() == 0
    assert (ids >= 0).all() and set(np.unique(dev)) == set(range(n_dev))   # every member took runs
    st = [pool.stats(i) for i in range(n_dev)]
    assert sum(s[0] for s in st) == 3000 and all(s[1] > 0 for s in st)
    assert pool.shutdown() == 0
    for k in range(0, 3000, 97):
        w = ws[int(dev[k])]
        kind = w.kind(k)
        args = w.pool.oracle_inputs(kind, int(w.in_idx[k]))
        ref = {"mb": lambda *a: oracle.mandelbrot_tile(*a), "mm": oracle.mm32, "fb": oracle.filterbank,
               "bf": oracle.beamformer, "conv": oracle.conv, "dct": oracle.dct,
               "tdes": lambda pk: oracle.tdes_ecb(pk, __import__("paper_conf_ppopp_yehsser17_b200.inputs",
                                                                  fromlist=["x"]).TDES_KEYS)}[kind](*args)
        assert np.array_equal(w.task_output(k), ref), (kind, k)


def test_pool_two_members_c5_parity_every_task():
    """Config 5's mix through the pool's least-loaded spawners on two members (two GPUs, or
    two 74-SM MasterKernels on one): every task runs once, on exactly one member, with that
    member's inputs, and matches the oracle (all 4000 tasks checked)."""
    import oracle
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, Pool
    devs, cfg = _pool_members()
    devs = devs[:2]
    n = 4000
    ws = [W.c5(n, pool_size=64, device=f"cuda:{d}", fill=0xCD) for d in devs]
    pool = Pool(devs, flags=NO_START, **cfg)
    pool.dct_register([w.dct_coef for w in ws])     # registered before any member starts
    assert pool.start() == 0
    ids, dev = pool.spawn_shapes(ws[0].shapes, [w.args for w in ws], chunk=32)
    assert pool.waitAll() == 0 and pool.stop() == 0
    assert pool.shutdown() == 0
    assert np.bincount(dev, minlength=2).min() > 0
    ref = {"mm": oracle.mm32, "fb": oracle.filterbank, "bf": oracle.beamformer, "conv": oracle.conv,
           "dct": oracle.dct, "mb": lambda *a: oracle.mandelbrot_tile(*a),
           "tdes": lambda pk: oracle.tdes_ecb(pk, I.TDES_KEYS)}
    cache = {}
    for k in range(n):
        mine, other = ws[int(dev[k])], ws[1 - int(dev[k])]
        kind = mine.kind(k)
        key = (kind, int(mine.in_idx[k]))
        if key not in cache:
            cache[key] = ref[kind](*mine.pool.oracle_inputs(kind, int(mine.in_idx[k])))
        assert np.array_equal(mine.task_output(k), cache[key]), (kind, k)
        assert not np.array_equal(other.task_output(k), cache[key]), (kind, k)   # ran on one member only


# ---------------------------------------------------------------- device errors and the paper-named device API
def test_paper_free_functions_body():
    """A body written only against the paper's free functions getTid() / syncBlock() /
    getSMPtr() (Table 1, PAGODA_PAPER): multi-warp TBs of sync tasks exchange
    values across warps through syncBlock, getTid covers [0, 32 w n_tb) once, no errors."""
    dev = Dev()
    shapes = [(64, 1, 1), (100, 3, 1), (256, 2, 1), (32, 4, 0), (1024, 1, 1)]   # threads, n_tb, sync
    span = [((th + 31) // 32) * 32 * nb for th, nb, _ in shapes]
    out = dev.zeros(4 * sum(span))
    err = dev.zeros(8)
    with Pagoda() as p:
        base = 0
        for (th, nb, sy), sp in zip(shapes, span):
            a = np.array([(ptr(out), ptr(err), base, 0)], T.ARGS[T.PAPER])
            assert p.taskSpawn(th, nb, 512, sy, T.PAPER, a) >= 0
            base += sp
        assert p.waitAll() == 0 and p.info().device_error == 0
    o = Dev.get(out, np.uint32)
    assert Dev.get(err, np.uint32)[0] == 0
    base = 0
    for (th, nb, _), sp in zip(shapes, span):
        w = (th + 31) // 32
        seg = o[base: base + sp].reshape(nb, 32 * w)
        tids = np.arange(sp).reshape(nb, 32 * w)
        assert (seg[:, :th] == tids[:, :th] + 1).all() and (seg[:, th:] == 0).all()
        base += sp


@pytest.mark.parametrize("body", ["paper", "env"])
def test_sync_without_flag_is_a_device_error(body):
    """syncBlock() in a multi-warp TB spawned with sync=0 (it has no barrier ID)
    sets PAGODA_DEVERR_SYNC_WITHOUT_FLAG — from the free function (PAPER body) and from the
    Env form (BAR body) alike — and every later host call on the context returns -EIO."""
    dev = Dev()
    out = dev.zeros(4 * 4096)
    err = dev.zeros(8)
    scratch = dev.zeros(4 * 4096)
    p = Pagoda()
    if body == "paper":
        good = np.array([(ptr(out), ptr(err), 0, 0)], T.ARGS[T.PAPER])
        bad = np.array([(ptr(out), ptr(err), 1024, 0)], T.ARGS[T.PAPER])
        func = T.PAPER
    else:
        good = bad = np.array([(ptr(err), ptr(scratch), 2, 0)], T.ARGS[T.BAR])
        func = T.BAR
    ok = p.taskSpawn(128, 2, 0, 1, func, good)
    one_warp = p.taskSpawn(32, 2, 0, 0, func, good)      # 1-warp TBs may syncBlock without the flag
    assert p.wait(ok) == 0 and p.wait(one_warp) == 0 and p.info().device_error == 0
    tid = p.taskSpawn(64, 1, 0, 0, func, bad)           # 2 warps, sync = 0: violation
    assert tid >= 0
    t0 = time.time()
    while p.info().device_error == 0 and time.time() - t0 < 5:
        time.sleep(0.001)
    assert p.info().device_error & 1
    E = -errno.EIO
    assert p.wait(tid) == E and p.check(tid) == E and p.check(ok) == E
    assert p.waitAll() == E
    assert p.taskSpawn(32, 1, 0, 0, T.NOP) == E
    assert p.shutdown() == E


def test_nonblocking_spawn_eagain_without_id_holes():
    """PAGODA_NONBLOCKING_SPAWN: while the ring is full, taskSpawn returns
    -EAGAIN at once and reserves no id; a stopped session with a full ring does the same
    even without the flag; the ids that were issued stay contiguous and all complete."""
    from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, NONBLOCKING_SPAWN, PagodaError
    R = 256
    for flags in (NO_START | NONBLOCKING_SPAWN, NO_START):
        with Pagoda(ring_entries=R, comp_entries=1024, flags=flags, watchdog_s=20.0) as p:
            ids = p.spawn_many(R, 64, 1, 0, False, T.NOP, None, ids=True)   # stopped: fills the ring
            assert np.array_equal(ids, np.arange(R))
            assert p.taskSpawn(64, 1, 0, False, T.NOP) == -errno.EAGAIN
            with pytest.raises(PagodaError) as ei:
                p.spawn_many(10, 64, 1, 0, False, T.NOP, None)
            assert ei.value.errno == errno.EAGAIN and ei.value.spawned == 0
            assert p.info().spawned == R                                   # no id was taken
            assert p.start() == 0
            assert p.waitAll() == 0
            tid = p.taskSpawn(64, 1, 0, False, T.NOP)
            assert tid == R and p.wait(tid) == 0


def test_shmem_grant_above_255_granules():
    """A request of more than 255 granules (here 140000 B = 274 granules, 1 MTB/SM with a
    200 KiB arena) gets its whole grant: the SMEM body fails if getSMBytes() < the request
    and verifies every word it filled."""
    dev = Dev()
    err = dev.zeros(8)
    with Pagoda(mtbs_per_sm=1, arena_bytes=200 * 1024) as p:
        for k, nbytes in enumerate((130560, 131072, 140000, 200 * 1024)):
            a = T.records(T.SMEM, 1)
            a["err"], a["bytes"], a["spin_ns"], a["seed"] = ptr(err), nbytes, 1000, k
            assert p.taskSpawn(256, 1, nbytes, True, T.SMEM, a) >= 0
        assert p.waitAll() == 0 and p.info().device_error == 0
    assert Dev.get(err, np.uint32)[0] == 0


@pytest.mark.parametrize("max_tasks", [1, 2])
def test_claim_cap_sessions_drain_every_task(max_tasks):
    """A claim cap holds claims back while a finished task's slot awaits its fold (the last warp frees
    itself before posting); a scheduler must still not leave the session while tickets remain
    unclaimed.  Back-to-back sessions of short tasks under caps of 1 and 2 all drain."""
    with Pagoda(max_tasks=max_tasks, flags=NO_START) as p:
        for s in range(6):
            assert p.start() == 0
            p.spawn_many(4000, 128, 1, 0, False, T.NOP, None)
            assert p.stop() == 0, s
        assert p.info().completed_low == 24000
