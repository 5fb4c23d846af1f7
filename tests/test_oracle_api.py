"""Pins for the oracle's Table-1 API semantics and the trace-ledger checker (CPU only)."""
import errno
import struct

import numpy as np
import pytest

import oracle as O


def test_spawn_ids_monotone_and_semantics(orc):
    ctx = O.Ctx()
    ids = [ctx.spawn(128, 1, 0, 0, O.NOP, None) for _ in range(5)]
    assert ids == list(range(5))
    assert all(ctx.check(i) == 1 for i in ids)
    assert ctx.wait(3) == 0 and ctx.waitAll() == 0
    assert ctx.wait(5) == -errno.EINVAL and ctx.check(-1) == -errno.EINVAL
    assert ctx.shutdown() == 0
    assert ctx.spawn(128, 1, 0, 0, O.NOP, None) == -errno.ESHUTDOWN


@pytest.mark.parametrize("threads,ntb,shmem,sync,func,nargs,ok", [
    (0, 1, 0, 0, O.NOP, 0, False),          # threads < 1
    (992, 1, 0, 0, O.NOP, 0, True),         # 31 warps: one whole MTB
    (993, 1, 0, 0, O.NOP, 0, False),        # one TB of 32 warps > 31 executor warps
    (1025, 1, 0, 0, O.NOP, 0, False),       # > 1024 threads per TB
    (128, 8, 0, 0, O.NOP, 0, True),         # 4 warps x 8 TBs = 32 > 31: spread over 2 MTBs
    (128, 7, 0, 1, O.NOP, 0, True),
    (32, 1, 96 * 1024, 0, O.NOP, 0, True),  # whole arena
    (32, 1, 96 * 1024 + 1, 0, O.NOP, 0, False),   # one TB larger than an MTB's arena
    (32, 2, 48 * 1024 + 1, 0, O.NOP, 0, True),    # 2 x 97 granules > 192: spread
    (32, 31, 0, 1, O.NOP, 0, True),         # 1-warp TBs need no barrier ID
    (64, 15, 0, 1, O.NOP, 0, True),         # 15 barrier IDs (16 minus ID 0)
    (64, 16, 0, 1, O.NOP, 0, True),         # 16 syncing TBs: spread (15 + 1)
    (32, 65536, 0, 0, O.NOP, 0, False),     # > 65535 TBs
    (1024, 1, 0, 0, O.NOP, 0, False),       # 32 warps > the 31 executor warps of this context
    (128, 1, 0, 0, 99, 0, False),           # unknown func
    (128, 1, 0, 0, O.NOP, 41, False),       # args > 40 B
    (128, 1, -1, 0, O.NOP, 0, False),
])
def test_validation_table(orc, threads, ntb, shmem, sync, func, nargs, ok):
    ctx = O.Ctx()
    args = bytes(nargs) if nargs else None
    rc = ctx.spawn(threads, ntb, shmem, sync, func, args)
    assert (rc >= 0) == ok, rc
    if not ok:
        assert rc == -errno.EINVAL


def test_spread_task_ids(orc):
    """A task larger than one MTB consumes k = ceil(n_tb / cap) ids (its id is
    the first), and runs every TB: MARK over 64 TBs of 4 warps (cap 7 per MTB
    of 31 warps -> 10 entries)."""
    ctx = O.Ctx()
    out = np.zeros(64 * 128, np.uint32)
    cnt = np.zeros(1, np.uint32)
    a = ctx.spawn(128, 1, 0, 0, O.NOP, None)
    args = struct.pack("<QQII", out.ctypes.data, cnt.ctypes.data, 0, 5)
    b = ctx.spawn(128, 64, 0, 1, O.MARK, args)
    c = ctx.spawn(128, 1, 0, 0, O.NOP, None)
    assert (a, b, c) == (0, 1, 1 + 10)
    assert (out == 5).all() and cnt[0] == 64 * 128
    assert ctx.wait(b) == 0 and ctx.check(b + 3) == 1 and ctx.waitAll() == 0
    ctx32 = O.Ctx(exec_warps=32)
    assert ctx32.spawn(1024, 3, 0, 1, O.NOP, None) == 0 and ctx32.spawn(32, 1, 0, 0, O.NOP, None) == 3


def test_mark_and_tid_bodies(orc):
    ctx = O.Ctx()
    out = np.zeros(4096, np.uint32)
    cnt = np.zeros(4, np.uint32)
    args = struct.pack("<QQII", out.ctypes.data, cnt.ctypes.data + 4, 100, 77)
    tid = ctx.spawn(100, 3, 0, 1, O.MARK, args)      # 100 threads = 4 warps per TB, 3 TBs
    assert tid == 0
    # live threads: TB j covers getTid in [128 j, 128 j + 100)
    want = np.zeros(4096, np.uint32)
    for j in range(3):
        want[100 + 128 * j: 100 + 128 * j + 100] = 77
    assert np.array_equal(out, want) and cnt[1] == 300
    out[:] = 0
    args = struct.pack("<QI4x", out.ctypes.data, 8)
    assert ctx.spawn(40, 2, 0, 0, O.TID, args) == 1
    for j in range(2):
        for t in range(40):
            assert out[8 + 64 * j + t] == (j << 16 | t)


# ------------------------------------------------------------------ ledger checker
def ev(seq, mtb, kind, task, tb, mask, goff=0, glen=0, bar=0):
    # field order of O.LEDGER_DTYPE
    return (seq, mtb, kind, bar, task, mask, tb, goff, glen, 0, 0)


def tasks(*rows):
    return np.array(list(rows), O.TASK_DTYPE)


def check(events, ts, n_mtb=2, exec_warps=31, gran=192, bars=15):   # workers = warps 0..30
    return O.ledger_check(np.array(events, O.LEDGER_DTYPE), n_mtb, exec_warps, gran, bars, ts)


def test_ledger_accepts_valid_trace(orc):
    evs = [ev(0, 0, 1, 7, 0, 0b11110, 0, 4, 1), ev(1, 0, 1, 8, 0, 0b1100000, 4, 2, 2),
           ev(2, 0, 2, 7, 0, 0b00110), ev(3, 0, 2, 7, 0, 0b11000), ev(4, 0, 3, 7, 0, 0, 0, 4, 1),
           ev(5, 0, 1, 9, 0, 0b11110, 0, 4, 1),   # reuse after free
           ev(6, 0, 2, 8, 0, 0b1100000), ev(7, 0, 3, 8, 0, 0, 4, 2, 2),
           ev(8, 0, 2, 9, 0, 0b11110), ev(9, 0, 3, 9, 0, 0, 0, 4, 1),
           ev(0, 1, 1, 10, 0, 0b10, 0, 0, 0), ev(1, 1, 1, 10, 1, 0b100), ev(2, 1, 2, 10, 1, 0b100),
           ev(3, 1, 3, 10, 1, 0), ev(4, 1, 2, 10, 0, 0b10), ev(5, 1, 3, 10, 0, 0)]
    ok, msg = check(evs, tasks((7, 4, 1), (8, 2, 1), (9, 4, 1), (10, 2, 2)))
    assert ok, msg


@pytest.mark.parametrize("bad,needle", [
    ([ev(0, 0, 1, 1, 0, 0b10), ev(1, 0, 1, 2, 0, 0b110)], "double-assigned"),
    ([ev(0, 0, 1, 1, 0, 0b10, 0, 4), ev(1, 0, 1, 2, 0, 0b100, 3, 2)], "granule 3 double"),
    ([ev(0, 0, 1, 1, 0, 0b10, 0, 0, 3), ev(1, 0, 1, 2, 0, 0b100, 0, 0, 3)], "barrier id 3"),
    ([ev(0, 0, 1, 1, 0, 0b10, 190, 4)], "exceed arena"),
    ([ev(0, 0, 1, 1, 0, 1 << 31)], "bad warp mask"),   # warp 31 > exec_warps - 1 = 30
    ([ev(0, 0, 1, 1, 0, 0b10), ev(1, 0, 2, 1, 0, 0b110)], "not live"),
    ([ev(0, 0, 1, 1, 0, 0b10, 0, 2), ev(1, 0, 2, 1, 0, 0b10), ev(2, 0, 3, 1, 0, 0, 0, 1)], "differ"),
    ([ev(0, 0, 1, 1, 0, 0b10)], "never freed"),
    ([ev(0, 0, 1, 1, 0, 0b10), ev(0, 1, 1, 1, 1, 0b10), ev(1, 0, 2, 1, 0, 0b10), ev(2, 0, 3, 1, 0, 0),
      ev(1, 1, 2, 1, 1, 0b10), ev(2, 1, 3, 1, 1, 0)], "TBs on MTBs"),
])
def test_ledger_rejects(orc, bad, needle):
    n_tb = 2 if needle == "TBs on MTBs" else 1
    ok, msg = check(bad, tasks((1, 1 * n_tb, n_tb), (2, 2, 1)))
    assert not ok and needle in msg, msg


# ------------------------------------------------------------------ executor-interval / completion checker
# Two tasks on MTB 0: task 1 (1 TB, warps 1-2), task 2 (1 TB, warp 1 after task 1 freed it).
def _valid_exec_case():
    evs = [ev(0, 0, 1, 1, 0, 0b110), ev(1, 0, 2, 1, 0, 0b110), ev(2, 0, 3, 1, 0, 0),
           ev(3, 0, 1, 2, 0, 0b10), ev(4, 0, 2, 2, 0, 0b10), ev(5, 0, 3, 2, 0, 0)]
    ex = [(1, 0, 0, 0, 1, 100, 200), (1, 0, 0, 0, 2, 110, 210), (2, 0, 0, 0, 1, 220, 300)]
    comps = [(1, 215), (2, 305)]
    return evs, ex, comps, tasks((1, 2, 1), (2, 1, 1))


def xcheck(evs, ex, comps, ts):
    return O.exec_check(np.array(evs, O.LEDGER_DTYPE), np.array(ex, O.EXEC_DTYPE),
                        np.array(comps, O.COMP_DTYPE), ts)


def test_exec_check_accepts_valid(orc):
    evs, ex, comps, ts = _valid_exec_case()
    ok, msg = xcheck(evs, ex, comps, ts)
    assert ok, msg
    ok, msg = check(evs, ts, n_mtb=1)        # the same trace passes the allocator replay too
    assert ok, msg


@pytest.mark.parametrize("mutate,needle", [
    (lambda e, x, c: x.__setitem__(2, (2, 0, 0, 0, 1, 190, 300)), "before task"),          # warp 1 overlap
    (lambda e, x, c: c.__setitem__(0, (1, 205)), "before its last warp ended"),          # early completion
    (lambda e, x, c: c.pop(), "no completion"),
    (lambda e, x, c: c.append((1, 400)), "completed twice"),
    (lambda e, x, c: x.__setitem__(2, (2, 0, 0, 0, 3, 220, 300)), "outside its ALLOC"),  # wrong warp
    (lambda e, x, c: x.__setitem__(2, (2, 0, 0, 1, 1, 220, 300)), "allocated on MTB"),   # wrong MTB
    (lambda e, x, c: x.pop(1), "allocated"),                                              # a warp never ran
    (lambda e, x, c: x.append((1, 0, 0, 0, 1, 500, 600)), "ran twice"),
    (lambda e, x, c: x.__setitem__(0, (1, 0, 0, 0, 1, 200, 100)), "ends before"),
    (lambda e, x, c: x.append((3, 0, 0, 0, 5, 500, 600)), "without an ALLOC"),
    (lambda e, x, c: c.append((9, 1)), "unlisted"),
])
def test_exec_check_rejects(orc, mutate, needle):
    evs, ex, comps, ts = _valid_exec_case()
    mutate(evs, ex, comps)
    ok, msg = xcheck(evs, ex, comps, ts)
    assert not ok and needle in msg, msg
