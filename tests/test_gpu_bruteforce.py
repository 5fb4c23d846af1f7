"""Tiny brute-forced schedules (SURVEY §4 layer 4, §8(c) "Brute-force mode"; BASELINE.json north
star: "warps and shared memory are never over-allocated on tiny brute-forced schedules").

Debug configuration: ONE MTB with 4 worker warps and an 8-granule (4 KiB) arena.  Every spawn
sequence of length 1..4 over the 6-shape alphabet (warps, shmem, sync) in
{(1,0,0), (2,0,1), (4,0,1), (1,512,0), (2,2048,1), (4,4096,1)} — 6 + 36 + 216 + 1296 = 1554
sequences — runs as HOLD tasks (fill the grant, hold until the host opens the task's gate,
verify the grant).  Each sequence runs once per order of opening its gates (L! orders: 32478
runs): when an opened task is running the host waits for it, so completions follow that order
wherever placement allows; tasks not yet placed run when resources free (FIFO, Alg. 1 L14-28).

Per session the oracle-side checkers replay the MasterKernel's ledger and executor records:
  orc_ledger_check — per-MTB allocator replay: no warp / granule / barrier ID double-assigned,
      capacities (4 warps, 8 granules, 15 IDs) never exceeded, frees match allocations
      (Alg. 2 P:821-859 warp counter; allocator invariant P:927-934);
  orc_exec_check  — a warp never runs two tasks at once, executed warps are the allocated ones,
      one completion per task after its last warp ended (Alg. 1 L41-43);
and liveness: every sequence completes (each task fits an empty MTB).
"""
import itertools
import time

import numpy as np
import pytest

import oracle
from gpu_util import Dev, ptr
from paper_conf_ppopp_yehsser17_b200 import tasks as T
from paper_conf_ppopp_yehsser17_b200.pagoda import LIFECYCLE, NO_START, TRACE, Pagoda

pytestmark = pytest.mark.gpu

ALPHABET = [(1, 0, 0), (2, 0, 1), (4, 0, 1), (1, 512, 0), (2, 2048, 1), (4, 4096, 1)]   # (warps, shmem, sync)
EXEC_WARPS, GRANULES, BAR_IDS = 4, 8, 15
ARENA = 2 * 128 * 64 + GRANULES * 512   # a single MTB lends 2 x 128 ingest entries of its arena


def runs():
    """(sequence, gate order) for every sequence of length <= 4 and every order of its gates."""
    for L in range(1, 5):
        for seq in itertools.product(range(len(ALPHABET)), repeat=L):
            for order in itertools.permutations(range(L)):
                yield seq, order


def test_alphabet_counts():
    seqs = {s for s, _ in runs()}
    assert len(seqs) == 1554
    assert sum(1 for _ in runs()) == 6 + 36 * 2 + 216 * 6 + 1296 * 24


def _check_session(p, info, metas, first_id, exec_warps=EXEC_WARPS, granules=GRANULES):
    """Replay one session's ledger + executor records + completion stamps (one ledger per
    scheduling group: the checker sees each group as an MTB with its own share)."""
    n_led = info.n_mtb * info.sched_groups
    evs = np.concatenate([p.trace(m) for m in range(n_led)])
    ex = np.concatenate([p.exec_trace(0, w) for w in range(32)])
    n_ids = metas[-1][0] - first_id + 1
    life = p.lifecycle(first_id, n_ids)
    tasks = np.array([(tid, w, 1) for tid, w in metas], oracle.TASK_DTYPE)
    if info.sched_groups == 1:
        ok, msg = oracle.ledger_check(evs.view(oracle.LEDGER_DTYPE), n_led, exec_warps, granules, BAR_IDS, tasks)
    else:
        # group g's workers are warps [16 g, 16 g + exec_warps / 2) and its granules / barrier IDs its own
        # halves: every ALLOC must lie in its group's share (the checker then replays all 32 warp bits)
        per = exec_warps // 2
        for g in range(2):
            e = evs[(evs["mtb"] == g) & (evs["kind"] == 1)]
            assert not (e["warp_mask"] & ~np.uint32(((1 << per) - 1) << (16 * g))).any(), g
            e2 = e[e["gran_len"] > 0]
            assert ((e2["gran_off"] >= granules // 2 * g) & (e2["gran_off"] + e2["gran_len"] <= granules // 2 * (g + 1))).all()
            b = e["bar_id"][e["bar_id"] > 0]
            assert ((b >= 1) & (b <= 7)).all() if g == 0 else ((b >= 8) & (b <= 15)).all()
        ok, msg = oracle.ledger_check(evs.view(oracle.LEDGER_DTYPE), n_led, 32, granules, BAR_IDS, tasks)
    assert ok, msg
    done = np.maximum(life[:, 6], life[:, 7])   # one MTB: the record goes to the host at stamp 6
    comps = np.array([(tid, done[tid - first_id]) for tid, _ in metas], oracle.COMP_DTYPE)
    assert (comps["t_done"] > 0).all()
    ok, msg = oracle.exec_check(evs.view(oracle.LEDGER_DTYPE), ex.view(oracle.EXEC_DTYPE), comps, tasks)
    assert ok, msg
    return len(evs), len(ex)


@pytest.mark.parametrize("groups", [1, 2])
def test_bruteforce_tiny_schedules(groups):
    """groups = 2: the same MTB split into two scheduling groups (pagoda_config.sched_groups),
    each with 4 warps, 8 granules and its own named barriers (1..7 / 8..15) and token."""
    import torch
    dev = Dev()
    err = dev.zeros(8)
    gate = torch.zeros(64, dtype=torch.int32).pin_memory()
    started = torch.zeros(64, dtype=torch.int32).pin_memory()
    g, s = gate.numpy(), started.numpy()
    all_runs = list(runs())
    per_session = 4096
    cap = 1 << 18
    ew, gr = EXEC_WARPS * groups, GRANULES * groups
    with Pagoda(num_sms=1, mtbs_per_sm=1, exec_warps=ew, arena_bytes=2 * 128 * 64 + gr * 512, ring_entries=1024,
                comp_entries=1 << 17, flags=TRACE | LIFECYCLE | NO_START, trace_events=cap,
                watchdog_s=30.0, sched_groups=groups) as p:
        info = p.info()
        assert info.n_mtb == 1 and info.exec_warps == ew and info.sched_groups == groups
        # the debug config's limits are enforced at spawn (one TB must fit the MTB)
        import errno
        assert p.taskSpawn(160, 1, 0, 1, T.NOP) == -errno.EINVAL            # 5 warps > 4
        assert p.taskSpawn(32, 1, GRANULES * 512 + 1, 0, T.NOP) == -errno.EINVAL
        a = T.records(T.HOLD, 1)
        n_events = n_exec = n_tasks = 0
        for s0 in range(0, len(all_runs), per_session):
            assert p.start() == 0
            metas, first = [], None
            for seq, order in all_runs[s0:s0 + per_session]:
                g[:4] = 0
                s[:4] = 0
                ids = []
                for i, k in enumerate(seq):
                    w, sh, sy = ALPHABET[k]
                    a["flag"], a["err"], a["started"], a["seed"] = gate.data_ptr() + 4 * i, ptr(err), \
                        started.data_ptr() + 4 * i, len(metas)
                    tid = p.taskSpawn(32 * w, 1, sh, sy, T.HOLD, a)
                    assert tid >= 0, tid
                    first = tid if first is None else first
                    ids.append(tid)
                    metas.append((tid, w))
                for i in order:
                    g[i] = 1
                    t0 = time.perf_counter()
                    while s[i] == 0 and time.perf_counter() - t0 < 30e-6:
                        pass
                    if s[i]:                   # running: let it finish before the next gate opens
                        assert p.wait(ids[i]) == 0
                assert p.waitAll() == 0       # liveness: every task of the sequence completed
            assert p.stop() == 0
            e, x = _check_session(p, info, metas, first, ew, gr)
            n_events += e
            n_exec += x
            n_tasks += len(metas)
        assert p.info().device_error == 0
    assert Dev.get(err, np.uint32)[0] == 0, "a HOLD task's granted shared memory was overwritten"
    assert n_tasks == sum(len(sq) for sq, _ in all_runs)
    print(f"brute force: {len(all_runs)} runs, {n_tasks} tasks, {n_events} ledger events, {n_exec} warp intervals")
