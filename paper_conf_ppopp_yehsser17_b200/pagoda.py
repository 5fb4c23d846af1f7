"""Thin ctypes binding of libpagoda.so (include/pagoda.h) — argument marshalling
only; every step of the hot path runs in the library's C++/CUDA code.

There is no fallback: if libpagoda.so is missing this module raises on use.
PyTorch (if used by the caller) only provides device memory; pass
tensor.data_ptr() values inside the args records.
"""
from __future__ import annotations

import ctypes as C
import errno
import os

import numpy as np

PKG = os.path.dirname(os.path.abspath(__file__))
# PAGODA_LIB selects another build of the same library (A/B experiments, scripts/build_variants.sh)
LIB_PATH = os.environ.get("PAGODA_LIB") or os.path.join(PKG, "libpagoda.so")

TRACE = 0x1
NO_START = 0x2
RESIDENT_TDES = 0x4
LIFECYCLE = 0x8
SPREAD = 0x10
NONBLOCKING_SPAWN = 0x20
CE_INGEST = 0x40
LIFE_EVENTS = ("pub", "load", "place", "start", "end", "done", "queued", "fwd")


class pagoda_config(C.Structure):
    _fields_ = [("device", C.c_int), ("mtbs_per_sm", C.c_int), ("num_sms", C.c_int),
                ("ring_entries", C.c_uint32), ("comp_entries", C.c_uint32), ("arena_bytes", C.c_uint32),
                ("exec_warps", C.c_uint32), ("flags", C.c_uint32), ("trace_events", C.c_uint32),
                ("watchdog_s", C.c_double), ("sched_groups", C.c_uint32), ("max_tasks", C.c_uint32)]


class pagoda_info(C.Structure):
    _fields_ = [("device", C.c_int), ("sm_count", C.c_int), ("n_mtb", C.c_int), ("mtbs_per_sm", C.c_int),
                ("exec_warps", C.c_int), ("arena_bytes", C.c_int), ("regs_per_thread", C.c_int),
                ("ring_entries", C.c_uint32), ("comp_entries", C.c_uint32), ("spawned", C.c_int64),
                ("completed_low", C.c_int64), ("device_error", C.c_uint32), ("running", C.c_int),
                ("sched_groups", C.c_int)]


LEDGER_DTYPE = np.dtype([("seq", "<u4"), ("mtb", "<u2"), ("kind", "u1"), ("bar_id", "u1"),
                         ("task_id", "<u8"), ("warp_mask", "<u4"), ("tb", "<u2"), ("gran_off", "<u2"),
                         ("gran_len", "<u2"), ("pad", "<u2"), ("pad2", "<u4")])
EXEC_DTYPE = np.dtype([("task_id", "<u8"), ("tb", "<u2"), ("smid", "<u2"), ("mtb", "<u2"), ("warp", "<u2"),
                       ("t_start", "<u8"), ("t_end", "<u8")])

# names declared in include/pagoda.h (the ABI test checks the library exports them)
_lib = None


def lib() -> C.CDLL:
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise RuntimeError(f"{LIB_PATH} is not built: run paper_conf_ppopp_yehsser17_b200.build.build() "
                               "(there is no CPU fallback)")
        L = C.CDLL(LIB_PATH)
        P, I, I64, SZ, U32 = C.c_void_p, C.c_int, C.c_int64, C.c_size_t, C.c_uint32
        L.pagoda_config_default.argtypes = [C.POINTER(pagoda_config)]
        L.pagoda_init.argtypes = [C.POINTER(pagoda_config), C.POINTER(P)]
        L.pagoda_shutdown.argtypes = [P]
        L.pagoda_taskSpawn.argtypes = [P, I, I, I, I, I, P, SZ]
        L.pagoda_taskSpawn.restype = I64
        L.pagoda_wait.argtypes = [P, I64]
        L.pagoda_check.argtypes = [P, I64]
        L.pagoda_waitAll.argtypes = [P]
        L.pagoda_waitBelow.argtypes = [P, I64]
        L.pagoda_taskSpawnMany.argtypes = [P, I, I, I, I, I, I, P, SZ, SZ, P]
        L.pagoda_taskSpawnMany.restype = I64
        L.pagoda_taskSpawnShapes.argtypes = [P, I, P, P, SZ, SZ, P]
        L.pagoda_taskSpawnShapes.restype = I64
        L.pagoda_taskSpawnShapesMT.argtypes = [P, I, P, P, SZ, SZ, P, I]
        L.pagoda_taskSpawnShapesMT.restype = I64
        L.pagoda_get_info.argtypes = [P, C.POINTER(pagoda_info)]
        L.pagoda_trace_read.argtypes = [P, I, P, SZ]
        L.pagoda_trace_read.restype = I64
        L.pagoda_trace_read_exec.argtypes = [P, I, I, P, SZ]
        L.pagoda_trace_read_exec.restype = I64
        L.pagoda_lifecycle_read.argtypes = [P, C.c_uint64, SZ, P]
        L.pagoda_lifecycle_read.restype = I64
        L.pagoda_tdes_tables.argtypes = [P, P]
        L.pagoda_naive_run.argtypes = [I, I, P, P, SZ, SZ, I, C.POINTER(I64)]
        L.pagoda_pingpong.argtypes = [I, I, P]
        L.pagoda_measure_pipe_peak.argtypes = [I, I, C.POINTER(C.c_double), C.POINTER(C.c_double)]
        L.pagoda_tdes_register.argtypes = [P, P]
        L.pagoda_dct_register.argtypes = [P, P]
        L.pagoda_fused_run.argtypes = [I, I, P, P, SZ, SZ, I, C.POINTER(I64), C.POINTER(C.c_float)]
        L.pagoda_pool_init.argtypes = [I, P, C.POINTER(pagoda_config), C.POINTER(P)]
        L.pagoda_pool_pick.argtypes = [P, I]
        L.pagoda_pool_ctx.argtypes = [P, I]
        L.pagoda_pool_ctx.restype = P
        L.pagoda_pool_size.argtypes = [P]
        L.pagoda_pool_spawn.argtypes = [P, I, I, I, I, I, P, SZ, C.POINTER(I)]
        L.pagoda_pool_spawn.restype = I64
        L.pagoda_pool_waitAll.argtypes = [P]
        L.pagoda_pool_spawn_shapes.argtypes = [P, I, P, P, SZ, SZ, I, P, P]
        L.pagoda_pool_spawn_shapes.restype = I64
        L.pagoda_pool_shutdown.argtypes = [P]
        L.pagoda_pool_numa_node.argtypes = [P, I]
        L.pagoda_pool_stats.argtypes = [P, I, P, P, P]
        L.pagoda_pool_may_claim.argtypes = [P, I, I, I64]
        L.pagoda_inflight_warps.argtypes = [P]
        L.pagoda_inflight_warps.restype = I64
        L.pagoda_pick_least_loaded.argtypes = [P, I]
        L.pagoda_version.restype = C.c_char_p
        L.pagoda_stop.argtypes = [P]
        L.pagoda_start.argtypes = [P]
        L.pagoda_start_drain.argtypes = [P]
        L.pagoda_session_ms.argtypes = [P, C.POINTER(C.c_float)]
        L.pagoda_run_timed.argtypes = [P, I, P, P, SZ, SZ, P, P]
        L.pagoda_run_timed.restype = I64
        L.pagoda_run_open_loop.argtypes = [P, I, P, P, SZ, SZ, P, P, P]
        L.pagoda_run_open_loop.restype = I64
        L.pagoda_latency_loop.argtypes = [P, I, I, I, I, I, I, P, SZ, P]
        L.pagoda_read_counters.argtypes = [P, P, I]
        _lib = L
    return _lib


class PagodaError(OSError):
    pass


def _check(rc: int, what: str) -> int:
    if rc < 0:
        raise PagodaError(-rc, f"{what}: {os.strerror(-rc)}")
    return rc


def _check_count(rc: int, n: int, what: str) -> None:
    """A batched spawn cut short by a full ring (PAGODA_NONBLOCKING_SPAWN or a stopped
    session) returns how many it spawned; `spawned` carries that count."""
    if rc == n:
        return
    if rc == -errno.EAGAIN or 0 <= rc < n:
        e = PagodaError(errno.EAGAIN, f"{what}: ring full after {max(rc, 0)} of {n} tasks")
        e.spawned = max(rc, 0)
        raise e
    _check(rc, what)


def _ptr(a):
    if a is None:
        return None
    if isinstance(a, np.ndarray):
        assert a.flags["C_CONTIGUOUS"]
        return a.ctypes.data_as(C.c_void_p)
    return a


def pool_may_claim(loads, me: int, slack: int) -> int:
    """The pool spawners' claim rule (host-only): 1 if loads[me] <= min(loads) + slack."""
    a = np.ascontiguousarray(loads, np.int64)
    return lib().pagoda_pool_may_claim(_ptr(a), len(a), me, slack)


def default_config(**kw) -> pagoda_config:
    cfg = pagoda_config()
    lib().pagoda_config_default(C.byref(cfg))
    for k, v in kw.items():
        setattr(cfg, k, v)
    return cfg


class Pagoda:
    """One Pagoda context (one MasterKernel on one GPU).  Method names follow
    the paper's Table 1."""

    def __init__(self, **config):
        self.cfg = default_config(**config)
        self.h = C.c_void_p()
        _check(lib().pagoda_init(C.byref(self.cfg), C.byref(self.h)), "pagoda_init")
        self._alive = True

    # --- Table 1 -----------------------------------------------------------
    def taskSpawn(self, threads: int, n_tb: int, shmem: int, sync: bool, func_id: int, args=None) -> int:
        """Returns the task id (>= 0) or a negative errno (no exception, as the C ABI)."""
        if args is None:
            return lib().pagoda_taskSpawn(self.h, threads, n_tb, shmem, int(sync), func_id, None, 0)
        b = args.tobytes() if isinstance(args, np.ndarray) else bytes(args)
        return lib().pagoda_taskSpawn(self.h, threads, n_tb, shmem, int(sync), func_id, b, len(b))

    def wait(self, task_id: int) -> int:
        return lib().pagoda_wait(self.h, task_id)

    def check(self, task_id: int) -> int:
        return lib().pagoda_check(self.h, task_id)

    def waitAll(self) -> int:
        return lib().pagoda_waitAll(self.h)

    def waitBelow(self, end: int) -> int:
        return lib().pagoda_waitBelow(self.h, end)

    # --- batch conveniences (each task is still one taskSpawn in C) --------
    def spawn_many(self, n, threads, n_tb, shmem, sync, func_id, args: np.ndarray | None, ids=False):
        out = np.empty(n, np.int64) if ids else None
        stride = args.dtype.itemsize if args is not None else 0
        rc = lib().pagoda_taskSpawnMany(self.h, n, threads, n_tb, shmem, int(sync), func_id, _ptr(args),
                                        stride, stride, _ptr(out))
        _check_count(rc, n, "pagoda_taskSpawnMany")
        return out

    def spawn_shapes(self, shapes: np.ndarray, args: np.ndarray, ids=False, producers: int = 1):
        """shapes: int32 [n,5] = threads, n_tb, shmem, sync, func_id; args: uint8 [n,40].
        producers > 1: pagoda_taskSpawnShapesMT (that many host threads)."""
        shapes = np.ascontiguousarray(shapes, np.int32)
        args = np.ascontiguousarray(args, np.uint8)
        n = len(shapes)
        out = np.empty(n, np.int64) if ids else None
        if producers > 1:
            rc = lib().pagoda_taskSpawnShapesMT(self.h, n, _ptr(shapes), _ptr(args), args.shape[1], args.shape[1],
                                                _ptr(out), producers)
            _check(rc, "pagoda_taskSpawnShapesMT")
        else:
            rc = lib().pagoda_taskSpawnShapes(self.h, n, _ptr(shapes), _ptr(args), args.shape[1], args.shape[1],
                                              _ptr(out))
            _check_count(rc, n, "pagoda_taskSpawnShapes")
        return out

    # --- sessions ------------------------------------------------------------
    def stop(self) -> int:
        return lib().pagoda_stop(self.h)

    def start(self) -> int:
        return lib().pagoda_start(self.h)

    def start_drain(self) -> int:
        return lib().pagoda_start_drain(self.h)

    def session_ms(self) -> float:
        ms = C.c_float(0)
        _check(lib().pagoda_session_ms(self.h, C.byref(ms)), "pagoda_session_ms")
        return ms.value

    # --- measurement ---------------------------------------------------------
    def run_timed(self, shapes: np.ndarray, args: np.ndarray):
        """Spawn all; returns (spawn_ns, done_ns) int64 arrays (CLOCK_MONOTONIC)."""
        shapes = np.ascontiguousarray(shapes, np.int32)
        args = np.ascontiguousarray(args, np.uint8)
        n = len(shapes)
        sp, dn = np.zeros(n, np.int64), np.zeros(n, np.int64)
        _check(lib().pagoda_run_timed(self.h, n, _ptr(shapes), _ptr(args), args.shape[1], args.shape[1],
                                      _ptr(sp), _ptr(dn)), "pagoda_run_timed")
        return sp, dn

    def run_open_loop(self, shapes: np.ndarray, args: np.ndarray, arrival_ns: np.ndarray):
        """Spawn task i at call time + arrival_ns[i]; returns (arrive_ns, done_ns) (CLOCK_MONOTONIC)."""
        shapes = np.ascontiguousarray(shapes, np.int32)
        args = np.ascontiguousarray(args, np.uint8)
        arr = np.ascontiguousarray(arrival_ns, np.int64)
        n = len(shapes)
        sp, dn = np.zeros(n, np.int64), np.zeros(n, np.int64)
        _check(lib().pagoda_run_open_loop(self.h, n, _ptr(shapes), _ptr(args), args.shape[1], args.shape[1],
                                          _ptr(arr), _ptr(sp), _ptr(dn)), "pagoda_run_open_loop")
        return sp, dn

    def latency_loop(self, n, threads, n_tb, shmem, sync, func_id, args=None) -> np.ndarray:
        lat = np.zeros(n, np.int64)
        b = (args.tobytes() if isinstance(args, np.ndarray) else bytes(args)) if args is not None else None
        _check(lib().pagoda_latency_loop(self.h, n, threads, n_tb, shmem, int(sync), func_id, b,
                                         len(b) if b else 0, _ptr(lat)), "pagoda_latency_loop")
        return lat

    def tdes_register(self, dev_tables) -> int:
        """Resident round keys for 3DES tasks using this tables pointer (context stopped)."""
        return _check(lib().pagoda_tdes_register(self.h, dev_tables), "pagoda_tdes_register")

    def dct_register(self, dev_coef) -> int:
        """Constant-bank DCT coefficients for DCT tasks using this coef pointer (context stopped)."""
        return _check(lib().pagoda_dct_register(self.h, dev_coef), "pagoda_dct_register")

    def info(self) -> pagoda_info:
        i = pagoda_info()
        _check(lib().pagoda_get_info(self.h, C.byref(i)), "pagoda_get_info")
        return i

    COUNTERS = ("ingest_batches", "ingest_entries", "ingest_ns_doorbell", "ingest_ns_copy", "ingest_ns_publish",
                "ingest_ring_full", "sched_rounds", "sched_progress", "tickets", "claim_empty", "load_not_ready",
                "placed", "place_nofit", "handoffs", "ingest_ns_fence", "ingest_ns_store",
                "sched_ns_fold", "sched_ns_load", "sched_ns_place", "sched_ns_claim", "sched_ns_sleep",
                "exec_ns_body", "exec_ns_fence", "exec_ns_post")

    def counters(self) -> dict:
        out = np.zeros(len(self.COUNTERS), np.uint64)
        _check(lib().pagoda_read_counters(self.h, _ptr(out), len(out)), "pagoda_read_counters")
        return {k: int(out[i]) for i, k in enumerate(self.COUNTERS)}

    def inflight_warps(self) -> int:
        return lib().pagoda_inflight_warps(self.h)

    def trace(self, mtb: int) -> np.ndarray:
        n = _check(lib().pagoda_trace_read(self.h, mtb, None, 0), "pagoda_trace_read")
        buf = np.zeros(min(n, self.cfg.trace_events), LEDGER_DTYPE)
        _check(lib().pagoda_trace_read(self.h, mtb, _ptr(buf), len(buf)), "pagoda_trace_read")
        if n > len(buf):
            raise PagodaError(errno.ENOSPC, f"trace overflow on MTB {mtb}: {n} events")
        return buf

    def exec_trace(self, mtb: int, warp: int) -> np.ndarray:
        n = _check(lib().pagoda_trace_read_exec(self.h, mtb, warp, None, 0), "pagoda_trace_read_exec")
        buf = np.zeros(min(n, self.cfg.trace_events), EXEC_DTYPE)
        _check(lib().pagoda_trace_read_exec(self.h, mtb, warp, _ptr(buf), len(buf)), "pagoda_trace_read_exec")
        return buf

    def lifecycle(self, first: int, n: int) -> np.ndarray:
        """PAGODA_LIFECYCLE stamps of tasks [first, first+n): uint64 [n, 8] (LIFE_EVENTS order, GPU ns)."""
        buf = np.zeros((n, 8), np.uint64)
        _check(lib().pagoda_lifecycle_read(self.h, first, n, _ptr(buf)), "pagoda_lifecycle_read")
        return buf

    def shutdown(self) -> int:
        if not self._alive:
            return 0
        self._alive = False
        return lib().pagoda_shutdown(self.h)

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.shutdown()


# --------------------------------------------------------------------- misc
def tdes_tables(key24: bytes) -> np.ndarray:
    out = np.zeros(2048 + 384 + 16384 + 16384, np.uint8)
    k = np.frombuffer(key24, np.uint8).copy()
    _check(lib().pagoda_tdes_tables(_ptr(k), _ptr(out)), "pagoda_tdes_tables")
    return out


def naive_run(device: int, shapes: np.ndarray, args: np.ndarray, n_streams: int = 32) -> int:
    """One kernel launch per task; returns elapsed host ns (launch of the first
    task -> all done)."""
    shapes = np.ascontiguousarray(shapes, np.int32)
    args = np.ascontiguousarray(args, np.uint8)
    ns = C.c_int64(0)
    _check(lib().pagoda_naive_run(device, len(shapes), _ptr(shapes), _ptr(args), args.shape[1], args.shape[1],
                                  n_streams, C.byref(ns)), "pagoda_naive_run")
    return ns.value


def fused_run(device: int, shapes: np.ndarray, args: np.ndarray, threads_per_task: int = 256):
    """Static fusion: all tasks in one kernel launch; returns (elapsed host ns
    incl. the task-table copy, kernel-only ms)."""
    shapes = np.ascontiguousarray(shapes, np.int32)
    args = np.ascontiguousarray(args, np.uint8)
    ns, ms = C.c_int64(0), C.c_float(0)
    _check(lib().pagoda_fused_run(device, len(shapes), _ptr(shapes), _ptr(args), args.shape[1], args.shape[1],
                                  threads_per_task, C.byref(ns), C.byref(ms)), "pagoda_fused_run")
    return ns.value, ms.value


def pingpong(device: int, n: int = 2000) -> np.ndarray:
    """PCIe round-trip floor: n host -> GPU -> host echoes (ns each)."""
    out = np.zeros(n, np.int64)
    _check(lib().pagoda_pingpong(device, n, _ptr(out)), "pagoda_pingpong")
    return out


def pipe_peak(device: int, which: str):
    """Measured pipe peak: which = 'lds' (3DES-pattern lookups) or 'int32' (lop3).
    Returns (ops per SM per clock, ops/s at the clock the kernel ran at)."""
    per, rate = C.c_double(), C.c_double()
    _check(lib().pagoda_measure_pipe_peak(device, {"lds": 0, "int32": 1}[which], C.byref(per), C.byref(rate)),
           "pagoda_measure_pipe_peak")
    return per.value, rate.value


def pick_least_loaded(loads) -> int:
    a = np.ascontiguousarray(loads, np.int64)
    return lib().pagoda_pick_least_loaded(_ptr(a), len(a))


def version() -> str:
    return lib().pagoda_version().decode()


class Pool:
    """One context per GPU plus the least-loaded picker."""

    def __init__(self, devices, **config):
        self.cfg = default_config(**config)
        self.devices = list(devices)
        d = np.array(self.devices, np.int32)
        self.h = C.c_void_p()
        _check(lib().pagoda_pool_init(len(d), _ptr(d), C.byref(self.cfg), C.byref(self.h)), "pagoda_pool_init")

    def pick(self, warps_hint: int) -> int:
        return lib().pagoda_pool_pick(self.h, warps_hint)

    def spawn(self, threads, n_tb, shmem, sync, func_id, args_per_dev):
        bufs = [C.create_string_buffer(bytes(a), len(bytes(a))) for a in args_per_dev]
        arr = (C.c_void_p * len(bufs))(*[C.cast(b, C.c_void_p) for b in bufs])
        idx = C.c_int(-1)
        nbytes = len(bytes(args_per_dev[0]))
        tid = lib().pagoda_pool_spawn(self.h, threads, n_tb, shmem, int(sync), func_id, arr, nbytes,
                                      C.byref(idx))
        return tid, idx.value

    def spawn_shapes(self, shapes: np.ndarray, args_per_dev, chunk: int = 256):
        """args_per_dev[i]: uint8 [n, 40] args valid on member i's device.  Every member's own
        spawner thread claims runs of `chunk` tasks least-loaded-first.  Returns (ids, member) per task."""
        shapes = np.ascontiguousarray(shapes, np.int32)
        args_per_dev = [np.ascontiguousarray(a, np.uint8) for a in args_per_dev]
        n = len(shapes)
        ids, dev = np.empty(n, np.int64), np.empty(n, np.int32)
        arr = (C.c_void_p * len(args_per_dev))(*[a.ctypes.data for a in args_per_dev])
        _check(lib().pagoda_pool_spawn_shapes(self.h, n, _ptr(shapes), arr, 40, 40, chunk, _ptr(ids), _ptr(dev)),
               "pagoda_pool_spawn_shapes")
        return ids, dev

    def ctx(self, i: int):
        return lib().pagoda_pool_ctx(self.h, i)

    def size(self) -> int:
        return lib().pagoda_pool_size(self.h)

    def numa_node(self, i: int) -> int:
        return lib().pagoda_pool_numa_node(self.h, i)

    def stats(self, i: int):
        """(tasks, spawn_ns, hold_ns) of member i in the last batched spawn."""
        t, s, h = C.c_int64(), C.c_int64(), C.c_int64()
        _check(lib().pagoda_pool_stats(self.h, i, C.byref(t), C.byref(s), C.byref(h)), "pagoda_pool_stats")
        return t.value, s.value, h.value

    def start(self) -> int:
        """pagoda_start on every member (a pool made with NO_START)."""
        for i in range(self.size()):
            rc = lib().pagoda_start(self.ctx(i))
            if rc:
                return rc
        return 0

    def stop(self) -> int:
        rc = 0
        for i in range(self.size()):
            r = lib().pagoda_stop(self.ctx(i))
            rc = rc or r
        return rc

    def session_ms(self, i: int) -> float:
        ms = C.c_float()
        _check(lib().pagoda_session_ms(self.ctx(i), C.byref(ms)), "pagoda_session_ms")
        return ms.value

    def dct_register(self, dev_coef_per_member):
        """dev_coef_per_member[i]: device pointer (int) of member i's coefficient matrix."""
        for i, t in enumerate(dev_coef_per_member):
            _check(lib().pagoda_dct_register(self.ctx(i), C.c_void_p(int(t))), "pagoda_dct_register")

    def tdes_register(self, dev_tables_per_member):
        """dev_tables_per_member[i]: device pointer (int) of member i's 3DES tables."""
        for i, t in enumerate(dev_tables_per_member):
            _check(lib().pagoda_tdes_register(self.ctx(i), C.c_void_p(int(t))), "pagoda_tdes_register")

    def waitAll(self) -> int:
        return lib().pagoda_pool_waitAll(self.h)

    def shutdown(self) -> int:
        return lib().pagoda_pool_shutdown(self.h)
