"""oracle — TEST INFRASTRUCTURE ONLY.

The plain sequential CPU definition of what the Pagoda hot path computes
(oracle.c; see its header).  Only tests/, __graft_entry__.smoke() and bench.py's
cpu_baseline / --impl reference legs may import this package.  It shares no
code with paper_conf_ppopp_yehsser17_b200 (the CUDA product); the product never
imports it.

Parity status of every function is listed in DESIGN.md "Oracle pins": all
body functions and the API are pinned by tests/test_oracle_*.py; nothing here
is "parity unpinned".
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess
import threading

import numpy as np

HERE = os.path.dirname(os.path.abspath(__file__))
SRC = os.path.join(HERE, "oracle.c")
LIB = os.path.join(HERE, "liboracle.so")
LIB_FAST = os.path.join(HERE, "liboracle_fast.so")

CFLAGS = ["-O2", "-std=c11", "-Wall", "-ffp-contract=off", "-fno-fast-math", "-fPIC", "-shared"]
# the TIMED build (SURVEY §8(d) "CPU oracle"): same source, -O3 -march=native, still no contraction
# (so its outputs equal the parity build's; bench.py checks a sample)
CFLAGS_FAST = ["-O3", "-march=native", "-std=c11", "-Wall", "-ffp-contract=off", "-fno-fast-math", "-fPIC",
               "-shared"]

# func ids — the oracle's own numbering (oracle.h)
NOP, MARK, TID, MB, TDES, MM, FB, BF, CONV, DCT, MM_TC = 0, 1, 2, 16, 17, 18, 19, 20, 21, 22, 23

_lock = threading.Lock()
_libs = {}


def build(force: bool = False, fast: bool = False) -> str:
    """Compile oracle.c -> liboracle.so (parity build) or liboracle_fast.so (timed build) with gcc (no CUDA)."""
    out, flags = (LIB_FAST, CFLAGS_FAST) if fast else (LIB, CFLAGS)
    stale = (not os.path.exists(out)) or any(
        os.path.getmtime(os.path.join(HERE, f)) > os.path.getmtime(out)
        for f in ("oracle.c", "oracle.h", "__init__.py"))
    if force or stale:
        tmp = out + f".tmp{os.getpid()}"
        subprocess.check_call(["gcc", *flags, "-o", tmp, SRC, "-lm"])
        os.replace(tmp, out)
    return out


def lib(fast: bool = False):
    """The parity build (default) or the -O3 -march=native timed build."""
    with _lock:
        if fast not in _libs:
            L = C.CDLL(build(fast=fast))
            P, I, I64, F, SZ = C.c_void_p, C.c_int, C.c_int64, C.c_float, C.c_size_t
            L.orc_mandelbrot_tile.argtypes = [P, F, F, F, I, I, I]
            L.orc_des_key_schedule.argtypes = [P, P]
            L.orc_des_block.argtypes = [C.c_uint64, P, I]
            L.orc_des_block.restype = C.c_uint64
            L.orc_tdes_ecb.argtypes = [P, P, SZ, P, I]
            L.orc_mm32.argtypes = [P, P, P]
            L.orc_mm32_f64.argtypes = [P, P, P]
            L.orc_mm64.argtypes = [P, P, P]
            L.orc_filterbank.argtypes = [P, P, P, P]
            L.orc_beamformer.argtypes = [P, P, P, P]
            L.orc_conv.argtypes = [P, P, P, P]
            L.orc_dct.argtypes = [P, P, P]
            L.orc_init.argtypes = [I, I, C.POINTER(P)]
            L.orc_taskSpawn.argtypes = [P, I, I, I, I, I, P, SZ]
            L.orc_taskSpawn.restype = I64
            L.orc_wait.argtypes = [P, I64]
            L.orc_check.argtypes = [P, I64]
            L.orc_waitAll.argtypes = [P]
            L.orc_shutdown.argtypes = [P]
            L.orc_destroy.argtypes = [P]
            L.orc_occupancy_pct.argtypes = [I, I]
            L.orc_occupancy_pct.restype = C.c_double
            L.orc_ledger_check.argtypes = [P, SZ, I, I, I, I, P, SZ, C.c_char_p, SZ]
            L.orc_exec_check.argtypes = [P, SZ, P, SZ, P, SZ, P, SZ, C.c_char_p, SZ]
            _libs[fast] = L
    return _libs[fast]


def _p(a: np.ndarray):
    assert a.flags["C_CONTIGUOUS"]
    return a.ctypes.data_as(C.c_void_p)


# ----------------------------------------------------------------- bodies
def mandelbrot_tile(tx: int, ty: int, x0=-2.0, y0=-1.5, dx=3.0 / 2048, maxit=256, L=None) -> np.ndarray:
    out = np.zeros((64, 64), np.uint16)
    (L or lib()).orc_mandelbrot_tile(_p(out), x0, y0, dx, tx, ty, maxit)
    return out


def des_key_schedule(key8: bytes) -> np.ndarray:
    k = np.frombuffer(key8, np.uint8).copy()
    sk = np.zeros(16, np.uint64)
    lib().orc_des_key_schedule(_p(k), _p(sk))
    return sk


def des_block(block: int, key8: bytes, decrypt=False) -> int:
    sk = des_key_schedule(key8)
    return int(lib().orc_des_block(C.c_uint64(block), _p(sk), int(decrypt)))


def tdes_ecb(data, key24: bytes, decrypt=False, L=None) -> np.ndarray:
    inp = np.ascontiguousarray(np.frombuffer(bytes(data), np.uint8) if not isinstance(data, np.ndarray) else data, dtype=np.uint8)
    out = np.zeros_like(inp)
    k = np.frombuffer(key24, np.uint8).copy()
    (L or lib()).orc_tdes_ecb(_p(inp), _p(out), inp.size, _p(k), int(decrypt))
    return out


def mm32(A, B, L=None) -> np.ndarray:
    A = np.ascontiguousarray(A, np.float32); B = np.ascontiguousarray(B, np.float32)
    Cm = np.zeros((32, 32), np.float32)
    (L or lib()).orc_mm32(_p(A), _p(B), _p(Cm))
    return Cm


def mm64(A, B, L=None) -> np.ndarray:
    """Table 4's 64x64x64 MatrixMul: fma chain over k ascending, as mm32."""
    A = np.ascontiguousarray(A, np.float32); B = np.ascontiguousarray(B, np.float32)
    Cm = np.zeros((64, 64), np.float32)
    (L or lib()).orc_mm64(_p(A), _p(B), _p(Cm))
    return Cm


def mm32_exact(A, B, L=None) -> np.ndarray:
    """C = A B accumulated in fp64, rounded once (the tensor-core MM variant's definition)."""
    A = np.ascontiguousarray(A, np.float32); B = np.ascontiguousarray(B, np.float32)
    Cm = np.zeros((32, 32), np.float32)
    (L or lib()).orc_mm32_f64(_p(A), _p(B), _p(Cm))
    return Cm


def filterbank(r, H, F, L=None) -> np.ndarray:
    r, H, F = (np.ascontiguousarray(v, np.float32) for v in (r, H, F))
    y = np.zeros(2048, np.float32)
    (L or lib()).orc_filterbank(_p(r), _p(H), _p(F), _p(y))
    return y


def beamformer(x, h, w, L=None) -> np.ndarray:
    x, h, w = (np.ascontiguousarray(v, np.float32) for v in (x, h, w))
    out = np.zeros((4, 512), np.float32)
    (L or lib()).orc_beamformer(_p(x), _p(h), _p(w), _p(out))
    return out


def conv(img, krow, kcol, L=None) -> np.ndarray:
    img, krow, kcol = (np.ascontiguousarray(v, np.float32) for v in (img, krow, kcol))
    out = np.zeros((128, 128), np.float32)
    (L or lib()).orc_conv(_p(img), _p(krow), _p(kcol), _p(out))
    return out


def dct(img, coef, L=None) -> np.ndarray:
    img, coef = (np.ascontiguousarray(v, np.float32) for v in (img, coef))
    out = np.zeros((128, 128), np.float32)
    (L or lib()).orc_dct(_p(img), _p(coef), _p(out))
    return out


def occupancy_pct(resident_warps: int, n_sm: int) -> float:
    return float(lib().orc_occupancy_pct(resident_warps, n_sm))


# ----------------------------------------------------------------- API
class Ctx:
    """Sequential Table-1 API: spawn runs the body at once (oracle.h)."""

    def __init__(self, exec_warps: int = 31, arena_bytes: int = 96 * 1024):
        self.h = C.c_void_p()
        rc = lib().orc_init(exec_warps, arena_bytes, C.byref(self.h))
        if rc:
            raise OSError(-rc, "orc_init")
        self._keep = []

    def spawn(self, threads, n_tb, shmem, sync, func_id, args: bytes | None) -> int:
        buf = C.create_string_buffer(args, len(args)) if args else None
        return int(lib().orc_taskSpawn(self.h, threads, n_tb, shmem, int(sync), func_id,
                                       buf, len(args) if args else 0))

    def wait(self, tid) -> int: return lib().orc_wait(self.h, tid)
    def check(self, tid) -> int: return lib().orc_check(self.h, tid)
    def waitAll(self) -> int: return lib().orc_waitAll(self.h)
    def shutdown(self) -> int: return lib().orc_shutdown(self.h)

    def __del__(self):
        try:
            lib().orc_destroy(self.h)
        except Exception:
            pass


# ----------------------------------------------------------------- ledger
LEDGER_DTYPE = np.dtype([("seq", "<u4"), ("mtb", "<u2"), ("kind", "u1"), ("bar_id", "u1"),
                         ("task_id", "<u8"), ("warp_mask", "<u4"), ("tb", "<u2"),
                         ("gran_off", "<u2"), ("gran_len", "<u2"), ("pad", "<u2"), ("pad2", "<u4")])
TASK_DTYPE = np.dtype([("task_id", "<u8"), ("warps_total", "<u4"), ("n_tb", "<u4")])
assert LEDGER_DTYPE.itemsize == 32 and TASK_DTYPE.itemsize == 16


def ledger_check(events: np.ndarray, n_mtb: int, exec_warps: int, arena_granules: int,
                 n_bar_ids: int, tasks: np.ndarray):
    """Return (ok, message)."""
    events = np.ascontiguousarray(events, LEDGER_DTYPE)
    tasks = np.ascontiguousarray(tasks, TASK_DTYPE)
    err = C.create_string_buffer(512)
    rc = lib().orc_ledger_check(_p(events) if len(events) else None, len(events), n_mtb, exec_warps,
                                arena_granules, n_bar_ids, _p(tasks) if len(tasks) else None,
                                len(tasks), err, 512)
    return rc == 0, err.value.decode()


EXEC_DTYPE = np.dtype([("task_id", "<u8"), ("tb", "<u2"), ("smid", "<u2"), ("mtb", "<u2"), ("warp", "<u2"),
                       ("t_start", "<u8"), ("t_end", "<u8")])
COMP_DTYPE = np.dtype([("task_id", "<u8"), ("t_done", "<u8")])
assert EXEC_DTYPE.itemsize == 32 and COMP_DTYPE.itemsize == 16


def exec_check(events: np.ndarray, execs: np.ndarray, comps: np.ndarray, tasks: np.ndarray):
    """Executor intervals + completion records against the ledger (oracle.h orc_exec_check).
    Return (ok, message)."""
    events = np.ascontiguousarray(events, LEDGER_DTYPE)
    execs = np.ascontiguousarray(execs, EXEC_DTYPE)
    comps = np.ascontiguousarray(comps, COMP_DTYPE)
    tasks = np.ascontiguousarray(tasks, TASK_DTYPE)
    err = C.create_string_buffer(512)

    def q(a):
        return _p(a) if len(a) else None
    rc = lib().orc_exec_check(q(events), len(events), q(execs), len(execs), q(comps), len(comps),
                              q(tasks), len(tasks), err, 512)
    return rc == 0, err.value.decode()
