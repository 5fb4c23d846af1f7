"""Seeded synthetic input generators — the ONLY module shared by the CUDA path's
tests/bench and by the oracle's tests.

It holds no arithmetic of the method (no task body, no scheduling): it only turns
(seed, task index, count) into bytes / fp32 values with splitmix64, exactly as
SURVEY.md §8(c) "Input generation" fixes it:

    state_i = seed ^ (i * 0xD1B54A32D192ED03)          (mod 2^64)
    next():  state += 0x9E3779B97F4A7C15; z = state
             z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9
             z = (z ^ (z >> 27)) * 0x94D049BB133111EB
             return z ^ (z >> 31)
    f32(z) = ((int32)(z >> 40) - 2^23) * 2^-23        (exact, in [-1, 1))
    bytes  = the u64 outputs in little-endian order

The workloads (which task gets which stream) are described in DESIGN.md
"Input recipe"; per-body seeds are SEED ^ body tag so that streams differ.
"""
from __future__ import annotations

import numpy as np

SEED = 0x5EED
_GOLDEN = np.uint64(0x9E3779B97F4A7C15)
_M1 = np.uint64(0xBF58476D1CE4E5B9)
_M2 = np.uint64(0x94D049BB133111EB)
_TASK_MUL = np.uint64(0xD1B54A32D192ED03)

# per-body stream tags (xor-ed into SEED) so that different bodies draw
# different numbers for the same task index
TAG = {
    "mb": 0x0, "tdes": 0x3DE5, "mm": 0x3232, "fb": 0xFB00, "bf": 0xBF00,
    "conv": 0xC0DE, "dct": 0xDC70, "mix": 0x4D1C, "misc": 0x7E57, "mm64": 0x6464,
}


def splitmix64(task_idx, count: int, seed: int = SEED) -> np.ndarray:
    """Return uint64 array [len(task_idx), count]: the first `count` outputs of
    each task's splitmix64 stream."""
    idx = np.atleast_1d(np.asarray(task_idx, dtype=np.uint64))
    with np.errstate(over="ignore"):
        state0 = np.uint64(seed) ^ (idx * _TASK_MUL)
        k = np.arange(1, count + 1, dtype=np.uint64)
        z = state0[:, None] + k[None, :] * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def to_f32(z: np.ndarray) -> np.ndarray:
    """Map u64 draws to exact fp32 values in [-1, 1)."""
    top = (z >> np.uint64(40)).astype(np.int64) - (1 << 23)
    return (top.astype(np.float64) * 2.0 ** -23).astype(np.float32)


def f32_stream(task_idx, count: int, seed: int) -> np.ndarray:
    return to_f32(splitmix64(task_idx, count, seed))


def byte_stream(task_idx, nbytes: int, seed: int) -> np.ndarray:
    assert nbytes % 8 == 0
    z = splitmix64(task_idx, nbytes // 8, seed)
    return z.astype("<u8").view(np.uint8).reshape(len(z), nbytes)


# ---------------------------------------------------------------- workloads
# Each generator returns plain numpy arrays; the caller (test / bench) moves
# them wherever its backend needs them.

MB_W = 64            # tile edge (SURVEY §8c MB)
MB_GRID = 32         # 32x32 tiles -> 2048^2 image, 1024 tasks
MB_X0, MB_Y0 = -2.0, -1.5
MB_DX = 3.0 / 2048   # exact in fp32
MB_MAXIT = 256

TDES_KEYS = bytes.fromhex("0123456789ABCDEF" "23456789ABCDEF01" "456789ABCDEF0123")
TDES_KAT_PLAIN = b"The qufck brown fox jump"   # SP 800-67 example plaintext


def tdes_packets(n_tasks: int, nbytes: int = 4096, first: int = 0) -> np.ndarray:
    """[n_tasks, nbytes] uint8 packets; packet 0 starts with the SP 800-67
    example plaintext."""
    p = byte_stream(np.arange(first, first + n_tasks), nbytes, SEED ^ TAG["tdes"])
    if first == 0 and n_tasks > 0:
        p[0, :24] = np.frombuffer(TDES_KAT_PLAIN, dtype=np.uint8)
    return np.ascontiguousarray(p)


def mm_inputs(n_tasks: int, first: int = 0, integer: bool = False):
    """A, B: [n_tasks, 32, 32] fp32 uniform in [-1,1) (or integers in [-8,8])."""
    z = splitmix64(np.arange(first, first + n_tasks), 2048, SEED ^ TAG["mm"])
    if integer:
        v = ((z >> np.uint64(40)) % np.uint64(17)).astype(np.int64) - 8
        v = v.astype(np.float32)
    else:
        v = to_f32(z)
    return (np.ascontiguousarray(v[:, :1024].reshape(-1, 32, 32)),
            np.ascontiguousarray(v[:, 1024:].reshape(-1, 32, 32)))


def mm64_inputs(n_tasks: int, first: int = 0, integer: bool = False):
    """A, B: [n_tasks, 64, 64] fp32 uniform in [-1,1) (or integers in [-8,8]); Table 4's MM size."""
    z = splitmix64(np.arange(first, first + n_tasks), 8192, SEED ^ TAG["mm64"])
    if integer:
        v = (((z >> np.uint64(40)) % np.uint64(17)).astype(np.int64) - 8).astype(np.float32)
    else:
        v = to_f32(z)
    return (np.ascontiguousarray(v[:, :4096].reshape(-1, 64, 64)),
            np.ascontiguousarray(v[:, 4096:].reshape(-1, 64, 64)))


FB_NSIM, FB_NCOL, FB_NSAMP = 2048, 32, 8


def fb_inputs(n_tasks: int, first: int = 0):
    """r [n,2048], H [n,32], F [n,32] fp32."""
    v = f32_stream(np.arange(first, first + n_tasks), FB_NSIM + 2 * FB_NCOL, SEED ^ TAG["fb"])
    return (np.ascontiguousarray(v[:, :FB_NSIM]),
            np.ascontiguousarray(v[:, FB_NSIM:FB_NSIM + FB_NCOL]),
            np.ascontiguousarray(v[:, FB_NSIM + FB_NCOL:]))


BF_NCH, BF_NT, BF_L, BF_NBEAM = 4, 512, 16, 4


def bf_inputs(n_tasks: int, first: int = 0):
    """x [n,4,512,2], h [n,4,16,2], w [n,4(beam),4(ch),2] fp32 (re, im pairs)."""
    nx = BF_NCH * BF_NT * 2
    nh = BF_NCH * BF_L * 2
    nw = BF_NBEAM * BF_NCH * 2
    v = f32_stream(np.arange(first, first + n_tasks), nx + nh + nw, SEED ^ TAG["bf"])
    return (np.ascontiguousarray(v[:, :nx].reshape(-1, BF_NCH, BF_NT, 2)),
            np.ascontiguousarray(v[:, nx:nx + nh].reshape(-1, BF_NCH, BF_L, 2)),
            np.ascontiguousarray(v[:, nx + nh:].reshape(-1, BF_NBEAM, BF_NCH, 2)))


IMG = 128            # CONV / DCT image edge
CONV_R = 8           # 17 taps


def conv_inputs(n_tasks: int, first: int = 0):
    """img [n,128,128], krow [n,17], kcol [n,17] fp32."""
    m = IMG * IMG
    v = f32_stream(np.arange(first, first + n_tasks), m + 2 * (2 * CONV_R + 1), SEED ^ TAG["conv"])
    return (np.ascontiguousarray(v[:, :m].reshape(-1, IMG, IMG)),
            np.ascontiguousarray(v[:, m:m + 17]),
            np.ascontiguousarray(v[:, m + 17:]))


def dct_inputs(n_tasks: int, first: int = 0):
    """img [n,128,128] fp32."""
    v = f32_stream(np.arange(first, first + n_tasks), IMG * IMG, SEED ^ TAG["dct"])
    return np.ascontiguousarray(v.reshape(-1, IMG, IMG))


def dct_coef() -> np.ndarray:
    """The 8x8 DCT-II coefficient matrix C[u][x] = a(u) cos((2x+1)u pi/16),
    computed in float64 and rounded to fp32. Per SURVEY §8(c) DCT it is an
    INPUT of the DCT body (so neither side evaluates cos itself)."""
    u = np.arange(8)[:, None]
    x = np.arange(8)[None, :]
    a = np.where(u == 0, np.sqrt(1.0 / 8.0), 0.5)
    return (a * np.cos((2 * x + 1) * u * np.pi / 16.0)).astype(np.float32)


# heterogeneous mix (config 4): body kind, threads, shmem per task
MIX_KINDS = ("fb", "bf", "conv", "dct")
MIX_THREADS = (32, 64, 128, 256, 512)
MIX_SHMEM_KB = tuple(range(0, 49, 4))


def mix_schedule(n_tasks: int, seed: int = SEED ^ TAG["mix"]):
    """Return (kind_idx[n], threads[n], shmem_bytes[n]): n/4 of each kind in a
    seeded random order, threads uniform in MIX_THREADS, shmem request uniform
    in MIX_SHMEM_KB."""
    z = splitmix64(np.arange(n_tasks), 3, seed)
    kinds = np.arange(n_tasks) % len(MIX_KINDS)
    # seeded permutation: stable argsort of each index's first draw
    order = np.argsort(z[:, 0], kind="stable")
    kinds = kinds[order]
    thr = np.array(MIX_THREADS)[(z[:, 1] % np.uint64(len(MIX_THREADS))).astype(np.int64)]
    shm = np.array(MIX_SHMEM_KB)[(z[:, 2] % np.uint64(len(MIX_SHMEM_KB))).astype(np.int64)] * 1024
    return kinds.astype(np.int32), thr.astype(np.int32), shm.astype(np.int32)


# ---------------------------------------------------------------- NEXT-1: irregular 3DES packets
TDES_VAR_MIN, TDES_VAR_MAX = 2048, 65536   # NetBench packet sizes 2K-64K (Table 3)


def tdes_var_sizes(n_tasks: int, first: int = 0) -> np.ndarray:
    """Packet bytes per task, log-uniform in [2 KiB, 64 KiB], whole 8-byte
    blocks: blocks = floor(256 * 32^u), u = the task's draw mapped to [0, 1)."""
    z = splitmix64(np.arange(first, first + n_tasks), 1, SEED ^ TAG["tdes"] ^ 0x5A5A)[:, 0]
    u = (z >> np.uint64(11)).astype(np.float64) * 2.0 ** -53
    blocks = np.floor((TDES_VAR_MIN // 8) * (TDES_VAR_MAX / TDES_VAR_MIN) ** u).astype(np.int64)
    return (np.clip(blocks, TDES_VAR_MIN // 8, TDES_VAR_MAX // 8) * 8).astype(np.int64)


def splitmix64_ragged(task_of: np.ndarray, k_of: np.ndarray, seed: int) -> np.ndarray:
    """Output number k_of[e] (0-based) of the stream of task task_of[e], per
    element (the same numbers splitmix64() gives, for ragged per-task counts)."""
    t = np.asarray(task_of, np.uint64)
    k = np.asarray(k_of, np.uint64) + np.uint64(1)
    with np.errstate(over="ignore"):
        z = (np.uint64(seed) ^ (t * _TASK_MUL)) + k * _GOLDEN
        z = (z ^ (z >> np.uint64(30))) * _M1
        z = (z ^ (z >> np.uint64(27))) * _M2
        z = z ^ (z >> np.uint64(31))
    return z


def tdes_var_packets(sizes: np.ndarray, first: int = 0):
    """Flat uint8 payload of the irregular 3DES workload and the byte offset of
    every packet: packet k is the first sizes[k] bytes of task (first+k)'s
    3DES stream (so equal-size packets equal tdes_packets()' bytes); packet 0
    of task 0 starts with the SP 800-67 plaintext."""
    sizes = np.asarray(sizes, np.int64)
    off = np.zeros(len(sizes) + 1, np.int64)
    np.cumsum(sizes, out=off[1:])
    nblk = sizes // 8
    task = np.repeat(np.arange(first, first + len(sizes), dtype=np.int64), nblk)
    k = np.arange(int(nblk.sum()), dtype=np.int64) - np.repeat(off[:-1] // 8, nblk)
    z = splitmix64_ragged(task, k, SEED ^ TAG["tdes"])
    flat = z.astype("<u8").view(np.uint8).copy()
    if first == 0 and len(sizes) > 0:
        flat[:24] = np.frombuffer(TDES_KAT_PLAIN, dtype=np.uint8)
    return flat, off


# ---------------------------------------------------------------- NEXT-1: MPE, config 5
MPE_KINDS = ("mb", "tdes", "fb", "mm")     # 8K tasks of each, 32K in total
C5_KINDS = ("mb", "tdes", "mm", "fb", "bf", "conv", "dct")


def mpe_schedule(n_tasks: int, seed: int = SEED ^ TAG["mix"] ^ 0x3E3E) -> np.ndarray:
    """Kind index (into MPE_KINDS) per task: n/4 of each in a seeded order."""
    z = splitmix64(np.arange(n_tasks), 1, seed)[:, 0]
    kinds = np.arange(n_tasks) % len(MPE_KINDS)
    return kinds[np.argsort(z, kind="stable")].astype(np.int32)


def c5_schedule(n_tasks: int, seed: int = SEED ^ TAG["mix"] ^ 0xC5C5):
    """Config 5: kind of task i = a seeded uniform draw over
    the 7 bodies (C5_KINDS); threads / shmem requests for FB, BF, CONV, DCT as
    in config 4 (uniform in MIX_THREADS / MIX_SHMEM_KB).  Returns (kind[n],
    threads[n], shmem[n]); the threads / shmem of MB, 3DES, MM are their
    configs' fixed shapes and are filled in by the workload."""
    z = splitmix64(np.arange(n_tasks), 3, seed)
    kinds = (z[:, 0] % np.uint64(len(C5_KINDS))).astype(np.int32)
    thr = np.array(MIX_THREADS)[(z[:, 1] % np.uint64(len(MIX_THREADS))).astype(np.int64)]
    shm = np.array(MIX_SHMEM_KB)[(z[:, 2] % np.uint64(len(MIX_SHMEM_KB))).astype(np.int64)] * 1024
    return kinds, thr.astype(np.int32), shm.astype(np.int32)
