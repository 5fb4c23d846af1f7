"""Synthetic workloads of BASELINE.json's configs: device buffers (torch, memory
only), per-task shapes and packed args for libpagoda.  No task arithmetic here:
inputs come from inputs.py (seeded generators), outputs are read back raw.

A Workload holds
    shapes : int32 [n, 5]  (threads, n_tb, shmem_bytes, sync, func_id)
    args   : uint8 [n, 40] (the task's inline args, device pointers inside)
    host   : dict of numpy inputs (what the oracle is fed)
    outputs(): numpy outputs read back from the device
Everything is allocated and filled with copies (no torch kernels), so it can
be prepared before Pagoda starts and read after it stops or while it idles.
"""
from __future__ import annotations

import numpy as np
import torch

from . import inputs as I
from . import tasks as T
from .pagoda import tdes_tables


def _dev(a: np.ndarray, device) -> torch.Tensor:
    a = np.ascontiguousarray(a)
    t = torch.empty(max(a.nbytes, 16), dtype=torch.uint8, device=device)
    t[:a.nbytes].copy_(torch.from_numpy(a.view(np.uint8).reshape(-1)))
    return t


def _zeros(nbytes: int, device) -> torch.Tensor:
    return _dev(np.zeros(nbytes, np.uint8), device)


def _read(t: torch.Tensor, dtype, shape) -> np.ndarray:
    n = int(np.prod(shape)) * np.dtype(dtype).itemsize
    return t[:n].cpu().numpy().view(dtype).reshape(shape)


class Workload:
    def __init__(self, name, shapes, args, host, outs, keep, in_bytes, out_bytes):
        self.name, self.shapes, self.args, self.host = name, shapes, args, host
        self._outs, self._keep = outs, keep
        self.in_bytes, self.out_bytes = in_bytes, out_bytes   # algorithmic HBM bytes per run
        self.tdes_tables = None   # device pointer of the 3DES tables its tasks use (pagoda_tdes_register)
        self.dct_coef = None      # device pointer of the DCT coefficients its tasks use (pagoda_dct_register)

    @property
    def n(self):
        return len(self.shapes)

    def outputs(self):
        return {k: _read(t, dt, sh) for k, (t, dt, sh) in self._outs.items()}


def _shapes(n, threads, n_tb, shmem, sync, func):
    s = np.zeros((n, 5), np.int32)
    s[:, 0], s[:, 1], s[:, 2], s[:, 3], s[:, 4] = threads, n_tb, shmem, int(sync), func
    return s


# ---------------------------------------------------------------- config 1: MB
def mandelbrot(n_tasks=1024, device="cuda", threads=128, maxit=I.MB_MAXIT):
    """Tiles k = 0..n-1 of the 32x32-tile grid (k mod 1024), 64x64 pixels each."""
    out = _zeros(n_tasks * 4096 * 2, device)
    a = T.records(T.MB, n_tasks)
    k = np.arange(n_tasks) % (I.MB_GRID * I.MB_GRID)
    a["out"] = out.data_ptr() + np.arange(n_tasks) * 8192
    a["x0"], a["y0"], a["dx"] = I.MB_X0, I.MB_Y0, I.MB_DX
    a["tx"], a["ty"], a["maxit"] = k % I.MB_GRID, k // I.MB_GRID, maxit
    host = {"tx": a["tx"].copy(), "ty": a["ty"].copy(), "maxit": maxit}
    return Workload("mb", _shapes(n_tasks, threads, 1, 0, False, T.MB), T.to_raw(a), host,
                    {"out": (out, np.uint16, (n_tasks, 64, 64))}, [out], 0, n_tasks * 8192)


# ---------------------------------------------------------------- config 2: 3DES
def tdes(n_tasks=32768, device="cuda", nbytes=4096, threads=128, shmem=2560, first=0):
    pk = I.tdes_packets(n_tasks, nbytes, first)
    inp = _dev(pk, device)
    out = _zeros(pk.nbytes, device)
    tab = _dev(tdes_tables(I.TDES_KEYS), device)
    a = T.records(T.TDES, n_tasks)
    a["inp"] = inp.data_ptr() + np.arange(n_tasks) * nbytes
    a["out"] = out.data_ptr() + np.arange(n_tasks) * nbytes
    a["tables"], a["nblk"] = tab.data_ptr(), nbytes // 8
    host = {"packets": pk, "key": I.TDES_KEYS}
    w = Workload("tdes", _shapes(n_tasks, threads, 1, shmem, True, T.TDES), T.to_raw(a), host,
                 {"out": (out, np.uint8, (n_tasks, nbytes))}, [inp, out, tab], pk.nbytes, pk.nbytes)
    w.tdes_tables = tab.data_ptr()
    return w


# ---------------------------------------------------------------- config 3: MM
def matmul(n_tasks=65536, device="cuda", threads=256, shmem=8192, first=0, func=T.MM, integer=False):
    """func = T.MM (fma chains) or T.MM_TC (3xTF32 tensor cores, NEXT-4)."""
    A, B = I.mm_inputs(n_tasks, first, integer=integer)
    dA, dB = _dev(A, device), _dev(B, device)
    dC = _zeros(A.nbytes, device)
    a = T.records(T.MM, n_tasks)
    off = np.arange(n_tasks) * 4096
    a["A"], a["B"], a["C"] = dA.data_ptr() + off, dB.data_ptr() + off, dC.data_ptr() + off
    return Workload("mm" if func == T.MM else "mm_tc", _shapes(n_tasks, threads, 1, shmem, True, func), T.to_raw(a),
                    {"A": A, "B": B},
                    {"C": (dC, np.float32, (n_tasks, 32, 32))}, [dA, dB, dC], 2 * A.nbytes, A.nbytes)


# ---------------------------------------------------------------- Table 4's 64x64 MM (NEXT-4)
def matmul64(n_tasks=32768, device="cuda", threads=256, shmem=32768, first=0, integer=False):
    """32K MatrixMul tasks of 64x64x64 fp32 (Table 4); A, B staged in 32 KiB of shmem."""
    A, B = I.mm64_inputs(n_tasks, first, integer=integer)
    dA, dB = _dev(A, device), _dev(B, device)
    dC = _zeros(A.nbytes, device)
    a = T.records(T.MM64, n_tasks)
    off = np.arange(n_tasks) * 16384
    a["A"], a["B"], a["C"] = dA.data_ptr() + off, dB.data_ptr() + off, dC.data_ptr() + off
    return Workload("mm64", _shapes(n_tasks, threads, 1, shmem, True, T.MM64), T.to_raw(a), {"A": A, "B": B},
                    {"C": (dC, np.float32, (n_tasks, 64, 64))}, [dA, dB, dC], 2 * A.nbytes, A.nbytes)


# ---------------------------------------------------------------- config 4: mix
def mix(n_tasks=32768, device="cuda", first=0):
    """FB / BF / CONV / DCT in a seeded random order; threads uniform in
    {32..512}; shmem request uniform in {0,4,...,48} KiB.
    Syncing bodies (FB, CONV) are spawned with sync=1, BF and DCT with sync=0."""
    kinds, thr, shm = I.mix_schedule(n_tasks)
    idx = {k: np.nonzero(kinds == i)[0] for i, k in enumerate(I.MIX_KINDS)}
    raw = np.zeros((n_tasks, 40), np.uint8)
    shapes = np.zeros((n_tasks, 5), np.int32)
    shapes[:, 0], shapes[:, 1], shapes[:, 2] = thr, 1, shm
    host, outs, keep = {"kinds": kinds}, {}, []
    in_b = out_b = 0
    # FB
    i = idx["fb"]; n = len(i)
    r, H, F = I.fb_inputs(n, first)
    dr, dH, dF = _dev(r, device), _dev(H, device), _dev(F, device)
    dy, ds = _zeros(r.nbytes, device), _zeros(n * 1024, device)
    a = T.records(T.FB, n)
    a["r"], a["H"], a["F"] = dr.data_ptr() + np.arange(n) * 8192, dH.data_ptr() + np.arange(n) * 128, \
        dF.data_ptr() + np.arange(n) * 128
    a["y"], a["scratch"] = dy.data_ptr() + np.arange(n) * 8192, ds.data_ptr() + np.arange(n) * 1024
    raw[i] = T.to_raw(a); shapes[i, 3], shapes[i, 4] = 1, T.FB
    host["fb"] = (r, H, F); outs["fb"] = (dy, np.float32, (n, 2048)); keep += [dr, dH, dF, dy, ds]
    in_b += r.nbytes + H.nbytes + F.nbytes; out_b += r.nbytes
    # BF
    i = idx["bf"]; n = len(i)
    x, h, w = I.bf_inputs(n, first)
    dx_, dh, dw = _dev(x, device), _dev(h, device), _dev(w, device)
    do = _zeros(n * 2048 * 4, device)
    a = T.records(T.BF, n)
    a["x"], a["h"], a["w"] = dx_.data_ptr() + np.arange(n) * x[0].nbytes, dh.data_ptr() + np.arange(n) * h[0].nbytes, \
        dw.data_ptr() + np.arange(n) * w[0].nbytes
    a["out"] = do.data_ptr() + np.arange(n) * 8192
    raw[i] = T.to_raw(a); shapes[i, 3], shapes[i, 4] = 0, T.BF
    host["bf"] = (x, h, w); outs["bf"] = (do, np.float32, (n, 4, 512)); keep += [dx_, dh, dw, do]
    in_b += x.nbytes + h.nbytes + w.nbytes; out_b += n * 8192
    # CONV
    i = idx["conv"]; n = len(i)
    img, kr, kc = I.conv_inputs(n, first)
    di, dkr, dkc = _dev(img, device), _dev(kr, device), _dev(kc, device)
    dout, dscr = _zeros(img.nbytes, device), _zeros(img.nbytes, device)
    a = T.records(T.CONV, n)
    a["img"], a["krow"], a["kcol"] = di.data_ptr() + np.arange(n) * 65536, dkr.data_ptr() + np.arange(n) * 68, \
        dkc.data_ptr() + np.arange(n) * 68
    a["out"], a["scratch"] = dout.data_ptr() + np.arange(n) * 65536, dscr.data_ptr() + np.arange(n) * 65536
    raw[i] = T.to_raw(a); shapes[i, 3], shapes[i, 4] = 1, T.CONV
    host["conv"] = (img, kr, kc); outs["conv"] = (dout, np.float32, (n, 128, 128)); keep += [di, dkr, dkc, dout, dscr]
    in_b += img.nbytes + kr.nbytes + kc.nbytes; out_b += img.nbytes
    # DCT
    i = idx["dct"]; n = len(i)
    im = I.dct_inputs(n, first)
    coef = I.dct_coef()
    dim_, dco = _dev(im, device), _dev(coef, device)
    dout2 = _zeros(im.nbytes, device)
    a = T.records(T.DCT, n)
    a["img"], a["coef"], a["out"] = dim_.data_ptr() + np.arange(n) * 65536, dco.data_ptr(), \
        dout2.data_ptr() + np.arange(n) * 65536
    raw[i] = T.to_raw(a); shapes[i, 3], shapes[i, 4] = 0, T.DCT
    host["dct"] = (im, coef); outs["dct"] = (dout2, np.float32, (n, 128, 128)); keep += [dim_, dco, dout2]
    in_b += im.nbytes; out_b += im.nbytes
    w = Workload("mix", shapes, raw, host, outs, keep, in_b, out_b)
    w.dct_coef = dco.data_ptr()   # every DCT task shares one coefficient matrix (pagoda_dct_register)
    return w


# ---------------------------------------------------------------- Table 5: DCT with / without shmem
def dct(n_tasks=32768, device="cuda", threads=64, n_tb=1, shmem=8192, sync=True, first=0):
    """Table 5: 32K DCT8x8 tasks of 64 threads over 128x128 images.  With
    shmem >= 4096 and sync the body stages bands of block rows by TMA; shmem=0 reads global."""
    im = I.dct_inputs(n_tasks, first)
    coef = I.dct_coef()
    dim_, dco = _dev(im, device), _dev(coef, device)
    dout = _zeros(im.nbytes, device)
    a = T.records(T.DCT, n_tasks)
    a["img"], a["coef"], a["out"] = dim_.data_ptr() + np.arange(n_tasks) * 65536, dco.data_ptr(), \
        dout.data_ptr() + np.arange(n_tasks) * 65536
    w = Workload("dct", _shapes(n_tasks, threads, n_tb, shmem, sync, T.DCT), T.to_raw(a), {"img": im, "coef": coef},
                 {"out": (dout, np.float32, (n_tasks, 128, 128))}, [dim_, dco, dout], im.nbytes, im.nbytes)
    w.dct_coef = dco.data_ptr()   # for pagoda_dct_register
    return w


def nop(n_tasks, threads=128, n_tb=1, shmem=0, sync=False):
    return Workload("nop", _shapes(n_tasks, threads, n_tb, shmem, sync, T.NOP), np.zeros((n_tasks, 40), np.uint8),
                    {}, {}, [], 0, 0)


# ---------------------------------------------------------------- pooled multi-body workloads
# MPE (NEXT-1) and config 5: per body kind a
# pool of distinct inputs in device memory; task i of kind K uses pool entry
# in_idx[i]; every task's output (and scratch) is bump-allocated in one buffer,
# so no two tasks ever write the same bytes.
KIND_FUNC = {"mb": T.MB, "tdes": T.TDES, "mm": T.MM, "fb": T.FB, "bf": T.BF, "conv": T.CONV, "dct": T.DCT}
OUT_BYTES = {"mb": 8192, "mm": 4096, "fb": 8192, "bf": 8192, "conv": 65536, "dct": 65536}   # tdes: its packet
SCRATCH_BYTES = {"fb": 1024, "conv": 65536}
SYNC = {"mb": 0, "tdes": 1, "mm": 1, "fb": 1, "bf": 0, "conv": 1, "dct": 0}
_ALIGN = 256


class InputPool:
    """`size` distinct inputs per kind (host numpy + device copies).  3DES
    packets are 4 KiB, or log-uniform 2-64 KiB with var_tdes (NEXT-1)."""

    def __init__(self, kinds, size, device="cuda", var_tdes=False, first=0):
        self.size, self.kinds, self.keep, self.host, self.dev = size, tuple(kinds), [], {}, {}
        for k in self.kinds:
            if k == "mb":
                j = (np.arange(size) + first) % (I.MB_GRID * I.MB_GRID)
                self.host[k] = (j % I.MB_GRID, j // I.MB_GRID)
            elif k == "tdes":
                sizes = I.tdes_var_sizes(size, first) if var_tdes else np.full(size, 4096, np.int64)
                flat, off = I.tdes_var_packets(sizes, first)
                d = _dev(flat, device)
                tab = _dev(tdes_tables(I.TDES_KEYS), device)
                self.host[k] = (flat, off)
                self.dev[k] = (d.data_ptr() + off[:-1], tab.data_ptr())
                self.keep += [d, tab]
            elif k == "mm":
                A, B = I.mm_inputs(size, first)
                dA, dB = _dev(A, device), _dev(B, device)
                self.host[k] = (A, B)
                o = np.arange(size, dtype=np.int64) * 4096
                self.dev[k] = (dA.data_ptr() + o, dB.data_ptr() + o)
                self.keep += [dA, dB]
            elif k == "fb":
                r, H, F = I.fb_inputs(size, first)
                dr, dH, dF = _dev(r, device), _dev(H, device), _dev(F, device)
                o = np.arange(size, dtype=np.int64)
                self.host[k] = (r, H, F)
                self.dev[k] = (dr.data_ptr() + o * 8192, dH.data_ptr() + o * 128, dF.data_ptr() + o * 128)
                self.keep += [dr, dH, dF]
            elif k == "bf":
                x, h, w = I.bf_inputs(size, first)
                dx_, dh, dw = _dev(x, device), _dev(h, device), _dev(w, device)
                o = np.arange(size, dtype=np.int64)
                self.host[k] = (x, h, w)
                self.dev[k] = (dx_.data_ptr() + o * x[0].nbytes, dh.data_ptr() + o * h[0].nbytes,
                               dw.data_ptr() + o * w[0].nbytes)
                self.keep += [dx_, dh, dw]
            elif k == "conv":
                img, kr, kc = I.conv_inputs(size, first)
                di, dkr, dkc = _dev(img, device), _dev(kr, device), _dev(kc, device)
                o = np.arange(size, dtype=np.int64)
                self.host[k] = (img, kr, kc)
                self.dev[k] = (di.data_ptr() + o * 65536, dkr.data_ptr() + o * 68, dkc.data_ptr() + o * 68)
                self.keep += [di, dkr, dkc]
            elif k == "dct":
                im, coef = I.dct_inputs(size, first), I.dct_coef()
                di, dco = _dev(im, device), _dev(coef, device)
                self.host[k] = (im, coef)
                self.dev[k] = (di.data_ptr() + np.arange(size, dtype=np.int64) * 65536, dco.data_ptr())
                self.keep += [di, dco]
            else:
                raise ValueError(k)

    def out_bytes(self, kind, j):
        if kind == "tdes":
            off = self.host["tdes"][1]
            return off[np.asarray(j) + 1] - off[np.asarray(j)]
        return np.full(np.shape(j), OUT_BYTES[kind], np.int64)

    def oracle_inputs(self, kind, j):
        """The host inputs of pool entry j (what the oracle is fed)."""
        h = self.host[kind]
        if kind == "mb":
            return int(h[0][j]), int(h[1][j])
        if kind == "tdes":
            flat, off = h
            return (flat[off[j]:off[j + 1]],)
        if kind == "dct":
            return h[0][j], h[1]
        return tuple(a[j] for a in h)


class PooledWorkload(Workload):
    """Tasks over an InputPool; outputs are read per task (task_output), since
    a full readback of config 5 is ~32 GB."""

    def __init__(self, name, pool, kinds, in_idx, shapes, args, out_buf, out_off, out_len, keep):
        self.pool, self.kinds, self.in_idx = pool, kinds, in_idx
        self.out_buf, self.out_off, self.out_len = out_buf, out_off, out_len
        super().__init__(name, shapes, args, {"kinds": kinds}, {}, keep, 0, int(out_len.sum()))

    def kind(self, k):
        return self.pool.kinds[self.kinds[k]]

    def task_output(self, k):
        kind = self.kind(k)
        raw = self.out_buf[int(self.out_off[k]):int(self.out_off[k] + self.out_len[k])].cpu().numpy()
        if kind == "mb":
            return raw.view(np.uint16).reshape(64, 64)
        if kind == "tdes":
            return raw
        if kind == "mm":
            return raw.view(np.float32).reshape(32, 32)
        if kind == "fb":
            return raw.view(np.float32)
        if kind == "bf":
            return raw.view(np.float32).reshape(4, 512)
        return raw.view(np.float32).reshape(128, 128)

    def outputs(self):
        raise NotImplementedError("pooled workloads are read per task: task_output(k)")


def pooled(name, pool: InputPool, kinds, in_idx, threads, shmem, device="cuda", resident=False, fill=None, n_tb=1):
    """kinds[i] indexes pool.kinds; in_idx[i] the pool entry; threads / shmem
    are used for FB, BF, CONV, DCT (MB, 3DES, MM take their configs' shapes).
    fill: byte value the output buffer is initialised with (None: left as
    allocated; tests pass one so stale results cannot pass for new ones)."""
    import torch
    n = len(kinds)
    kinds = np.asarray(kinds, np.int32)
    in_idx = np.asarray(in_idx, np.int64)
    shapes = np.zeros((n, 5), np.int32)
    shapes[:, 0], shapes[:, 1], shapes[:, 2] = threads, n_tb, shmem
    out_len = np.zeros(n, np.int64)
    scr_len = np.zeros(n, np.int64)
    for ki, k in enumerate(pool.kinds):
        i = np.nonzero(kinds == ki)[0]
        out_len[i] = pool.out_bytes(k, in_idx[i])
        scr_len[i] = SCRATCH_BYTES.get(k, 0) * n_tb   # FB / CONV: one scratch region per TB
        shapes[i, 3], shapes[i, 4] = SYNC[k], KIND_FUNC[k]
        if k == "mb":
            shapes[i, 0], shapes[i, 1], shapes[i, 2] = 128, 1, 0
        elif k == "tdes":
            shapes[i, 0], shapes[i, 1], shapes[i, 2] = 128, 1, (512 if resident else 2560)
        elif k == "mm":
            shapes[i, 0], shapes[i, 1], shapes[i, 2] = 256, 1, 8192
    span = (out_len + scr_len + _ALIGN - 1) // _ALIGN * _ALIGN
    base = np.zeros(n + 1, np.int64)
    np.cumsum(span, out=base[1:])
    buf = torch.empty(max(int(base[-1]), 16), dtype=torch.uint8, device=device)
    if fill is not None:
        buf.fill_(fill)
        torch.cuda.synchronize()
    out_ptr = buf.data_ptr() + base[:-1]
    scr_ptr = out_ptr + out_len
    raw = np.zeros((n, 40), np.uint8)
    for ki, k in enumerate(pool.kinds):
        i = np.nonzero(kinds == ki)[0]
        if len(i) == 0:
            continue
        j = in_idx[i]
        a = T.records(KIND_FUNC[k], len(i))
        d = pool.dev.get(k)
        if k == "mb":
            a["out"], a["x0"], a["y0"], a["dx"] = out_ptr[i], I.MB_X0, I.MB_Y0, I.MB_DX
            a["tx"], a["ty"], a["maxit"] = pool.host[k][0][j], pool.host[k][1][j], I.MB_MAXIT
        elif k == "tdes":
            a["inp"], a["out"], a["tables"], a["nblk"] = d[0][j], out_ptr[i], d[1], out_len[i] // 8
        elif k == "mm":
            a["A"], a["B"], a["C"] = d[0][j], d[1][j], out_ptr[i]
        elif k == "fb":
            a["r"], a["H"], a["F"], a["y"], a["scratch"] = d[0][j], d[1][j], d[2][j], out_ptr[i], scr_ptr[i]
        elif k == "bf":
            a["x"], a["h"], a["w"], a["out"] = d[0][j], d[1][j], d[2][j], out_ptr[i]
        elif k == "conv":
            a["img"], a["krow"], a["kcol"], a["out"], a["scratch"] = d[0][j], d[1][j], d[2][j], out_ptr[i], scr_ptr[i]
        elif k == "dct":
            a["img"], a["coef"], a["out"] = d[0][j], d[1], out_ptr[i]
        raw[i] = T.to_raw(a)
    w = PooledWorkload(name, pool, kinds, in_idx, shapes, raw, buf, base[:-1], out_len, [buf] + pool.keep)
    if "tdes" in pool.dev:
        w.tdes_tables = pool.dev["tdes"][1]
    if "dct" in pool.dev:
        w.dct_coef = pool.dev["dct"][1]
    return w


def mpe(n_tasks=32768, device="cuda", resident=False, fill=None):
    """NEXT-1 MPE: MB, 3DES (irregular 2-64 KiB packets), FB and
    MM, n/4 tasks each in a seeded order, each task its own input; FB runs 128
    threads with 1 KiB of shared memory."""
    kinds = I.mpe_schedule(n_tasks)
    pool = InputPool(I.MPE_KINDS, max(1, (n_tasks + 3) // 4), device, var_tdes=True)
    in_idx = np.zeros(n_tasks, np.int64)
    for ki in range(len(I.MPE_KINDS)):
        i = np.nonzero(kinds == ki)[0]
        in_idx[i] = np.arange(len(i))
    return pooled("mpe", pool, kinds, in_idx, 128, 1024, device, resident, fill)


def c5(n_tasks=1_000_000, device="cuda", resident=False, shard=(0, 1), pool_size=4096, fill=None, pool=None):
    """Config 5: 1M tasks, the kind of task i a seeded draw
    over the 7 bodies, task i uses pool entry i mod pool_size of its kind (the
    pool is replicated on every GPU).  shard = (rank, world): this GPU's
    contiguous block of task indices (strong scaling: the total stays 1M)."""
    kinds, thr, shm = I.c5_schedule(n_tasks)
    r, wsz = shard
    lo, hi = n_tasks * r // wsz, n_tasks * (r + 1) // wsz
    pool = pool or InputPool(I.C5_KINDS, pool_size, device)
    idx = np.arange(lo, hi, dtype=np.int64)
    w = pooled("c5", pool, kinds[lo:hi], idx % pool_size, thr[lo:hi], shm[lo:hi], device, resident, fill)
    w.first = lo
    return w


def tdes_var(n_tasks=32768, device="cuda", resident=False, fill=None):
    """NEXT-1 irregular 3DES: packets log-uniform 2-64 KiB (NetBench sizes,
    Table 3), one task of 128 threads each."""
    pool = InputPool(("tdes",), n_tasks, device, var_tdes=True)
    return pooled("tdes_var", pool, np.zeros(n_tasks, np.int32), np.arange(n_tasks), 128, 0, device, resident, fill)


def conv_only(n_tasks, device="cuda", threads=256, shmem=0, fill=None, n_tb=1):
    """CONV tasks alone (each its own 128x128 input), for the large-task sweep;
    n_tb thread blocks per task (a task larger than an MTB is spread)."""
    pool = InputPool(("conv",), n_tasks, device)
    return pooled("conv", pool, np.zeros(n_tasks, np.int32), np.arange(n_tasks), threads, shmem, device, fill=fill,
                  n_tb=n_tb)
