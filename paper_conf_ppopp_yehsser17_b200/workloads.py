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
    return Workload("tdes", _shapes(n_tasks, threads, 1, shmem, True, T.TDES), T.to_raw(a), host,
                    {"out": (out, np.uint8, (n_tasks, nbytes))}, [inp, out, tab], pk.nbytes, pk.nbytes)


# ---------------------------------------------------------------- config 3: MM
def matmul(n_tasks=65536, device="cuda", threads=256, shmem=8192, first=0):
    A, B = I.mm_inputs(n_tasks, first)
    dA, dB = _dev(A, device), _dev(B, device)
    dC = _zeros(A.nbytes, device)
    a = T.records(T.MM, n_tasks)
    off = np.arange(n_tasks) * 4096
    a["A"], a["B"], a["C"] = dA.data_ptr() + off, dB.data_ptr() + off, dC.data_ptr() + off
    return Workload("mm", _shapes(n_tasks, threads, 1, shmem, True, T.MM), T.to_raw(a), {"A": A, "B": B},
                    {"C": (dC, np.float32, (n_tasks, 32, 32))}, [dA, dB, dC], 2 * A.nbytes, A.nbytes)


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
    return Workload("mix", shapes, raw, host, outs, keep, in_b, out_b)


def nop(n_tasks, threads=128, n_tb=1, shmem=0, sync=False):
    return Workload("nop", _shapes(n_tasks, threads, n_tb, shmem, sync, T.NOP), np.zeros((n_tasks, 40), np.uint8),
                    {}, {}, [], 0, 0)
