"""Parity of the pooled multi-body workloads through the C-ABI against the
oracle: NEXT-1 (irregular 3DES packets, the MPE mix) and
config 5 (1M mixed tasks over the 7 bodies).

Bar as in test_gpu_parity.py: integer outputs bit-exact, fp32 within 1e-5
relative and bit-exact (both sides fix the operation order).  Output buffers
are pre-filled with 0xAB so a task that never ran cannot pass.
"""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_yehsser17_b200 import inputs as I
from paper_conf_ppopp_yehsser17_b200 import workloads as W
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, RESIDENT_TDES, Pagoda

pytestmark = pytest.mark.gpu

TOL = 1e-5


def ref_of(w, k):
    kind = w.kind(k)
    args = w.pool.oracle_inputs(kind, int(w.in_idx[k]))
    if kind == "mb":
        return oracle.mandelbrot_tile(*args)
    if kind == "tdes":
        return oracle.tdes_ecb(args[0], I.TDES_KEYS)
    return {"mm": oracle.mm32, "fb": oracle.filterbank, "bf": oracle.beamformer, "conv": oracle.conv,
            "dct": oracle.dct}[kind](*args)


def check_tasks(w, ks):
    seen = set()
    for k in ks:
        k = int(k)
        g, o = w.task_output(k), ref_of(w, k)
        if o.dtype.kind == "f":
            den = np.maximum(np.abs(o.astype(np.float64)), 1e-6 * np.abs(o).max())
            assert (np.abs(g.astype(np.float64) - o) / den).max() <= TOL, (w.kind(k), k)
        assert np.array_equal(g, o), (w.kind(k), k)
        seen.add(w.kind(k))
    return seen


def run(w, **cfg):
    with Pagoda(**cfg) as p:
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0
        assert p.info().device_error == 0


RES = {"flags": RESIDENT_TDES, "arena_bytes": 40 * 1024}


# ---------------------------------------------------------------- irregular 3DES (NEXT-1)
@pytest.mark.parametrize("resident", [False, True])
def test_tdes_var_small_bit_exact(resident):
    w = W.tdes_var(200, resident=resident, fill=0xAB)
    run(w, **(RES if resident else {}))
    check_tasks(w, range(200))
    assert w.task_output(0)[:24].tobytes().hex() == "a826fd8ce53b855fcce21c8112256fe668d5c05dd9b6b900"


def test_tdes_var_full_size():
    """All 32768 irregular packets (2-64 KiB, 600 MB) against an independent
    library implementation; a sample against the oracle."""
    from cryptography.hazmat.decrepit.ciphers.algorithms import TripleDES
    from cryptography.hazmat.primitives.ciphers import Cipher, modes
    w = W.tdes_var(32768, resident=True, fill=0xAB)
    run(w, **RES)
    flat, off = w.pool.host["tdes"]
    enc = Cipher(TripleDES(I.TDES_KEYS), modes.ECB()).encryptor()
    ref = np.frombuffer(enc.update(flat.tobytes()) + enc.finalize(), np.uint8)
    buf = w.out_buf.cpu().numpy()   # outputs are bump-allocated (256 B aligned), in task order
    for k in range(32768):
        o = int(w.out_off[k])
        assert np.array_equal(buf[o:o + int(w.out_len[k])], ref[off[k]:off[k + 1]]), k
    rng = np.random.default_rng(11)
    check_tasks(w, list(rng.choice(32768, 12, replace=False)) + [0, 32767])


# ---------------------------------------------------------------- MPE (NEXT-1)
def test_mpe_small_all_tasks():
    w = W.mpe(240, fill=0xAB)
    run(w)
    assert check_tasks(w, range(240)) == set(I.MPE_KINDS)


def test_mpe_full_size_sampled():
    w = W.mpe(32768, resident=True, fill=0xAB)
    run(w, **RES)
    rng = np.random.default_rng(12)
    assert check_tasks(w, list(rng.choice(32768, 300, replace=False)) + [0, 32767]) == set(I.MPE_KINDS)


# ---------------------------------------------------------------- config 5
@pytest.mark.parametrize("cfg", [{}, {"flags": RESIDENT_TDES, "mtbs_per_sm": 1, "arena_bytes": 144 * 1024}])
def test_c5_small_all_tasks(cfg):
    w = W.c5(2000, pool_size=64, resident=bool(cfg), fill=0xAB)
    run(w, **cfg)
    assert check_tasks(w, range(2000)) == set(I.C5_KINDS)


def test_c5_full_size_sampled():
    """The bench's N=1 launch configuration: 1M tasks on one GPU."""
    w = W.c5(1_000_000, resident=True, fill=0xAB)
    with Pagoda(flags=RESIDENT_TDES | NO_START, mtbs_per_sm=1, arena_bytes=144 * 1024) as p:
        p.dct_register(w.dct_coef)       # as bench.py: the pool's DCT coefficients registered
        assert p.start() == 0
        ids = p.spawn_shapes(w.shapes, w.args, ids=True)
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert np.array_equal(ids, np.arange(1_000_000))
        assert p.info().completed_low == 1_000_000
    rng = np.random.default_rng(13)
    ks = list(rng.choice(1_000_000, 350, replace=False)) + [0, 999_999]
    assert check_tasks(w, ks) == set(I.C5_KINDS)


def test_c5_shards_partition_the_tasks():
    """Strong scaling shards: ranks' blocks are disjoint and cover all tasks,
    and a shard's task k is global task first + k (same kind, same input)."""
    pool = W.InputPool(I.C5_KINDS, 64)
    full = W.c5(1000, pool_size=64, pool=pool)
    parts = [W.c5(1000, pool_size=64, shard=(r, 3), pool=pool) for r in range(3)]
    assert sum(p.n for p in parts) == 1000
    assert [p.first for p in parts] == [0, 333, 666]
    for p in parts:
        assert np.array_equal(p.kinds, full.kinds[p.first:p.first + p.n])
        assert np.array_equal(p.in_idx, full.in_idx[p.first:p.first + p.n])
        assert np.array_equal(p.shapes, full.shapes[p.first:p.first + p.n])


# ---------------------------------------------------------------- large tasks spread over MTBs (NEXT-3)
@pytest.mark.parametrize("threads,n_tb,shmem", [(1024, 16, 0), (512, 8, 48 * 1024), (256, 3, 4096)])
def test_conv_large_tasks(threads, n_tb, shmem):
    """CONV with up to 16384 threads per task (16 TBs spread over MTBs; each TB
    computes the row pass its own outputs need, Fig. 8's large tasks)."""
    w = W.conv_only(12, threads=threads, shmem=shmem, fill=0xAB, n_tb=n_tb)
    assert (w.shapes[:, 1] == n_tb).all()
    run(w)
    assert check_tasks(w, range(12)) == {"conv"}

