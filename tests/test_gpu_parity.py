"""Parity: the CUDA path (through the C-ABI) against the oracle, element by
element, on the same seeded inputs.

Bar (BASELINE.json north star): bit-exact for integer tasks (Mandelbrot counts,
3DES ciphertext); fp32 tasks within rel = |g-o| / max(|o|, 1e-6 max|o|) <= 1e-5
elementwise.  The fp32 bodies fix their operation order on both sides, so they
are also expected to be bit-exact, and that is asserted too.

Sizes: the oracle-sized cases span several tiles / MTBs and ragged shapes; the
BASELINE.json full sizes run in the launch configuration bench.py times and are
checked on sampled tasks the oracle computes one by one (plus, for 3DES, every
packet against an independent library implementation).
"""
import numpy as np
import pytest

import oracle
from paper_conf_ppopp_yehsser17_b200 import inputs as I
from paper_conf_ppopp_yehsser17_b200 import workloads as W
from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, RESIDENT_TDES, Pagoda, naive_run
from paper_conf_ppopp_yehsser17_b200.presets import ctx_kwargs

pytestmark = pytest.mark.gpu

TOL = 1e-5


def fp32_close(g, o):
    g = np.asarray(g, np.float64)
    o = np.asarray(o, np.float64)
    den = np.maximum(np.abs(o), 1e-6 * np.abs(o).max())
    rel = np.abs(g - o) / den
    return rel.max()


def run(w, **cfg):
    with Pagoda(**cfg) as p:
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0
        assert p.info().device_error == 0
    return w.outputs()


# ---------------------------------------------------------------- MB (config 1)
# 2 and 1 MTBs per SM (32 / 64 registers per thread), spread-first claims, claim caps (max_tasks: 1 per
# MTB, and 2 per MTB at 1 MTB/SM = the bench preset)
MB_CFGS = [{}, {"mtbs_per_sm": 1, "arena_bytes": 96 * 1024}, {"flags": 0x10},   # 0x10: PAGODA_SPREAD
           {"mtbs_per_sm": 1, "arena_bytes": 96 * 1024, "flags": 0x10}, {"max_tasks": 1},
           ctx_kwargs("mb")]


@pytest.mark.parametrize("cfg", MB_CFGS)
def test_mandelbrot_config1_bit_exact(cfg):
    w = W.mandelbrot(1024)
    out = run(w, **cfg)["out"]
    for k in range(1024):
        ref = oracle.mandelbrot_tile(int(w.host["tx"][k]), int(w.host["ty"][k]))
        assert np.array_equal(out[k], ref), k
    assert int(out.astype(np.int64).sum()) == 199370695


@pytest.mark.parametrize("cfg", MB_CFGS)
@pytest.mark.parametrize("threads", [32, 100, 992])
def test_mandelbrot_other_thread_counts(threads, cfg):
    w = W.mandelbrot(96, threads=threads)
    out = run(w, **cfg)["out"]
    for k in range(0, 96, 7):
        assert np.array_equal(out[k], oracle.mandelbrot_tile(int(w.host["tx"][k]), int(w.host["ty"][k])))


# ---------------------------------------------------------------- 3DES (config 2)
def _tdes_ref(packet):
    return oracle.tdes_ecb(packet, I.TDES_KEYS)


@pytest.mark.parametrize("shmem,threads,resident", [(2560, 128, 0), (0, 128, 0), (2560, 96, 0), (2560, 32, 0),
                                                   (512, 128, 1), (0, 128, 1), (512, 32, 1), (2560, 256, 1)])
def test_tdes_small_bit_exact(shmem, threads, resident):
    w = W.tdes(48, shmem=shmem, threads=threads)
    cfg = {"flags": RESIDENT_TDES, "arena_bytes": 40 * 1024} if resident else {}
    out = run(w, **cfg)["out"]
    for k in range(48):
        assert np.array_equal(out[k], _tdes_ref(w.host["packets"][k])), k
    assert out[0, :24].tobytes().hex() == "a826fd8ce53b855fcce21c8112256fe668d5c05dd9b6b900"


@pytest.mark.parametrize("cfg", [{}, {"flags": RESIDENT_TDES, "arena_bytes": 40 * 1024},
                                 {"flags": RESIDENT_TDES, "mtbs_per_sm": 1, "arena_bytes": 128 * 1024}])
def test_tdes_config2_full_size(cfg):
    from cryptography.hazmat.decrepit.ciphers.algorithms import TripleDES
    from cryptography.hazmat.primitives.ciphers import Cipher, modes
    w = W.tdes(32768, shmem=512 if cfg else 2560)
    out = run(w, **cfg)["out"]
    pk = w.host["packets"]
    enc = Cipher(TripleDES(I.TDES_KEYS), modes.ECB()).encryptor()
    ref_all = np.frombuffer(enc.update(pk.tobytes()) + enc.finalize(), np.uint8).reshape(pk.shape)
    assert np.array_equal(out, ref_all)                    # every packet, independent library
    rng = np.random.default_rng(2)
    for k in list(rng.choice(32768, 24, replace=False)) + [0, 32767]:
        assert np.array_equal(out[k], _tdes_ref(pk[k])), k  # sampled, the oracle


# ---------------------------------------------------------------- MM (config 3)
def _mm_check(w, out, ks):
    for k in ks:
        ref = oracle.mm32(w.host["A"][k], w.host["B"][k])
        assert fp32_close(out[k], ref) <= TOL
        assert np.array_equal(out[k], ref), k


@pytest.mark.parametrize("shmem,threads", [(8192, 256), (0, 256), (8192, 64), (8192, 32), (4096, 1000 // 4)])
def test_mm_small(shmem, threads):
    w = W.matmul(300, shmem=shmem, threads=threads)
    _mm_check(w, run(w)["C"], range(300))


def _pool_map(fn, ks):
    """The oracle over many tasks on the host's cores (its ctypes calls release the GIL)."""
    import concurrent.futures as cf
    import os
    with cf.ThreadPoolExecutor(max_workers=min(16, os.cpu_count() or 1)) as ex:
        return list(ex.map(fn, ks, chunksize=256))


def test_mm_config3_full_size():
    """Every one of the 65,536 tasks against the oracle, in the bench's launch configuration."""
    w = W.matmul(65536)
    out = run(w, **ctx_kwargs("mm"))["C"]   # the bench's launch configuration
    A, B = w.host["A"], w.host["B"]
    ref = np.stack(_pool_map(lambda k: oracle.mm32(A[k], B[k]), range(65536)))
    assert fp32_close(out, ref) <= TOL
    bad = np.nonzero((out != ref).reshape(65536, -1).any(axis=1))[0]
    assert len(bad) == 0, bad[:10]


# ---------------------------------------------------------------- MM on the tensor cores (NEXT-4, 3xTF32)
def _mm_tc_check(w, out, ks):
    for k in ks:
        a, b = w.host["A"][k].astype(np.float64), w.host["B"][k].astype(np.float64)
        ref = oracle.mm32_exact(w.host["A"][k], w.host["B"][k]).astype(np.float64)
        bound = TOL * (np.abs(a) @ np.abs(b))      # normwise: the summation order is the hardware's
        assert (np.abs(out[k].astype(np.float64) - ref) <= bound).all(), k


@pytest.mark.parametrize("shmem,threads", [(8192, 256), (0, 256), (8192, 64), (8192, 32), (0, 96)])
def test_mm_tc_small(shmem, threads):
    from paper_conf_ppopp_yehsser17_b200 import tasks as T
    w = W.matmul(300, shmem=shmem, threads=threads, func=T.MM_TC)
    _mm_tc_check(w, run(w)["C"], range(300))


def test_mm_tc_integer_exact_and_full_size():
    from paper_conf_ppopp_yehsser17_b200 import tasks as T
    w = W.matmul(64, func=T.MM_TC, integer=True)    # integer inputs: every partial sum exact in fp32
    out = run(w)["C"]
    for k in range(64):
        assert np.array_equal(out[k], oracle.mm32_exact(w.host["A"][k], w.host["B"][k])), k
    w = W.matmul(65536, func=T.MM_TC)
    out = run(w, **ctx_kwargs("mm_tc"))["C"]   # the bench's launch configuration
    rng = np.random.default_rng(5)
    _mm_tc_check(w, out, list(rng.choice(65536, 256, replace=False)) + [0, 65535])


# ---------------------------------------------------------------- DCT with / without shmem (Table 5, NEXT-4)
def _dct_check(w, out, ks):
    for k in ks:
        ref = oracle.dct(w.host["img"][k], w.host["coef"])
        assert fp32_close(out[k], ref) <= TOL and np.array_equal(out[k], ref), k


# (threads, n_tb, shmem, sync): one band of 16 block rows; bands of 4, 3 (ragged last band: 16 = 5*3 + 1)
# and 1 block row; several TBs sharing the bands (more TBs than bands too); 1-warp TBs without a
# barrier (canSync by construction); no shmem; a grant below one block row (global path)
DCT_SHAPES = [(64, 1, 16384, True), (64, 1, 65536, True), (128, 1, 12288, True), (32, 1, 4096, False),
              (96, 3, 8192, True), (64, 20, 4096, True), (64, 1, 0, False), (256, 1, 2048, True)]


@pytest.mark.parametrize("threads,n_tb,shmem,sync", DCT_SHAPES)
def test_dct_table5_small(threads, n_tb, shmem, sync):
    w = W.dct(200, threads=threads, n_tb=n_tb, shmem=shmem, sync=sync)
    _dct_check(w, run(w, arena_bytes=96 * 1024)["out"], range(200))


@pytest.mark.parametrize("name", ["dct", "dct_noshm"])
def test_dct_table5_full_size(name):
    w = W.dct(32768, shmem=8192 if name == "dct" else 0, sync=name == "dct")
    kw = ctx_kwargs(name, NO_START)           # the bench's launch configuration, registered coefficients
    with Pagoda(**kw) as p:
        p.dct_register(w.dct_coef)
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert p.stop() == 0
        p.dct_register(None)
    out = w.outputs()["out"]
    rng = np.random.default_rng(11)
    _dct_check(w, out, list(rng.choice(32768, 96, replace=False)) + [0, 32767])


@pytest.mark.parametrize("shmem,sync", [(8192, True), (0, False)])
def test_dct_registered_coefficients(shmem, sync):
    """pagoda_dct_register: tasks with the registered coef pointer read the constant-bank copy
    (bit-identical outputs); another coef buffer with the same values takes the load path."""
    w = W.dct(300, shmem=shmem, sync=sync)
    w2 = W.dct(100, shmem=shmem, sync=sync, first=300)   # its own coef buffer (a different pointer)
    with Pagoda(flags=NO_START, arena_bytes=96 * 1024) as p:
        p.dct_register(w.dct_coef)
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        p.spawn_shapes(w2.shapes, w2.args)
        assert p.waitAll() == 0
        assert p.stop() == 0
        p.dct_register(None)
    _dct_check(w, w.outputs()["out"], range(300))
    _dct_check(w2, w2.outputs()["out"], range(100))


def test_dct_table5_naive_baseline():
    w = W.dct(300, threads=64, shmem=16384)
    naive_run(0, w.shapes, w.args, 32)
    _dct_check(w, w.outputs()["out"], range(300))


def _mm64_check(w, out, ks):
    for k in ks:
        ref = oracle.mm64(w.host["A"][k], w.host["B"][k])
        assert fp32_close(out[k], ref) <= TOL and np.array_equal(out[k], ref), k


# staged (32 KiB, sync), global (no shmem), threads not a multiple of 64 (own column per item),
# 1-warp TBs (stage both operands), a grant below 32 KiB (global path), 1024 threads
@pytest.mark.parametrize("shmem,threads,sync", [(32768, 256, True), (0, 256, False), (32768, 96, True),
                                                (32768, 32, False), (16384, 128, True), (32768, 1024, True)])
def test_mm64_small(shmem, threads, sync):
    w = W.matmul64(150, shmem=shmem, threads=threads)
    w.shapes[:, 3] = int(sync)
    _mm64_check(w, run(w, arena_bytes=96 * 1024)["C"], range(150))


def test_mm64_integer_exact_naive_and_full_size():
    w = W.matmul64(40, integer=True)    # integer inputs: every partial sum exact in fp32
    out = run(w, arena_bytes=96 * 1024)["C"]
    for k in range(40):
        assert np.array_equal(out[k].astype(np.int64), w.host["A"][k].astype(np.int64) @ w.host["B"][k].astype(np.int64))
    w = W.matmul64(200)
    naive_run(0, w.shapes, w.args, 32)
    _mm64_check(w, w.outputs()["C"], range(200))
    w = W.matmul64(32768)
    out = run(w, **ctx_kwargs("mm64"))["C"]   # the bench's launch configuration
    rng = np.random.default_rng(17)
    _mm64_check(w, out, list(rng.choice(32768, 96, replace=False)) + [0, 32767])


def test_mm_noshm_full_size():
    w = W.matmul(65536, shmem=0)
    out = run(w, **ctx_kwargs("mm_noshm"))["C"]
    rng = np.random.default_rng(13)
    _mm_check(w, out, list(rng.choice(65536, 128, replace=False)) + [0, 65535])


# ---------------------------------------------------------------- mix (config 4)
def _mix_check(w, out, frac=1.0, seed=0):
    rng = np.random.default_rng(seed)

    def pick(n):
        return range(n) if frac >= 1 else rng.choice(n, max(1, int(n * frac)), replace=False)

    r, H, F = w.host["fb"]
    for k in pick(len(r)):
        ref = oracle.filterbank(r[k], H[k], F[k])
        assert fp32_close(out["fb"][k], ref) <= TOL and np.array_equal(out["fb"][k], ref), ("fb", k)
    x, h, ww = w.host["bf"]
    for k in pick(len(x)):
        ref = oracle.beamformer(x[k], h[k], ww[k])
        assert fp32_close(out["bf"][k], ref) <= TOL and np.array_equal(out["bf"][k], ref), ("bf", k)
    img, kr, kc = w.host["conv"]
    for k in pick(len(img)):
        ref = oracle.conv(img[k], kr[k], kc[k])
        assert fp32_close(out["conv"][k], ref) <= TOL and np.array_equal(out["conv"][k], ref), ("conv", k)
    im, coef = w.host["dct"]
    for k in pick(len(im)):
        ref = oracle.dct(im[k], coef)
        assert fp32_close(out["dct"][k], ref) <= TOL and np.array_equal(out["dct"][k], ref), ("dct", k)


def test_mix_small_all_shapes():
    w = W.mix(160)     # threads 32..512, shmem 0..48 KiB, ragged per task
    _mix_check(w, run(w))


def test_mix_config4_full_size_every_task():
    """Every one of the 32,768 FB / BF / CONV / DCT tasks against the oracle, in the bench's launch
    configuration (the oracle on the host's cores)."""
    w = W.mix(32768)
    out = run(w, **ctx_kwargs("mix"))
    fns = {"fb": (oracle.filterbank, w.host["fb"]), "bf": (oracle.beamformer, w.host["bf"]),
           "conv": (oracle.conv, w.host["conv"]), "dct": (oracle.dct, None)}
    for kind, (fn, ins) in fns.items():
        if kind == "dct":
            im, coef = w.host["dct"]
            ref = np.stack(_pool_map(lambda k: oracle.dct(im[k], coef), range(len(im))))
        else:
            ref = np.stack(_pool_map(lambda k: fn(*(x[k] for x in ins)), range(len(ins[0]))))
        got = out[kind].reshape(ref.shape)
        assert fp32_close(got, ref) <= TOL, kind
        bad = np.nonzero((got != ref).reshape(len(ref), -1).any(axis=1))[0]
        assert len(bad) == 0, (kind, bad[:10])


def test_mix_config4_registered_coefficients():
    """The bench's launch configuration: config 4 with its DCT coefficients registered."""
    w = W.mix(32768)
    with Pagoda(**ctx_kwargs("mix", NO_START)) as p:
        p.dct_register(w.dct_coef)
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert p.stop() == 0
        p.dct_register(None)
    _mix_check(w, w.outputs(), frac=0.004, seed=6)


# ---------------------------------------------------------------- the naive baseline runs the same bodies
def test_naive_baseline_parity():
    w = W.mandelbrot(64)
    naive_run(0, w.shapes, w.args, 32)
    out = w.outputs()["out"]
    for k in range(0, 64, 5):
        assert np.array_equal(out[k], oracle.mandelbrot_tile(int(w.host["tx"][k]), int(w.host["ty"][k])))
    w = W.mix(40)
    naive_run(0, w.shapes, w.args, 32)
    _mix_check(w, w.outputs())
    w = W.tdes(16)
    naive_run(0, w.shapes, w.args, 32)
    out = w.outputs()["out"]
    for k in range(16):
        assert np.array_equal(out[k], _tdes_ref(w.host["packets"][k]))


# ---------------------------------------------------------------- static fusion (NEXT-2) runs the same bodies
def test_static_fusion_parity():
    from paper_conf_ppopp_yehsser17_b200.pagoda import PagodaError, fused_run
    w = W.mix(120)
    ns, ms = fused_run(0, w.shapes, w.args, 256)
    assert ns > 0 and ms > 0
    _mix_check(w, w.outputs())
    w = W.tdes(40)
    fused_run(0, w.shapes, w.args, 64)
    out = w.outputs()["out"]
    for k in range(40):
        assert np.array_equal(out[k], _tdes_ref(w.host["packets"][k]))
    w = W.mandelbrot(64)
    fused_run(0, w.shapes, w.args, 256)
    out = w.outputs()["out"]
    for k in range(64):
        assert np.array_equal(out[k], oracle.mandelbrot_tile(int(w.host["tx"][k]), int(w.host["ty"][k])))
    w = W.matmul(50)
    fused_run(0, w.shapes, w.args, 256)
    _mm_check(w, w.outputs()["C"], range(50))
    bad = w.shapes.copy()
    bad[3, 1] = 2   # multi-block tasks cannot be fused one block per task
    with pytest.raises(PagodaError):
        fused_run(0, bad, w.args, 256)


# ---------------------------------------------------------------- 3DES with registered (constant-bank) round keys
@pytest.mark.parametrize("threads", [128, 96, 32, 256])
def test_tdes_registered_keys(threads):
    """Resident SP tables + the registered key schedule: tasks using the
    registered tables take no shared memory for keys; tasks with another
    tables buffer (same key) still stage theirs; both bit-exact."""
    w = W.tdes(64, shmem=512, threads=threads)
    w2 = W.tdes(16, shmem=512, threads=threads, first=64)   # its own tables buffer: not registered
    with Pagoda(flags=RESIDENT_TDES | NO_START, arena_bytes=40 * 1024) as p:
        p.tdes_register(w.tdes_tables)
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        p.spawn_shapes(w2.shapes, w2.args)
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert p.stop() == 0
        p.tdes_register(None)
    for ww in (w, w2):
        out = ww.outputs()["out"]
        for k in range(ww.n):
            assert np.array_equal(out[k], _tdes_ref(ww.host["packets"][k])), k


def test_tdes_registered_keys_full_size():
    from cryptography.hazmat.decrepit.ciphers.algorithms import TripleDES
    from cryptography.hazmat.primitives.ciphers import Cipher, modes
    w = W.tdes(32768, shmem=512)
    with Pagoda(flags=RESIDENT_TDES | NO_START, arena_bytes=40 * 1024) as p:
        p.tdes_register(w.tdes_tables)
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        assert p.waitAll() == 0 and p.info().device_error == 0
        assert p.stop() == 0
        p.tdes_register(None)
    out = w.outputs()["out"]
    pk = w.host["packets"]
    enc = Cipher(TripleDES(I.TDES_KEYS), modes.ECB()).encryptor()
    ref = np.frombuffer(enc.update(pk.tobytes()) + enc.finalize(), np.uint8).reshape(pk.shape)
    assert np.array_equal(out, ref)
    for k in (0, 1, 16383, 32767):
        assert np.array_equal(out[k], _tdes_ref(pk[k]))


# ---------------------------------------------------------------- two scheduling groups per MTB
@pytest.mark.parametrize("wl", ["tdes", "mm", "mix"])
def test_two_scheduling_groups_parity(wl):
    """pagoda_config.sched_groups = 2 (two token holders per MTB, each with half the warps, task
    slots, TB records, arena and named barriers): full-size 3DES (resident tables shared by both
    groups) and sampled MM / mix tasks match the oracle."""
    import oracle
    from paper_conf_ppopp_yehsser17_b200 import inputs as I
    from paper_conf_ppopp_yehsser17_b200 import workloads as W
    from paper_conf_ppopp_yehsser17_b200.pagoda import NO_START, RESIDENT_TDES, Pagoda
    if wl == "tdes":
        w = W.tdes(32768, shmem=512)
        cfg = dict(flags=RESIDENT_TDES | NO_START, arena_bytes=40 * 1024)
    elif wl == "mm":
        w = W.matmul(16384)
        cfg = dict(flags=NO_START)
    else:
        w = W.mix(2048)
        cfg = dict(flags=NO_START, mtbs_per_sm=1, arena_bytes=200 * 1024)
    with Pagoda(sched_groups=2, **cfg) as p:
        assert p.info().sched_groups == 2
        if wl == "tdes":
            p.tdes_register(w.tdes_tables)
        assert p.start() == 0
        p.spawn_shapes(w.shapes, w.args)
        assert p.stop() == 0 and p.info().device_error == 0
    out = w.outputs()
    if wl == "tdes":
        for k in list(range(0, 32768, 509)) + [32767]:
            assert np.array_equal(out["out"][k], oracle.tdes_ecb(w.host["packets"][k], I.TDES_KEYS)), k
    elif wl == "mm":
        for k in range(0, 16384, 97):
            assert np.array_equal(out["C"][k], oracle.mm32(w.host["A"][k], w.host["B"][k])), k
    else:
        kinds = w.host["kinds"]
        for kind, fn in (("fb", oracle.filterbank), ("bf", oracle.beamformer), ("conv", oracle.conv),
                         ("dct", oracle.dct)):
            idx = np.nonzero(kinds == I.MIX_KINDS.index(kind))[0]
            for j in range(0, len(idx), 37):
                args = [a[j] for a in w.host[kind]] if kind != "dct" else [w.host[kind][0][j], w.host[kind][1]]
                assert np.array_equal(out[kind][j], fn(*args)), (kind, j)
