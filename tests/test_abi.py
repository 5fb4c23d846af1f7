"""CPU-only checks of the product library: it builds, loads, exports every
symbol include/*.h declares, and its host-only logic is right (no compute
calls that need a GPU)."""
import ctypes as C
import errno
import os
import re

import numpy as np
import pytest

from conftest import ROOT

import paper_conf_ppopp_yehsser17_b200.pagoda as PG
from paper_conf_ppopp_yehsser17_b200 import inputs as I
from paper_conf_ppopp_yehsser17_b200 import tasks as T


@pytest.fixture(scope="module")
def L():
    from paper_conf_ppopp_yehsser17_b200 import build
    build.build()
    return PG.lib()


def declared_functions():
    src = open(os.path.join(ROOT, "include", "pagoda.h")).read()
    src = re.sub(r"/\*.*?\*/", "", src, flags=re.S)
    return sorted(set(re.findall(r"\b(pagoda_\w+)\s*\(", src)))


def test_exports_every_declared_symbol(L):
    names = declared_functions()
    assert len(names) >= 24
    for n in names:
        assert hasattr(L, n), n


def test_no_oracle_in_product():
    pkg = os.path.join(ROOT, "paper_conf_ppopp_yehsser17_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cuh", ".h", ".cpp")):
                s = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in s and "from oracle" not in s and "oracle.h" not in s, f


def test_config_default(L):
    c = PG.default_config()
    assert (c.mtbs_per_sm, c.ring_entries, c.comp_entries, c.arena_bytes, c.exec_warps) == (2, 65536, 1 << 20,
                                                                                          96 * 1024, 32)


def test_init_without_gpu_fails_loudly(L):
    import torch
    if torch.cuda.is_available():
        pytest.skip("GPU present")
    h = C.c_void_p()
    rc = L.pagoda_init(None, C.byref(h))
    assert rc == -errno.ENODEV
    with pytest.raises(PG.PagodaError):
        PG.Pagoda()


def test_picker_rule(L):
    assert PG.pick_least_loaded([5, 3, 3, 9]) == 1
    assert PG.pick_least_loaded([0]) == 0
    assert PG.pick_least_loaded([7, 7, 7]) == 0
    assert L.pagoda_pick_least_loaded(None, 0) == -errno.EINVAL


def test_pool_claim_rule(L):
    """A pool member claims the next run of tasks only while it is within `slack` warps of
    the least-loaded member (SURVEY §8(e) least-loaded-first)."""
    assert PG.pool_may_claim([10, 3, 7], 1, 0) == 1           # the least loaded always may
    assert PG.pool_may_claim([10, 3, 7], 2, 0) == 0
    assert PG.pool_may_claim([10, 3, 7], 2, 4) == 1           # within slack
    assert PG.pool_may_claim([5, 5], 0, 0) == 1 and PG.pool_may_claim([5, 5], 1, 0) == 1   # ties: both
    assert PG.pool_may_claim([5], 0, 0) == 1
    assert L.pagoda_pool_may_claim(None, 0, 0, 0) == -errno.EINVAL
    assert PG.pool_may_claim([1, 2], 2, 0) == -errno.EINVAL


def test_args_layouts_fit_the_entry():
    for f, d in T.ARGS.items():
        assert d.itemsize <= 40
    assert T.ARGS[T.MB].itemsize == 32 and T.ARGS[T.TDES].itemsize == 32 and T.ARGS[T.FB].itemsize == 40


# --------------------------------------------------------------- 3DES tables
def _perm_bytes(t, x):
    r = 0
    for b in range(8):
        r |= int(t[b, (x >> (56 - 8 * b)) & 0xFF])
    return r


def _swap(a, b, n, m):     # tdes_swap in csrc/bodies.cuh
    t = ((a >> n) ^ b) & m
    return a ^ ((t << n) & 0xFFFFFFFF), b ^ t


def _ip_swaps(l, r):       # tdes_ip
    l, r = _swap(l, r, 4, 0x0F0F0F0F)
    l, r = _swap(l, r, 16, 0x0000FFFF)
    r, l = _swap(r, l, 2, 0x33333333)
    r, l = _swap(r, l, 8, 0x00FF00FF)
    l, r = _swap(l, r, 1, 0x55555555)
    return l, r


def _fp_swaps(l, r):       # tdes_fp
    l, r = _swap(l, r, 1, 0x55555555)
    r, l = _swap(r, l, 8, 0x00FF00FF)
    r, l = _swap(r, l, 2, 0x33333333)
    l, r = _swap(l, r, 16, 0x0000FFFF)
    l, r = _swap(l, r, 4, 0x0F0F0F0F)
    return l, r


def test_ip_fp_swap_networks_equal_the_product_tables(L):
    """The body's register-only IP/FP equal the table-driven permutations
    (FIPS 46-3 IP and IP^-1) the product also ships, and invert each other."""
    tab = PG.tdes_tables(bytes(range(24)))
    ipt = tab[2432:2432 + 16384].view(np.uint64).reshape(8, 256)
    fpt = tab[2432 + 16384:].view(np.uint64).reshape(8, 256)
    rng = np.random.default_rng(7)
    blocks = [int(v) for v in rng.integers(0, 2 ** 63, 300, dtype=np.int64)] + [0, 2 ** 64 - 1, 1, 2 ** 63]
    blocks += [1 << k for k in range(64)]
    for x in blocks:
        l, r = _ip_swaps(x >> 32, x & 0xFFFFFFFF)
        assert (l << 32) | r == _perm_bytes(ipt, x)
        l2, r2 = _fp_swaps(x >> 32, x & 0xFFFFFFFF)
        assert (l2 << 32) | r2 == _perm_bytes(fpt, x)
        assert _fp_swaps(l, r) == (x >> 32, x & 0xFFFFFFFF)


def _des_with_product_tables(tab: np.ndarray, block: int) -> int:
    """Run the GPU body's round structure on the CPU with the product's tables
    (same index arithmetic as body_tdes in csrc/bodies.cuh)."""
    sp = tab[:2048].view(np.uint32).reshape(8, 64)
    keys = tab[2048:2432].view(np.uint32).reshape(48, 2)

    def rotl(x, s):   # __funnelshift_l(x, x, s) takes s mod 32
        s %= 32
        return ((x << s) | (x >> (32 - s))) & 0xFFFFFFFF

    l, r = _ip_swaps(block >> 32, block & 0xFFFFFFFF)
    for st in range(3):
        for rd in range(16):
            kx, ky = (int(v) for v in keys[st * 16 + rd])
            x = rotl(r, 5) ^ kx          # bytes 0..3: inputs of S-boxes 0, 6, 4, 2
            y = rotl(r, 1) ^ ky          # bytes 0..3: inputs of S-boxes 7, 5, 3, 1
            f = 0
            for b, (jx, jy) in enumerate(zip((0, 6, 4, 2), (7, 5, 3, 1))):
                f ^= int(sp[jx, (x >> 8 * b) & 63]) ^ int(sp[jy, (y >> 8 * b) & 63])
            l, r = r, l ^ f
        l, r = r, l
    l, r = _fp_swaps(l, r)
    return (l << 32) | r


def test_tdes_tables_reproduce_known_answers(L):
    from conftest import read_golden
    for key, pt, ct in read_golden("tdes_kat.txt"):
        tab = PG.tdes_tables(bytes.fromhex(key))
        assert len(tab) == T.TDES_TABLE_BYTES
        p, c = bytes.fromhex(pt), bytes.fromhex(ct)
        for b in range(0, len(p), 8):
            got = _des_with_product_tables(tab, int.from_bytes(p[b:b + 8], "big"))
            assert got == int.from_bytes(c[b:b + 8], "big")


def test_inputs_generator_is_deterministic_and_exact():
    a = I.splitmix64([0, 1, 2], 4)
    b = I.splitmix64([0, 1, 2], 4)
    assert np.array_equal(a, b) and a.dtype == np.uint64
    # reference value of the splitmix64 step for state = seed ^ 0: first output
    s = (0x5EED + 0x9E3779B97F4A7C15) & (2 ** 64 - 1)
    z = ((s ^ (s >> 30)) * 0xBF58476D1CE4E5B9) & (2 ** 64 - 1)
    z = ((z ^ (z >> 27)) * 0x94D049BB133111EB) & (2 ** 64 - 1)
    assert int(a[0, 0]) == z ^ (z >> 31)
    f = I.to_f32(a)
    assert (f >= -1).all() and (f < 1).all()
    assert np.array_equal(f.astype(np.float64) * 2 ** 23, np.round(f.astype(np.float64) * 2 ** 23))
    k, th, sh = I.mix_schedule(400)
    assert np.bincount(k).tolist() == [100] * 4
    assert set(th) <= set(I.MIX_THREADS) and set(sh // 1024) <= set(I.MIX_SHMEM_KB)
