/*
 * bodies.cuh — the task bodies, written once as __device__ subroutines over an
 * Env (pagoda_device.cuh) and instantiated twice: inside the MasterKernel
 * (TaskEnv) and as the naive one-launch-per-task baseline (NativeEnv).
 *
 * What each body computes is DESIGN.md "Task bodies" (the paper gives the
 * benchmark names and sizes only: Tables 3-4).  fp32 bodies use
 * explicitly rounded intrinsics (__fmul_rn / __fadd_rn / __fmaf_rn) so that
 * nvcc cannot contract or reorder: the operation order is the definition's.
 *
 * Work partition: thread getTid() of a task with T = n_tb * warps_tb * 32
 * threads (idle padding lanes included) takes output items getTid(), +T, ...
 * Bodies with two dependent passes (FB, CONV) keep each thread block
 * self-contained: a TB computes the intermediate values its own outputs need,
 * into its own shared memory or scratch region, and only syncBlock()s itself.
 */
#ifndef PAGODA_BODIES_CUH
#define PAGODA_BODIES_CUH
#include <stdint.h>

#include "pagoda_device.cuh"
#include "pagoda_tasks.h"

namespace pagoda {

/* Benchmark bodies as calls (PAGODA_BODIES_NOINLINE): a body inlined into the executor loop shares
 * its register allocation, and at 32 registers per thread (2 or 4 MTBs per SM) every inlined body
 * adds spills around all of them (3DES as a call: 3DES +1.6 %, MM +6 %, MPE +8 %). */
#ifndef PAGODA_BODIES_NOINLINE
#define PAGODA_BODIES_NOINLINE 0
#endif
#if PAGODA_BODIES_NOINLINE
#define PAGODA_BODY_ATTR __noinline__
#else
#define PAGODA_BODY_ATTR
#endif
#if PAGODA_BODIES_NOINLINE
#define PAGODA_CONV_BODY_ATTR __noinline__
#else
#define PAGODA_CONV_BODY_ATTR __forceinline__
#endif

template <class Env>
__device__ __forceinline__ int total_threads(const Env& e)
{
    return e.getNumBlocks() * e.getBlockWarps() * 32;
}
template <class Env>
__device__ __forceinline__ int tb_threads(const Env& e)
{
    return e.getBlockWarps() * 32;
}

/* ------------------------------------------------------------- test bodies */
template <class Env>
__device__ void body_mark(const Env& e, const pagoda_mark_args& a)
{
    if (e.getBlockTid() < e.getBlockDim()) {
        a.out[a.base + (uint32_t)e.getTid()] = a.tag;
        atomicAdd(a.cnt, 1u);
    }
}

template <class Env>
__device__ void body_tid(const Env& e, const pagoda_tid_args& a)
{
    if (e.getBlockTid() < e.getBlockDim())
        a.out[a.base + (uint32_t)e.getTid()] = ((uint32_t)e.getBlockIdx() << 16) | (uint32_t)e.getBlockTid();
}

/* P phases of: write my word, syncBlock, read the word of the thread 32 lanes
 * further on (another warp of the same TB), syncBlock.  Scratch: shared memory
 * if granted, else args.scratch[tb * threads_tb_rounded + ...]. */
template <class Env>
__device__ void body_bar(const Env& e, const pagoda_bar_args& a)
{
    const int n = tb_threads(e), bt = e.getBlockTid();
    volatile uint32_t* buf = (e.getSMBytes() >= (uint32_t)n * 4u)
                                 ? reinterpret_cast<volatile uint32_t*>(e.getSMPtr())
                                 : reinterpret_cast<volatile uint32_t*>(a.scratch) + e.getBlockIdx() * n;
    uint32_t errs = 0;
    for (uint32_t p = 0; p < a.phases; p++) {
        buf[bt] = p * 1000003u + (uint32_t)bt;
        e.syncBlock();
        int nb = (bt + 32) % n;
        if (buf[nb] != p * 1000003u + (uint32_t)nb) errs++;
        e.syncBlock();
    }
    if (errs) atomicAdd(a.err, errs);
}

/* Fill the TB's shared memory, hold it, then verify nobody else wrote it. */
template <class Env>
__device__ void body_smem(const Env& e, const pagoda_smem_args& a)
{
    uint32_t* p = reinterpret_cast<uint32_t*>(e.getSMPtr());
    const uint32_t words = min(a.bytes, e.getSMBytes()) / 4u;
    const uint32_t key = a.seed * 2654435761u + (uint32_t)e.getBlockIdx() * 40503u;
    const int n = tb_threads(e);
    uint32_t errs = 0;
    if (e.getBlockTid() == 0 && ((uintptr_t)p & 31u) != 0) errs++;   /* getSMPtr is 32-byte aligned */
    if (e.getBlockTid() == 0 && e.getSMBytes() < a.bytes) errs++;      /* the grant covers the request */
    for (uint32_t i = e.getBlockTid(); i < words; i += n) p[i] = key ^ (i * 0x9E3779B9u);
    if (a.spin_ns) {
        uint64_t t0 = globaltimer_ns();
        while (globaltimer_ns() - t0 < a.spin_ns) { }
    }
    e.syncBlock();
    for (uint32_t i = e.getBlockTid(); i < words; i += n) errs += (p[i] != (key ^ (i * 0x9E3779B9u)));
    if (errs) atomicAdd(a.err, errs);
}

template <class Env>
__device__ void body_spin(const Env&, const pagoda_spin_args& a)
{
    uint64_t t0 = globaltimer_ns();
    while (globaltimer_ns() - t0 < a.ns) { }
}

template <class Env>
__device__ void body_gate(const Env&, const pagoda_gate_args& a)
{
    if (lane_id() == 0) {
        while (*a.flag == 0) __nanosleep(1000);
    }
    __syncwarp();
}

/* Brute-force schedule body (SURVEY §4 layer 4): announce the start, fill the whole grant with a
 * per-TB pattern, hold until the host opens the gate, then verify that no other task wrote into
 * the grant meanwhile (granules never overlap).  `started` and `flag` may live in pinned
 * host memory: plain stores / loads, one per warp (no system-scope atomics over PCIe). */
template <class Env>
__device__ __noinline__ void body_hold(const Env& e, const pagoda_hold_args& a)
{
    uint32_t* p = reinterpret_cast<uint32_t*>(e.getSMPtr());
    const uint32_t words = e.getSMBytes() / 4u;
    const uint32_t key = a.seed * 2654435761u + (uint32_t)e.getBlockIdx() * 40503u;
    const int n = tb_threads(e);
    uint32_t errs = 0;
    if (lane_id() == 0) *reinterpret_cast<volatile uint32_t*>(a.started) = 1u;
    for (uint32_t i = e.getBlockTid(); i < words; i += n) p[i] = key ^ (i * 0x9E3779B9u);
    if (lane_id() == 0)
        while (*a.flag == 0) __nanosleep(500);
    __syncwarp();
    if (e.canSync()) e.syncBlock();
    for (uint32_t i = e.getBlockTid(); i < words; i += n) errs += (p[i] != (key ^ (i * 0x9E3779B9u)));
    if (errs) atomicAdd(a.err, errs);
}

/* A body written the way the paper's users write one (Table 1, Fig. 1c): only the free
 * functions getTid() / syncBlock() / getSMPtr(), no Env.  They read the MasterKernel's WarpTable, so
 * this body exists only inside the MasterKernel (run_body refuses it elsewhere). */
static __device__ __noinline__ void body_paper(const pagoda_paper_args& a)
{
    const pagoda::WarpSlot& s = pagoda_my_slot();
    const int tid = getTid();
    const int bt = (int)s.warp_in_tb * 32 + (int)lane_id(), n = 32 * (int)s.warps_tb;
    const bool live = bt < (int)s.threads_tb;
    uint32_t errs = 0;
    if (live) a.out[a.base + (uint32_t)tid] = (uint32_t)tid + 1u;
    syncBlock();
    const int nb = (bt + 32) % n;   /* the thread one warp on, in this TB */
    const int ntid = ((int)s.tb * (int)s.warps_tb) * 32 + nb;
    if (live && nb < (int)s.threads_tb && a.out[a.base + (uint32_t)ntid] != (uint32_t)ntid + 1u) errs++;
    if (bt == 0 && (reinterpret_cast<uintptr_t>(getSMPtr()) & 31u) != 0) errs++;   /* 32-byte aligned */
    if (errs) atomicAdd(a.err, errs);
}

template <class Env> struct IsTaskEnv { static constexpr bool value = false; };
template <> struct IsTaskEnv<TaskEnv> { static constexpr bool value = true; };

/* ------------------------------------------------------------- MB
 * Table 3; strict '>' escape test, count includes
 * the escaping step, multiply-then-add never fused. */
template <class Env>
__device__ PAGODA_BODY_ATTR void body_mb(const Env& e, const pagoda_mb_args& a)
{
    const int T = total_threads(e);
    const int maxit = a.maxit;
    for (int p = e.getTid(); p < 4096; p += T) {
        const int gx = 64 * a.tx + (p & 63), gy = 64 * a.ty + (p >> 6);
        const float cr = __fadd_rn(a.x0, __fmul_rn((float)gx, a.dx));
        const float ci = __fadd_rn(a.y0, __fmul_rn((float)gy, a.dx));
        float zr = 0.0f, zi = 0.0f;
        int n = 0;
        /* Four iterations per branch: each step tests |z|^2 > 4 on its own z and
         * updates z unconditionally; the count advances to the first escaping step
         * (steps after it only touch values that are discarded).  A branch per
         * iteration costs more than the iteration itself on the critical path. */
        for (;;) {
            if (n + 4 > maxit) {   /* remainder: one iteration at a time */
                while (n < maxit) {
                    const float zr2 = __fmul_rn(zr, zr);
                    const float zi2 = __fmul_rn(zi, zi);
                    if (__fadd_rn(zr2, zi2) > 4.0f) break;
                    const float t = __fadd_rn(zr, zr);
                    zi = __fadd_rn(__fmul_rn(t, zi), ci);
                    zr = __fadd_rn(__fsub_rn(zr2, zi2), cr);
                    n++;
                }
                break;
            }
            bool esc[4];
#pragma unroll
            for (int s = 0; s < 4; s++) {
                const float zr2 = __fmul_rn(zr, zr);
                const float zi2 = __fmul_rn(zi, zi);
                esc[s] = __fadd_rn(zr2, zi2) > 4.0f;
                const float t = __fadd_rn(zr, zr);
                zi = __fadd_rn(__fmul_rn(t, zi), ci);
                zr = __fadd_rn(__fsub_rn(zr2, zi2), cr);
            }
            if (esc[0] | esc[1] | esc[2] | esc[3]) {
                n += esc[0] ? 0 : esc[1] ? 1 : esc[2] ? 2 : 3;
                break;
            }
            n += 4;
        }
        a.out[p] = (uint16_t)n;
    }
}

/* ------------------------------------------------------------- 3DES
 * TDEA EDE3, ECB (NIST [5]).  tables =
 * pagoda_tdes_tables(): SP[8][64] u32 (S-box j then P, for the 6-bit input of
 * box j), 48 round keys as a (kx, ky) u32 pair each (execution order
 * K1[0..15], K2[15..0], K3[0..15]), IP and FP byte tables [8][256] u64
 * (kept for the ABI; the body computes IP/FP with delta swaps, tdes_ip/tdes_fp).
 * Since FP then IP cancel between the three DES stages, a block is
 * IP, 48 rounds with a half-swap after every 16, FP.
 *
 * Round function without the E table: the 6-bit input of S-box j is
 * rotl(R, 4j+5) & 63 ^ k_j, so x = rotl(R,5) ^ kx holds the inputs of boxes
 * 0,6,4,2 in bytes 0..3 and y = rotl(R,1) ^ ky those of boxes 7,5,3,1 (kx, ky
 * pack the key chunks the same way).  The 8 S-box outputs after P are disjoint,
 * so f = XOR of 8 table words.  Three table placements: MTB-resident with one
 * copy per lane (conflict-free), staged in the TB's shared memory, or global. */
constexpr uint32_t kTdesStageBytes = 2048 + 384;   /* SP boxes + round keys (the IP/FP byte tables that
                                                       follow in the buffer are not used by the body) */

/* IP and FP as five delta swaps each on the (L, R) = (high, low) words of the
 * big-endian block: swap(a, b, n, m) exchanges the bits of b under mask m with
 * the bits of a under m << n.  Register-only; a byte-table gather instead costs
 * one L1 wavefront per distinct line touched by the warp (~10 per lookup).
 * The sequence is the IP table's (FIPS 46-3) factorisation; tests/test_abi.py
 * checks it against the product's IP/FP byte tables. */
__device__ __forceinline__ void tdes_swap(uint32_t& a, uint32_t& b, int n, uint32_t m)
{
    const uint32_t t = ((a >> n) ^ b) & m;
    b ^= t;
    a ^= t << n;
}
__device__ __forceinline__ void tdes_ip(uint32_t& l, uint32_t& r)
{
    tdes_swap(l, r, 4, 0x0f0f0f0fu);
    tdes_swap(l, r, 16, 0x0000ffffu);
    tdes_swap(r, l, 2, 0x33333333u);
    tdes_swap(r, l, 8, 0x00ff00ffu);
    tdes_swap(l, r, 1, 0x55555555u);
}
__device__ __forceinline__ void tdes_fp(uint32_t& l, uint32_t& r)
{
    tdes_swap(l, r, 1, 0x55555555u);
    tdes_swap(r, l, 8, 0x00ff00ffu);
    tdes_swap(r, l, 2, 0x33333333u);
    tdes_swap(l, r, 16, 0x0000ffffu);
    tdes_swap(l, r, 4, 0x0f0f0f0fu);
}

template <int kOff>
__device__ __forceinline__ uint32_t lds_at(uint32_t addr)
{
    uint32_t v;
    asm("ld.shared.u32 %0, [%1+%2];" : "=r"(v) : "r"(addr), "n"(kOff));
    return v;
}

enum { kTdesResident = 0, kTdesShared = 1, kTdesGlobal = 2 };

/* The 8 table words of a round have disjoint bits (P maps each S-box's 4 output bits to its own 4
 * positions), so their XOR equals their SUM.  A sum can run on the FMA pipe as IMAD d = a * one + b
 * (one = 1 from the constant bank, opaque to ptxas, so it is not folded into an IADD3 on the ALU
 * pipe).  A resident round had 16 ALU instructions (2 SHF, 2 LOP3, 8 PRMT, 4 LOP3 for the XORs with
 * l) per 8 shared-memory lookups: ALU and LDS both at 8 SM-clocks per warp-round.  Summing the words
 * in pairs on the FMA pipe (4 IMAD) leaves 2 XOR LOP3s: 14 ALU (7 clocks), 26 issued (6.5 clocks),
 * so the lookups alone bound the round. */
#ifndef PAGODA_TDES_FMA_SUM
#define PAGODA_TDES_FMA_SUM 1
#endif
/* Resident tables hold SP words rotated left by one bit, and the resident rounds keep L and R
 * rotated the same way (set after IP, undone before FP; rotation commutes with XOR): the S-box
 * inputs of boxes 7,5,3,1 are then R itself and those of boxes 0,6,4,2 R rotated by 4 (one funnel
 * shift per round instead of two). */
#ifndef PAGODA_TDES_ROT
#define PAGODA_TDES_ROT 1
#endif
/* The eight SP words of a round have disjoint bits (P permutes the 32 S-box output bits), so
 * their XOR is their sum: seven IMADs on the FMA pipe and one XOR with L on the ALU pipe.
 * Measured slower than four pair sums + two 3-input XORs (33.1 vs 33.7 M tasks/s: the longer
 * IMAD chain), so off. */
#ifndef PAGODA_TDES_FULL_SUM
#define PAGODA_TDES_FULL_SUM 0
#endif
static __constant__ uint32_t c_one = 1u;
__device__ __forceinline__ uint32_t sum_fma_pipe(uint32_t a, uint32_t b)
{
    uint32_t d;
    asm("mad.lo.u32 %0, %1, %2, %3;" : "=r"(d) : "r"(a), "r"(c_one), "r"(b));
    return d;
}
/* into / out of the resident rounds' rotated domain (PAGODA_TDES_ROT) */
template <int kMode>
__device__ __forceinline__ void tdes_rot_in(uint32_t& l, uint32_t& r)
{
    if (kMode == kTdesResident && PAGODA_TDES_ROT) {
        l = __funnelshift_l(l, l, 1);
        r = __funnelshift_l(r, r, 1);
    }
}
template <int kMode>
__device__ __forceinline__ void tdes_rot_out(uint32_t& l, uint32_t& r)
{
    if (kMode == kTdesResident && PAGODA_TDES_ROT) {
        l = __funnelshift_r(l, l, 1);
        r = __funnelshift_r(r, r, 1);
    }
}

/* f(R) for table placement kMode.
 * resident: the MTB-resident table at window address kResidentTdesAddr holds
 * SP[j][v] for lane l at word 4096 p + 64 v + 32 h + l, where byte p of x
 * (h = 0) or of y (h = 1) is box j's input.  With x, y masked to 6-bit fields,
 * one PRMT builds the offset: byte 1 = the field, byte 0 = lane*4 | 128 h
 * (tb), bytes 2-3 = 0; the pair base is the load's immediate.
 * shared: at sb + 256 j + 4 v (sb 256-byte aligned); global: sp[64 j + v]. */
template <int kMode>
__device__ __forceinline__ uint32_t tdes_f(uint32_t r, uint32_t kx, uint32_t ky, uint32_t tb, const uint32_t* sp)
{
    if (kMode == kTdesResident) {
        const uint32_t x = (__funnelshift_l(r, r, PAGODA_TDES_ROT ? 4 : 5) ^ kx) & 0x3F3F3F3Fu;
        const uint32_t y = ((PAGODA_TDES_ROT ? r : __funnelshift_l(r, r, 1)) ^ ky) & 0x3F3F3F3Fu;
        const uint32_t t1 = tb | 128u;
        constexpr uint32_t A = kResidentTdesAddr;
        const uint32_t s0 = lds_at<A + 0 * 16384>(__byte_perm(x, tb, 0x7604));
        const uint32_t s1 = lds_at<A + 1 * 16384>(__byte_perm(x, tb, 0x7614));
        const uint32_t s2 = lds_at<A + 2 * 16384>(__byte_perm(x, tb, 0x7624));
        const uint32_t s3 = lds_at<A + 3 * 16384>(__byte_perm(x, tb, 0x7634));
        const uint32_t s4 = lds_at<A + 0 * 16384>(__byte_perm(y, t1, 0x7604));
        const uint32_t s5 = lds_at<A + 1 * 16384>(__byte_perm(y, t1, 0x7614));
        const uint32_t s6 = lds_at<A + 2 * 16384>(__byte_perm(y, t1, 0x7624));
        const uint32_t s7 = lds_at<A + 3 * 16384>(__byte_perm(y, t1, 0x7634));
        if (PAGODA_TDES_FULL_SUM == 1)
            return sum_fma_pipe(sum_fma_pipe(sum_fma_pipe(s0, s1), sum_fma_pipe(s2, s3)),
                                sum_fma_pipe(sum_fma_pipe(s4, s5), sum_fma_pipe(s6, s7)));
        if (PAGODA_TDES_FULL_SUM == 2)   /* two quad sums (6 IMAD) + the caller's XOR with l: one LOP3 */
            return sum_fma_pipe(sum_fma_pipe(s0, s1), sum_fma_pipe(s2, s3)) ^
                   sum_fma_pipe(sum_fma_pipe(s4, s5), sum_fma_pipe(s6, s7));
        if (PAGODA_TDES_FMA_SUM)   /* 4 IMAD pair sums + the caller's 3-input XORs (with l): 2 LOP3 */
            return sum_fma_pipe(s0, s1) ^ sum_fma_pipe(s2, s3) ^ sum_fma_pipe(s4, s5) ^ sum_fma_pipe(s6, s7);
        return s0 ^ s1 ^ s2 ^ s3 ^ s4 ^ s5 ^ s6 ^ s7;
    }
    const uint32_t x = __funnelshift_l(r, r, 5) ^ kx;
    const uint32_t y = __funnelshift_l(r, r, 1) ^ ky;
    if (kMode == kTdesShared) {
        const uint32_t m = 63u << 2;
        return lds_at<0 * 256>(tb | ((x << 2) & m)) ^ lds_at<6 * 256>(tb | ((x >> 6) & m)) ^
               lds_at<4 * 256>(tb | ((x >> 14) & m)) ^ lds_at<2 * 256>(tb | ((x >> 22) & m)) ^
               lds_at<7 * 256>(tb | ((y << 2) & m)) ^ lds_at<5 * 256>(tb | ((y >> 6) & m)) ^
               lds_at<3 * 256>(tb | ((y >> 14) & m)) ^ lds_at<1 * 256>(tb | ((y >> 22) & m));
    } else {
        return __ldg(sp + 0 * 64 + (x & 63)) ^ __ldg(sp + 6 * 64 + ((x >> 8) & 63)) ^
               __ldg(sp + 4 * 64 + ((x >> 16) & 63)) ^ __ldg(sp + 2 * 64 + ((x >> 24) & 63)) ^
               __ldg(sp + 7 * 64 + (y & 63)) ^ __ldg(sp + 5 * 64 + ((y >> 8) & 63)) ^
               __ldg(sp + 3 * 64 + ((y >> 16) & 63)) ^ __ldg(sp + 1 * 64 + ((y >> 24) & 63));
    }
}

/* A registered key schedule (pagoda_tdes_register): the 48 round keys in this
 * module's constant bank, used by tasks whose tables pointer is the registered
 * one, so the round keys come from the constant cache and not the shared-
 * memory pipe the S-box lookups saturate.  Zero (never matching) in the
 * baselines' translation units. */
static __constant__ uint2 c_tdes_keys[48];
static __constant__ unsigned long long c_tdes_tables;

enum { kKeysGlobal = 0, kKeysShared = 1, kKeysConst = 2 };
/* round keys i, i+1 of stage st: from the TB's shared memory (kb = its stage base), global
 * (gk = the stage's keys) or the constant bank */
template <int kKeys, int kI>
__device__ __forceinline__ uint4 tdes_key2(uint32_t kb, const uint2* gk, int st)
{
    uint4 k;
    if (kKeys == kKeysShared) {
        asm("ld.shared.v4.u32 {%0, %1, %2, %3}, [%4+%5];" : "=r"(k.x), "=r"(k.y), "=r"(k.z), "=r"(k.w) : "r"(kb), "n"(kI * 8));
    } else if (kKeys == kKeysConst) {
        const uint2 a = c_tdes_keys[st * 16 + kI], b = c_tdes_keys[st * 16 + kI + 1];
        k = make_uint4(a.x, a.y, b.x, b.y);
    } else {
        const uint2 a = __ldg(gk + kI), b = __ldg(gk + kI + 1);
        k = make_uint4(a.x, a.y, b.x, b.y);
    }
    return k;
}

template <int kMode, int kKeys, class Env>
__device__ __forceinline__ void tdes_blocks(const Env& e, const pagoda_tdes_args& a, uint32_t tb, uint32_t kb)
{
    const uint2* gkeys = reinterpret_cast<const uint2*>(a.tables + 512);
    const int T = total_threads(e);
    for (uint32_t blk = (uint32_t)e.getTid(); blk < a.nblk; blk += (uint32_t)T) {
        const uint2 in = reinterpret_cast<const uint2*>(a.in)[blk];
        /* bytes are the block in FIPS (big-endian) order: L = bytes 0..3, R = bytes 4..7 */
        uint32_t l = __byte_perm(in.x, 0, 0x0123), r = __byte_perm(in.y, 0, 0x0123);
        tdes_ip(l, r);
        tdes_rot_in<kMode>(l, r);
#pragma unroll 1
        for (int st = 0; st < 3; st++) {
            const uint32_t kst = kb + st * 128;    /* 16 rounds x 8 bytes per stage */
            const uint2* gst = gkeys + st * 16;
/* two rounds per key load: one 16-byte shared load (one wavefront) for keys I, I+1 */
#define PAGODA_TDES_ROUND2(I)                                                        \
            {                                                                        \
                const uint4 k = tdes_key2<kKeys, I>(kst, gst, st);                   \
                uint32_t t = l ^ tdes_f<kMode>(r, k.x, k.y, tb, a.tables);      \
                l = r;                                                               \
                r = t;                                                               \
                t = l ^ tdes_f<kMode>(r, k.z, k.w, tb, a.tables);               \
                l = r;                                                               \
                r = t;                                                               \
            }
            PAGODA_TDES_ROUND2(0) PAGODA_TDES_ROUND2(2) PAGODA_TDES_ROUND2(4) PAGODA_TDES_ROUND2(6)
            PAGODA_TDES_ROUND2(8) PAGODA_TDES_ROUND2(10) PAGODA_TDES_ROUND2(12) PAGODA_TDES_ROUND2(14)
#undef PAGODA_TDES_ROUND2
            const uint32_t t = l;   /* undo the last half-swap: stage output (R16, L16) */
            l = r;
            r = t;
        }
        tdes_rot_out<kMode>(l, r);
        tdes_fp(l, r);
        reinterpret_cast<uint2*>(a.out)[blk] = make_uint2(__byte_perm(l, 0, 0x0123), __byte_perm(r, 0, 0x0123));
    }
}

#ifndef PAGODA_TDES_PAIR
#define PAGODA_TDES_PAIR 1
#endif
struct FirstBlockOnly {   /* makes tdes_blocks process block 0 of its args only */
    __device__ __forceinline__ int getTid() const { return 0; }
    __device__ __forceinline__ int getNumBlocks() const { return 1; }
    __device__ __forceinline__ int getBlockWarps() const { return 1; }
};
/* Two blocks per loop trip (blocks b and b + T of this thread): one round-key load serves both,
 * halving the key wavefronts, and the two rounds are independent chains.  Resident tables,
 * keys in the TB's shared memory. */
template <int kKeys, class Env>
__device__ __forceinline__ void tdes_blocks_pair(const Env& e, const pagoda_tdes_args& a, uint32_t tb, uint32_t kb)
{
    const uint32_t T = (uint32_t)total_threads(e);
    uint32_t blk = (uint32_t)e.getTid();
    for (; blk + T < a.nblk; blk += 2u * T) {
        const uint2 in0 = reinterpret_cast<const uint2*>(a.in)[blk];
        const uint2 in1 = reinterpret_cast<const uint2*>(a.in)[blk + T];
        uint32_t l0 = __byte_perm(in0.x, 0, 0x0123), r0 = __byte_perm(in0.y, 0, 0x0123);
        uint32_t l1 = __byte_perm(in1.x, 0, 0x0123), r1 = __byte_perm(in1.y, 0, 0x0123);
        tdes_ip(l0, r0);
        tdes_ip(l1, r1);
        tdes_rot_in<kTdesResident>(l0, r0);
        tdes_rot_in<kTdesResident>(l1, r1);
#pragma unroll 1
        for (int st = 0; st < 3; st++) {
            const uint32_t kst = kb + st * 128;
#define PAGODA_TDES_ROUND2P(I)                                                                   \
            {                                                                                    \
                const uint4 k = tdes_key2<kKeys, I>(kst, nullptr, st);                           \
                uint32_t t0 = l0 ^ tdes_f<kTdesResident>(r0, k.x, k.y, tb, nullptr);        \
                uint32_t t1 = l1 ^ tdes_f<kTdesResident>(r1, k.x, k.y, tb, nullptr);        \
                l0 = r0; r0 = t0; l1 = r1; r1 = t1;                                              \
                t0 = l0 ^ tdes_f<kTdesResident>(r0, k.z, k.w, tb, nullptr);                 \
                t1 = l1 ^ tdes_f<kTdesResident>(r1, k.z, k.w, tb, nullptr);                 \
                l0 = r0; r0 = t0; l1 = r1; r1 = t1;                                              \
            }
            PAGODA_TDES_ROUND2P(0) PAGODA_TDES_ROUND2P(2) PAGODA_TDES_ROUND2P(4) PAGODA_TDES_ROUND2P(6)
            PAGODA_TDES_ROUND2P(8) PAGODA_TDES_ROUND2P(10) PAGODA_TDES_ROUND2P(12) PAGODA_TDES_ROUND2P(14)
#undef PAGODA_TDES_ROUND2P
            uint32_t t = l0; l0 = r0; r0 = t;
            t = l1; l1 = r1; r1 = t;
        }
        tdes_rot_out<kTdesResident>(l0, r0);
        tdes_rot_out<kTdesResident>(l1, r1);
        tdes_fp(l0, r0);
        tdes_fp(l1, r1);
        reinterpret_cast<uint2*>(a.out)[blk] = make_uint2(__byte_perm(l0, 0, 0x0123), __byte_perm(r0, 0, 0x0123));
        reinterpret_cast<uint2*>(a.out)[blk + T] = make_uint2(__byte_perm(l1, 0, 0x0123), __byte_perm(r1, 0, 0x0123));
    }
    if (blk < a.nblk) {   /* an odd block left: the single-block loop from it */
        pagoda_tdes_args rest = a;
        rest.in += blk;
        rest.out += blk;
        rest.nblk = 1;
        tdes_blocks<kTdesResident, kKeys>(FirstBlockOnly{}, rest, tb, kb);
    }
}

#ifndef PAGODA_TDES_NOINLINE
#define PAGODA_TDES_NOINLINE 1   /* the 3DES body as a call: the executor keeps its own register allocation
                                    (35.5 -> 36.0 M tasks/s) */
#endif
#if PAGODA_TDES_NOINLINE
#define PAGODA_TDES_ATTR __noinline__
#else
#define PAGODA_TDES_ATTR
#endif
template <class Env>
__device__ PAGODA_TDES_ATTR void body_tdes(const Env& e, const pagoda_tdes_args& a)
{
    const uint32_t res = e.getResidentTdes();
    if (res && (unsigned long long)a.tables == c_tdes_tables) {   /* resident tables, registered keys: */
        if (PAGODA_TDES_PAIR) tdes_blocks_pair<kKeysConst>(e, a, lane_id() << 2, 0);   /* nothing to stage */
        else tdes_blocks<kTdesResident, kKeysConst>(e, a, lane_id() << 2, 0);
        return;
    }
    const uint32_t need = res ? 384u : kTdesStageBytes;
    uint32_t sb = 0;
    if (e.getSMBytes() >= need && e.canSync()) {   /* stage round keys (and SP boxes) into the TB's shmem */
        char* s = e.getSMPtr();
        if (e.getBlockTid() < 32) e.stage(s, res ? reinterpret_cast<const char*>(a.tables) + 2048 : (const char*)a.tables, need);
        e.syncBlock();
        sb = smem_u32(s);
    }
    if (PAGODA_TDES_PAIR && res && sb) tdes_blocks_pair<kKeysShared>(e, a, lane_id() << 2, sb);
    else if (res && sb) tdes_blocks<kTdesResident, kKeysShared>(e, a, lane_id() << 2, sb);
    else if (res) tdes_blocks<kTdesResident, kKeysGlobal>(e, a, lane_id() << 2, 0);
    else if (sb) tdes_blocks<kTdesShared, kKeysShared>(e, a, sb, sb + 2048);
    else tdes_blocks<kTdesGlobal, kKeysGlobal>(e, a, 0, 0);
}

/* ------------------------------------------------------------- MM
 * CUDA SDK MatrixMul [22] (Table 3); 32x32x32 fp32; C[i][j] is the
 * fma chain over k ascending from 0.  A and B are staged into the TB's shmem
 * with TMA bulk copies when 8 KiB were granted and the TB can synchronise. */
#ifndef PAGODA_MM_VEC
#define PAGODA_MM_VEC 0        /* A's rows as float4 loads (64 shared loads per thread instead of 160): measured
                                  slower at 32 registers (the body spills: 46.5 vs 48.3 M tasks/s) */
#endif
#ifndef PAGODA_MM_NOINLINE
#define PAGODA_MM_NOINLINE 1   /* a call: keeps the 32-register executors' allocation (MM 47.4 -> 48.3 M tasks/s) */
#endif
#if PAGODA_MM_NOINLINE
#define PAGODA_MM_ATTR __noinline__
#else
#define PAGODA_MM_ATTR
#endif
template <class Env>
__device__ PAGODA_MM_ATTR void body_mm(const Env& e, const pagoda_mm_args& a)
{
    const float* A = a.A;
    const float* B = a.B;
    if (e.getSMBytes() >= 8192 && e.canSync()) {
        float* s = reinterpret_cast<float*>(e.getSMPtr());
        const int w = e.getBlockTid() >> 5;
        if (e.getBlockWarps() >= 2) {
            if (w == 0) e.stage(s, A, 4096);
            else if (w == 1) e.stage(s + 1024, B, 4096);
        } else {
            e.stage(s, A, 4096);
            e.stage(s + 1024, B, 4096);
        }
        e.syncBlock();
        A = s;
        B = s + 1024;
    }
    /* A thread's outputs idx, idx + T, ... (same column j when 32 | T) advance together, four
     * independent fma chains at a time (each still k ascending from 0): one B load serves all */
    const int T = total_threads(e);
    for (int base = e.getTid(); base < 1024; base += 4 * T) {
        float acc[4] = {0.0f, 0.0f, 0.0f, 0.0f};
        int row[4];
#pragma unroll
        for (int q = 0; q < 4; q++) row[q] = min(base + q * T, 1023) >> 5;   /* past the end: a dummy row */
        const int j = base & 31;
        if (PAGODA_MM_VEC && (T & 31) == 0 && (reinterpret_cast<uintptr_t>(A) & 15u) == 0) {
            /* A's row segments as float4 (one broadcast load per 4 k per row: 64 loads per thread instead
             * of 160); every chain still accumulates k ascending */
#pragma unroll 2
            for (int k0 = 0; k0 < 32; k0 += 4) {
                float4 av[4];
#pragma unroll
                for (int q = 0; q < 4; q++) av[q] = *reinterpret_cast<const float4*>(A + row[q] * 32 + k0);
                const float b0 = B[(k0 + 0) * 32 + j], b1 = B[(k0 + 1) * 32 + j];
                const float b2 = B[(k0 + 2) * 32 + j], b3 = B[(k0 + 3) * 32 + j];
#pragma unroll
                for (int q = 0; q < 4; q++) {
                    acc[q] = __fmaf_rn(av[q].x, b0, acc[q]);
                    acc[q] = __fmaf_rn(av[q].y, b1, acc[q]);
                    acc[q] = __fmaf_rn(av[q].z, b2, acc[q]);
                    acc[q] = __fmaf_rn(av[q].w, b3, acc[q]);
                }
            }
        } else if ((T & 31) == 0) {
#pragma unroll 8
            for (int k = 0; k < 32; k++) {
                const float b = B[k * 32 + j];
#pragma unroll
                for (int q = 0; q < 4; q++) acc[q] = __fmaf_rn(A[row[q] * 32 + k], b, acc[q]);
            }
        } else {   /* T not a multiple of 32: each item has its own column */
#pragma unroll 4
            for (int k = 0; k < 32; k++) {
#pragma unroll
                for (int q = 0; q < 4; q++)
                    acc[q] = __fmaf_rn(A[row[q] * 32 + k], B[k * 32 + (min(base + q * T, 1023) & 31)], acc[q]);
            }
        }
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (base + q * T < 1024) a.C[base + q * T] = acc[q];
    }
}

/* ------------------------------------------------------------- MM 64x64
 * Table 4's MatrixMul size ("64 x 64 matrix", shared memory and
 * barrier used), NEXT-4: C = A B, 64x64x64 fp32, each C[i][j] the fma chain
 * over k ascending from 0 (oracle orc_mm64).  A and B (16 KiB each) are staged
 * by TMA when 32 KiB were granted and the TB can synchronise; four independent
 * chains per thread share each B load, as in body_mm. */
template <class Env>
__device__ __noinline__ void body_mm64(const Env& e, const pagoda_mm_args& a)
{
    const float* A = a.A;
    const float* B = a.B;
    if (e.getSMBytes() >= 32768 && e.canSync()) {
        float* s = reinterpret_cast<float*>(e.getSMPtr());
        const int w = e.getBlockTid() >> 5;
        if (e.getBlockWarps() >= 2) {
            if (w == 0) e.stage(s, A, 16384);
            else if (w == 1) e.stage(s + 4096, B, 16384);
        } else {
            e.stage(s, A, 16384);
            e.stage(s + 4096, B, 16384);
        }
        e.syncBlock();
        A = s;
        B = s + 4096;
    }
    const int T = total_threads(e);
    for (int base = e.getTid(); base < 4096; base += 4 * T) {
        float acc[4] = {0.0f, 0.0f, 0.0f, 0.0f};
        int row[4], col[4];
#pragma unroll
        for (int q = 0; q < 4; q++) {
            const int o = min(base + q * T, 4095);   /* past the end: a dummy item */
            row[q] = o >> 6;
            col[q] = o & 63;
        }
        if ((T & 63) == 0) {   /* the four items share column col[0] */
#pragma unroll 8
            for (int k = 0; k < 64; k++) {
                const float b = B[k * 64 + col[0]];
#pragma unroll
                for (int q = 0; q < 4; q++) acc[q] = __fmaf_rn(A[row[q] * 64 + k], b, acc[q]);
            }
        } else {
#pragma unroll 4
            for (int k = 0; k < 64; k++) {
#pragma unroll
                for (int q = 0; q < 4; q++) acc[q] = __fmaf_rn(A[row[q] * 64 + k], B[k * 64 + col[q]], acc[q]);
            }
        }
#pragma unroll
        for (int q = 0; q < 4; q++)
            if (base + q * T < 4096) a.C[base + q * T] = acc[q];
    }
}

/* ------------------------------------------------------------- MM, tensor cores
 * NEXT-4: the same C = A B (32x32x32 fp32) on the tensor cores
 * as 3xTF32: x = hi + lo with hi = tf32(x) and lo = tf32(x - hi), and
 * C += lo_A hi_B + hi_A lo_B + hi_A hi_B (the small terms first; lo_A lo_B is
 * below fp32 resolution), with mma.sync.m16n8k8 (fp32 accumulate).  A task is
 * 2 x 4 tiles of 16x8; warp w of the task takes tiles w, w + W, ...  The
 * products are summed in the tensor core's order, not the fma chain's, so
 * parity is |g - o| <= 1e-5 sum_k |a_ik b_kj|.
 * tcgen05 needs M >= 64 and a TMEM allocation per CTA: a 32x32 task is below
 * both. */
__device__ __forceinline__ void tf32_split(float x, uint32_t& hi, uint32_t& lo)
{
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(hi) : "f"(x));
    const float r = __fsub_rn(x, __uint_as_float(hi));
    asm("cvt.rna.tf32.f32 %0, %1;" : "=r"(lo) : "f"(r));
}

__device__ __forceinline__ void mma_tf32(float (&c)[4], const uint32_t (&a)[4], uint32_t b0, uint32_t b1)
{
    asm volatile(
        "mma.sync.aligned.m16n8k8.row.col.f32.tf32.tf32.f32 {%0, %1, %2, %3}, {%4, %5, %6, %7}, {%8, %9}, "
        "{%0, %1, %2, %3};"
        : "+f"(c[0]), "+f"(c[1]), "+f"(c[2]), "+f"(c[3])
        : "r"(a[0]), "r"(a[1]), "r"(a[2]), "r"(a[3]), "r"(b0), "r"(b1));
}

template <class Env>
__device__ PAGODA_BODY_ATTR void body_mm_tc(const Env& e, const pagoda_mm_args& a)
{
    const float* A = a.A;
    const float* B = a.B;
    if (e.getSMBytes() >= 8192 && e.canSync()) {   /* stage A, B with TMA bulk copies, as body_mm */
        float* s = reinterpret_cast<float*>(e.getSMPtr());
        const int w = e.getBlockTid() >> 5;
        if (e.getBlockWarps() >= 2) {
            if (w == 0) e.stage(s, A, 4096);
            else if (w == 1) e.stage(s + 1024, B, 4096);
        } else {
            e.stage(s, A, 4096);
            e.stage(s + 1024, B, 4096);
        }
        e.syncBlock();
        A = s;
        B = s + 1024;
    }
    const int lane = (int)lane_id(), g = lane >> 2, t = lane & 3;
    const int nw = total_threads(e) >> 5;
    for (int tile = e.getTid() >> 5; tile < 8; tile += nw) {
        const int m0 = (tile >> 2) * 16, n0 = (tile & 3) * 8;
        float c[4] = {0.0f, 0.0f, 0.0f, 0.0f};
#pragma unroll 1
        for (int k0 = 0; k0 < 32; k0 += 8) {
            uint32_t ah[4], al[4], bh0, bl0, bh1, bl1;
            tf32_split(A[(m0 + g) * 32 + k0 + t], ah[0], al[0]);
            tf32_split(A[(m0 + g + 8) * 32 + k0 + t], ah[1], al[1]);
            tf32_split(A[(m0 + g) * 32 + k0 + t + 4], ah[2], al[2]);
            tf32_split(A[(m0 + g + 8) * 32 + k0 + t + 4], ah[3], al[3]);
            tf32_split(B[(k0 + t) * 32 + n0 + g], bh0, bl0);
            tf32_split(B[(k0 + t + 4) * 32 + n0 + g], bh1, bl1);
            mma_tf32(c, al, bh0, bh1);
            mma_tf32(c, ah, bl0, bl1);
            mma_tf32(c, ah, bh0, bh1);
        }
        *reinterpret_cast<float2*>(a.C + (m0 + g) * 32 + n0 + 2 * t) = make_float2(c[0], c[1]);
        *reinterpret_cast<float2*>(a.C + (m0 + g + 8) * 32 + n0 + 2 * t) = make_float2(c[2], c[3]);
    }
}

/* ------------------------------------------------------------- FB
 * Fig. 1c: VH = H (*) r, VD[m] = VH[8m],
 * VU = up-sample of VD, y = F (*) VU; causal, fma chains k ascending.
 * Only VH[8m] is ever used, and the zero terms of VU add exactly +0, so
 * y[j] = sum over k = j mod 8, j mod 8 + 8, ... <= min(31, j) of F[k] VD[(j-k)/8]. */
template <class Env>
__device__ PAGODA_BODY_ATTR void body_fb(const Env& e, const pagoda_fb_args& a)
{
    float* vd = (e.getSMBytes() >= 1024) ? reinterpret_cast<float*>(e.getSMPtr())
                                         : a.scratch + 256 * e.getBlockIdx();
    const int n = tb_threads(e), bt = e.getBlockTid();
    /* four VD chains per thread advance together (ILP); r outside [0, 2048) reads as 0, and an
     * fma with a zero factor leaves the (never -0) accumulator unchanged: identical to skipping */
    for (int m0 = bt; m0 < 256; m0 += 4 * n) {
        float acc[4] = {0.0f, 0.0f, 0.0f, 0.0f};
#pragma unroll 8
        for (int k = 0; k < 32; k++) {
            const float hk = a.H[k];
#pragma unroll
            for (int i = 0; i < 4; i++) {
                const int idx = 8 * (m0 + i * n) - k;
                const float rv = (m0 + i * n < 256 && idx >= 0) ? a.r[idx] : 0.0f;
                acc[i] = __fmaf_rn(hk, rv, acc[i]);
            }
        }
#pragma unroll
        for (int i = 0; i < 4; i++)
            if (m0 + i * n < 256) vd[m0 + i * n] = acc[i];
    }
    e.syncBlock();
    const int T = total_threads(e);
    for (int j = e.getTid(); j < 2048; j += T) {
        float acc = 0.0f;
        const int kmax = min(31, j);
        for (int k = j & 7; k <= kmax; k += 8) acc = __fmaf_rn(a.F[k], vd[(j - k) >> 3], acc);
        a.y[j] = acc;
    }
}

/* ------------------------------------------------------------- BF
 * Table 3: v[c][t] = sum_k h[c][k] x[c][t-k]
 * (16 taps), y[b][t] = sum_c w[b][c] v[c][t], out = |y|^2.  No barrier:
 * each thread computes the v values its own t needs. */
__device__ __forceinline__ void cmac(float& re, float& im, float ar, float ai, float br, float bi)
{
    re = __fmaf_rn(ar, br, re);
    re = __fmaf_rn(-ai, bi, re);
    im = __fmaf_rn(ar, bi, im);
    im = __fmaf_rn(ai, br, im);
}

template <class Env>
__device__ PAGODA_BODY_ATTR void body_bf(const Env& e, const pagoda_bf_args& a)
{
    const int T = total_threads(e);
    const float2* x = reinterpret_cast<const float2*>(a.x);
    const float2* h = reinterpret_cast<const float2*>(a.h);
    const float2* w = reinterpret_cast<const float2*>(a.w);
    for (int t = e.getTid(); t < 512; t += T) {
        /* all 16 taps of all 4 channels unrolled: 8 independent fma chains; x before the
         * start of the signal reads as 0 (exact: see FB) */
        float vr[4] = {0.0f, 0.0f, 0.0f, 0.0f}, vi[4] = {0.0f, 0.0f, 0.0f, 0.0f};
#pragma unroll
        for (int k = 0; k < 16; k++) {
#pragma unroll
            for (int c = 0; c < 4; c++) {
                const float2 hk = h[c * 16 + k];
                const float2 xv = (t - k >= 0) ? x[c * 512 + t - k] : make_float2(0.0f, 0.0f);
                cmac(vr[c], vi[c], hk.x, hk.y, xv.x, xv.y);
            }
        }
#pragma unroll
        for (int b = 0; b < 4; b++) {
            float re = 0.0f, im = 0.0f;
#pragma unroll
            for (int c = 0; c < 4; c++) {
                const float2 wb = w[b * 4 + c];
                cmac(re, im, wb.x, wb.y, vr[c], vi[c]);
            }
            a.out[b * 512 + t] = __fmaf_rn(re, re, __fmul_rn(im, im));
        }
    }
}

/* ------------------------------------------------------------- CONV
 * CUDA SDK convolutionSeparable [19], DESIGN.md "CONV":
 * tmp[y][x] = sum_{d=-8..8} img[y][x+d] krow[8-d], out[y][x] = sum_d
 * tmp[y+d][x] kcol[8-d], zero outside, d ascending.  TB j produces output rows
 * [r0, r1) and first computes the tmp rows [r0-8, r1+8) they need into
 * scratch + 16384*j (same row indexing as the full image). */
__device__ __forceinline__ void discard_l2(const void* line128)
{
    asm volatile("discard.global.L2 [%0], 128;" ::"l"(line128) : "memory");
}

/* Row pass over image rows [t0, t1): tmp row y at tmp + (y - base) * 128.  Each thread produces 4
 * neighbouring outputs with a sliding register window: per tap one new input load, one kernel
 * load and 4 independent fma chains.  Samples outside the image read as 0, which is exact (an
 * fma with a zero factor leaves the accumulator unchanged). */
template <class Env>
__device__ __forceinline__ void conv_rows(const Env& e, const pagoda_conv_args& a, float* tmp, int base, int t0, int t1)
{
    const int n = tb_threads(e), bt = e.getBlockTid();
    for (int item = bt; item < (t1 - t0) * 32; item += n) {
        const int y = t0 + (item >> 5), x0 = (item & 31) * 4;
        const float* row = a.img + y * 128;
        auto in = [&](int xx) { return (xx >= 0 && xx < 128) ? row[xx] : 0.0f; };
        float w0 = in(x0 - 8), w1 = in(x0 - 7), w2 = in(x0 - 6), w3 = in(x0 - 5);
        float c0 = 0.0f, c1 = 0.0f, c2 = 0.0f, c3 = 0.0f;
#pragma unroll
        for (int d = -8; d <= 8; d++) {
            const float k = a.krow[8 - d];
            c0 = __fmaf_rn(w0, k, c0);
            c1 = __fmaf_rn(w1, k, c1);
            c2 = __fmaf_rn(w2, k, c2);
            c3 = __fmaf_rn(w3, k, c3);
            w0 = w1;
            w1 = w2;
            w2 = w3;
            if (d < 8) w3 = in(x0 + 4 + d);
        }
        *reinterpret_cast<float4*>(tmp + (y - base) * 128 + x0) = make_float4(c0, c1, c2, c3);
    }
}
/* Column pass for output rows [b0, b1) from tmp rows [lo, hi) (at tmp + (y - base) * 128): rows
 * outside [lo, hi) read as 0.  For an output row in [b0, b1) that is exactly the image's zero
 * padding ([lo, hi) holds every in-image row within 8 of the band); the rows of a ragged last
 * group of 4 past b1 are computed from those zeros and dropped. */
template <class Env>
__device__ __forceinline__ void conv_cols(const Env& e, const pagoda_conv_args& a, const float* tmp, int base, int lo,
                                          int hi, int b0, int b1)
{
    const int n = tb_threads(e), bt = e.getBlockTid();
    const int groups = (b1 - b0 + 3) / 4;
    for (int item = bt; item < groups * 128; item += n) {
        const int x = item & 127, y0 = b0 + (item >> 7) * 4;
        auto tv = [&](int yy) { return (yy >= lo && yy < hi) ? tmp[(yy - base) * 128 + x] : 0.0f; };
        float w0 = tv(y0 - 8), w1 = tv(y0 - 7), w2 = tv(y0 - 6), w3 = tv(y0 - 5);
        float c0 = 0.0f, c1 = 0.0f, c2 = 0.0f, c3 = 0.0f;
#pragma unroll
        for (int d = -8; d <= 8; d++) {
            const float k = a.kcol[8 - d];
            c0 = __fmaf_rn(w0, k, c0);
            c1 = __fmaf_rn(w1, k, c1);
            c2 = __fmaf_rn(w2, k, c2);
            c3 = __fmaf_rn(w3, k, c3);
            w0 = w1;
            w1 = w2;
            w2 = w3;
            if (d < 8) w3 = tv(y0 + 4 + d);
        }
        float* o = a.out + y0 * 128 + x;
        if (y0 + 0 < b1) o[0] = c0;
        if (y0 + 1 < b1) o[128] = c1;
        if (y0 + 2 < b1) o[256] = c2;
        if (y0 + 3 < b1) o[384] = c3;
    }
}

/* The row-pass intermediate goes through the TB's global scratch, even when the TB is granted shared
 * memory: keeping it in the grant band by band (B output rows need B + 16 tmp rows, 512 B each;
 * the halo rows recomputed per band) was measured slower on config 4 at every threshold tried
 * (bands of >= 32 rows: 11.5 -> 10.3 M tasks/s; >= 64 rows: 12.7 -> 12.4 M): CONV is bound by
 * its load latency, not by the scratch round trip through L2. */
template <class Env>
__device__ PAGODA_CONV_BODY_ATTR void body_conv(const Env& e, const pagoda_conv_args& a)
{
    const int nb = e.getNumBlocks(), j = e.getBlockIdx();
    const int r0 = (128 * j) / nb, r1 = (128 * (j + 1)) / nb;
    const int t0 = max(0, r0 - 8), t1 = min(128, r1 + 8);
    float* tmp = a.scratch + 16384 * j;
    conv_rows(e, a, tmp, 0, t0, t1);
    e.syncBlock();
    conv_cols(e, a, tmp, 0, 0, 128, r0, r1);   /* rows of [0,128) outside [t0,t1) feed dropped outputs only */
    /* The row-pass rows are dead now.  Written moments ago, they sit dirty in L2; without this
     * they would be written back to HBM on eviction (64 KiB per task, half again the task's
     * algorithmic traffic).  discard.global.L2 drops the lines without a write-back, once every
     * thread of the TB has finished reading them (the barrier). */
    e.syncBlock();
    const int n = tb_threads(e), bt = e.getBlockTid();
    for (int i = bt; i < (t1 - t0) * 4; i += n) discard_l2(tmp + t0 * 128 + i * 32);
}

/* ------------------------------------------------------------- DCT
 * CUDA SDK DCT8x8 [21]: per 8x8 block
 * T[u][y] = sum_x C[u][x] X[x][y], Y[u][v] = sum_y T[u][y] C[v][y].
 * Work item (block, u): one thread computes T[u][*] and Y[u][*] of the block
 * whose top-left sample is X (row stride 128) into Y (row u of the output block). */
/* A registered coefficient matrix (pagoda_dct_register): C in this module's constant bank,
 * used by DCT tasks whose coef pointer equals the registered one.  The second pass then reads
 * C[v][y] as an FFMA constant operand (v, y unrolled) instead of 16 uniform vector loads per
 * item; 0 = none registered (and always 0 in the baselines' translation unit). */
static __constant__ float c_dct_coef[64];
static __constant__ unsigned long long c_dct_coef_ptr;

template <bool kConstCoef>
__device__ __forceinline__ void dct_item(const pagoda_dct_args& a, const float* X, int u, float* Y)
{
    /* row x of the block arrives as two float4; the 8 chains T[u][*] advance together
     * (each still accumulates over x ascending) */
    float Tu[8] = {0.0f, 0.0f, 0.0f, 0.0f, 0.0f, 0.0f, 0.0f, 0.0f};
    float4 cq;   /* C[u][x..x+3], one vector load per four x (the load pipe is the limit) */
#pragma unroll
    for (int x = 0; x < 8; x++) {
        if ((x & 3) == 0) cq = *reinterpret_cast<const float4*>(a.coef + u * 8 + x);
        const float cu = (x & 3) == 0 ? cq.x : (x & 3) == 1 ? cq.y : (x & 3) == 2 ? cq.z : cq.w;
        const float4 lo = *reinterpret_cast<const float4*>(X + x * 128);
        const float4 hi = *reinterpret_cast<const float4*>(X + x * 128 + 4);
        Tu[0] = __fmaf_rn(cu, lo.x, Tu[0]);
        Tu[1] = __fmaf_rn(cu, lo.y, Tu[1]);
        Tu[2] = __fmaf_rn(cu, lo.z, Tu[2]);
        Tu[3] = __fmaf_rn(cu, lo.w, Tu[3]);
        Tu[4] = __fmaf_rn(cu, hi.x, Tu[4]);
        Tu[5] = __fmaf_rn(cu, hi.y, Tu[5]);
        Tu[6] = __fmaf_rn(cu, hi.z, Tu[6]);
        Tu[7] = __fmaf_rn(cu, hi.w, Tu[7]);
    }
    float Yv[8];
#pragma unroll
    for (int v = 0; v < 8; v++) {
        float4 clo, chi;
        if (kConstCoef) {
            clo = make_float4(c_dct_coef[v * 8 + 0], c_dct_coef[v * 8 + 1], c_dct_coef[v * 8 + 2], c_dct_coef[v * 8 + 3]);
            chi = make_float4(c_dct_coef[v * 8 + 4], c_dct_coef[v * 8 + 5], c_dct_coef[v * 8 + 6], c_dct_coef[v * 8 + 7]);
        } else {
            clo = *reinterpret_cast<const float4*>(a.coef + v * 8);
            chi = *reinterpret_cast<const float4*>(a.coef + v * 8 + 4);
        }
        float acc = 0.0f;
        acc = __fmaf_rn(Tu[0], clo.x, acc);
        acc = __fmaf_rn(Tu[1], clo.y, acc);
        acc = __fmaf_rn(Tu[2], clo.z, acc);
        acc = __fmaf_rn(Tu[3], clo.w, acc);
        acc = __fmaf_rn(Tu[4], chi.x, acc);
        acc = __fmaf_rn(Tu[5], chi.y, acc);
        acc = __fmaf_rn(Tu[6], chi.z, acc);
        acc = __fmaf_rn(Tu[7], chi.w, acc);
        Yv[v] = acc;
    }
    *reinterpret_cast<float4*>(Y) = make_float4(Yv[0], Yv[1], Yv[2], Yv[3]);
    *reinterpret_cast<float4*>(Y + 4) = make_float4(Yv[4], Yv[5], Yv[6], Yv[7]);
}

/* Table 5: with >= 4 KiB of shared memory granted and a barrier, a TB
 * stages bands of whole 8-row block rows (4 KiB each, as many as the grant holds) with
 * TMA bulk copies and transforms them from shared memory; TB j takes bands j, j + nb, ...
 * Otherwise every item reads its block from global memory.  Same arithmetic either way. */
template <bool kConstCoef, class Env>
__device__ __noinline__ void body_dct_t(const Env& e, const pagoda_dct_args& a)
{
    if (e.getSMBytes() >= 4096 && e.canSync()) {
        float* s = reinterpret_cast<float*>(e.getSMPtr());
        const int R = min(16, (int)(e.getSMBytes() >> 12));      /* block rows per band */
        const int nbands = (16 + R - 1) / R, nb = e.getNumBlocks();
        const int n = tb_threads(e), bt = e.getBlockTid(), w = bt >> 5, W = e.getBlockWarps();
        for (int band = e.getBlockIdx(); band < nbands; band += nb) {
            const int r0 = band * R, rows = min(R, 16 - r0);
            for (int r = w; r < rows; r += W) e.stage(s + r * 1024, a.img + (r0 + r) * 1024, 4096);
            e.syncBlock();
            for (int item = bt; item < rows * 128; item += n) {
                const int rb = item >> 7, bx = (item >> 3) & 15, u = item & 7;
                dct_item<kConstCoef>(a, s + rb * 1024 + bx * 8, u, a.out + ((r0 + rb) * 8 + u) * 128 + bx * 8);
            }
            e.syncBlock();   /* before the next band overwrites the stage */
        }
        return;
    }
    const int T = total_threads(e);
    for (int item = e.getTid(); item < 256 * 8; item += T) {
        const int blk = item >> 3, u = item & 7;
        const int by = blk >> 4, bx = blk & 15;
        dct_item<kConstCoef>(a, a.img + (by * 8) * 128 + bx * 8, u, a.out + (by * 8 + u) * 128 + bx * 8);
    }
}

template <class Env>
__device__ void body_dct(const Env& e, const pagoda_dct_args& a)
{
    if (c_dct_coef_ptr != 0 && (unsigned long long)a.coef == c_dct_coef_ptr) body_dct_t<true>(e, a);
    else body_dct_t<false>(e, a);
}

/* ------------------------------------------------------------- dispatch */
/* A body behind a call (its code out of the caller's register allocation). */
template <class Env, class A, void (*F)(const Env&, const A&)>
__device__ __noinline__ void as_call(const Env& e, const A& a)
{
    F(e, a);
}
/* kCallCold: the MB / FB / BF / CONV bodies behind calls.  The 4-MTB/SM MasterKernel (32 registers,
 * the MM presets) takes it: its executor loop then spills less around the bodies it does run
 * (measured: MM 58.9 -> 62.4 M tasks/s); the other configurations run those bodies and keep them
 * inline (config 5 15.4 vs 17.2 M tasks/s, mix 12.2 vs 12.7 M as calls). */
template <bool kCallCold = false, class Env>
__device__ __forceinline__ bool run_body(int func_id, const Env& e, const void* args)
{
    if constexpr (kCallCold) {
        switch (func_id) {
        case PAGODA_MB: as_call<Env, pagoda_mb_args, body_mb<Env>>(e, *static_cast<const pagoda_mb_args*>(args)); return true;
        case PAGODA_FB: as_call<Env, pagoda_fb_args, body_fb<Env>>(e, *static_cast<const pagoda_fb_args*>(args)); return true;
        case PAGODA_BF: as_call<Env, pagoda_bf_args, body_bf<Env>>(e, *static_cast<const pagoda_bf_args*>(args)); return true;
        case PAGODA_CONV:
            as_call<Env, pagoda_conv_args, body_conv<Env>>(e, *static_cast<const pagoda_conv_args*>(args));
            return true;
        default: break;
        }
    }
    switch (func_id) {
    case PAGODA_NOP: return true;
    case PAGODA_MARK: body_mark(e, *static_cast<const pagoda_mark_args*>(args)); return true;
    case PAGODA_TID: body_tid(e, *static_cast<const pagoda_tid_args*>(args)); return true;
    case PAGODA_BAR: body_bar(e, *static_cast<const pagoda_bar_args*>(args)); return true;
    case PAGODA_SMEM: body_smem(e, *static_cast<const pagoda_smem_args*>(args)); return true;
    case PAGODA_SPIN: body_spin(e, *static_cast<const pagoda_spin_args*>(args)); return true;
    case PAGODA_GATE: body_gate(e, *static_cast<const pagoda_gate_args*>(args)); return true;
    case PAGODA_HOLD: body_hold(e, *static_cast<const pagoda_hold_args*>(args)); return true;
    case PAGODA_PAPER:
        if constexpr (IsTaskEnv<Env>::value) {
            body_paper(*static_cast<const pagoda_paper_args*>(args));
            return true;
        } else {
            return false;
        }
    case PAGODA_MB: body_mb(e, *static_cast<const pagoda_mb_args*>(args)); return true;
    case PAGODA_TDES: body_tdes(e, *static_cast<const pagoda_tdes_args*>(args)); return true;
    case PAGODA_MM: body_mm(e, *static_cast<const pagoda_mm_args*>(args)); return true;
    case PAGODA_FB: body_fb(e, *static_cast<const pagoda_fb_args*>(args)); return true;
    case PAGODA_BF: body_bf(e, *static_cast<const pagoda_bf_args*>(args)); return true;
    case PAGODA_CONV: body_conv(e, *static_cast<const pagoda_conv_args*>(args)); return true;
    case PAGODA_DCT: body_dct(e, *static_cast<const pagoda_dct_args*>(args)); return true;
    case PAGODA_MM_TC: body_mm_tc(e, *static_cast<const pagoda_mm_args*>(args)); return true;
    case PAGODA_MM64: body_mm64(e, *static_cast<const pagoda_mm_args*>(args)); return true;
    default: return false;
    }
}

__host__ __device__ inline bool known_func(int f)
{
    return (f >= PAGODA_NOP && f <= PAGODA_PAPER) || (f >= PAGODA_MB && f <= PAGODA_MM64);
}

} // namespace pagoda
#endif
