/*
 * master_kernel.cu — the persistent MasterKernel (Fig. 1b).
 *
 * Grid: one cooperative launch of n_mtb = num_sms * mtbs_per_sm thread blocks
 * ("MTBs") of 1024 threads.  The paper makes warp 0 of every MTB its
 * scheduler and warps 1..31 executors; here every warp executes and
 * the scheduler is a token the warps pass around (self-scheduling, see below).
 * Warp 31 of MTB 0 is instead the ingest warp that moves published TaskTable
 * entries from the pinned host ring into the device ring.
 *
 *   host ring --(ingest: LDGSTS over PCIe -> smem -> L2 device ring)--> device ring
 *   device ring --(scheduler: fetch-add tickets, per-cell sequence numbers)--> MTB task slots
 *   task slot --(place: warps / granules / barrier from bitmaps)--> WarpTable + mbarrier arrive
 *   executor warp --(body)--> mailboxes (deferred free) + completion record (D->H)
 *
 * Memory-model notes are inline; DESIGN.md "Ordering" has the full argument.
 */
#include <cuda_runtime.h>
#include <stdint.h>
#include <stdio.h>

#include "bodies.cuh"
#include "mk_layout.cuh"
/* A/B switches (scripts/build_variants.sh) */
#ifndef PAGODA_IDLE_NS
#define PAGODA_IDLE_NS 1024   /* longest back-off of an idle scheduler / I/O warp between polls */
#endif
#ifndef PAGODA_CTA_FENCE
#define PAGODA_CTA_FENCE 1    /* executors release with a CTA-scope fence (the poster's GPU fence covers them) */
#endif
#ifndef PAGODA_CLAIM_FIRST
#define PAGODA_CLAIM_FIRST 0  /* a scheduling round claims before it loads: fresh tickets load in the same round */
#endif
#ifndef PAGODA_CELL_ACQ
#define PAGODA_CELL_ACQ 1     /* ring cells are read with acquire loads and handed back with relaxed stores */
#endif
#ifndef PAGODA_LOOKAHEAD
#define PAGODA_LOOKAHEAD 1    /* tickets claimed beyond what the free warps fit now */
#endif
#ifndef PAGODA_CLAIM_MIN
#define PAGODA_CLAIM_MIN 1    /* with tickets queued, claim only when at least this many are wanted */
#endif
#ifndef PAGODA_WAKE_HINT_NS
#define PAGODA_WAKE_HINT_NS 1000000   /* suspend-time hint of an idle executor's mbarrier try_wait */
#endif
#ifndef PAGODA_FUSED_CLAIM
#define PAGODA_FUSED_CLAIM 0  /* claim, tail/head reads and publication checks in one round trip */
#endif
#ifndef PAGODA_CLAIM_FAIR
#define PAGODA_CLAIM_FAIR 0   /* claims take at most max(CLAIM_SMALL, backlog / n_mtb) tickets */
#endif
#ifndef PAGODA_SMALL_MULT
#define PAGODA_SMALL_MULT 8   /* (not FAIR) backlog below n_mtb x this: CLAIM_SMALL tickets per claim */
#endif
#ifndef PAGODA_CLAIM_SMALL
#define PAGODA_CLAIM_SMALL 1  /* tickets per claim while the backlog is below what all MTBs could take */
#endif
#ifndef PAGODA_FAST_LOAD
#define PAGODA_FAST_LOAD 0    /* ring cells are copied 4 lanes per cell with relaxed 16-byte loads all in
                                 flight together (one L2 round trip; the cells' sequence words were already
                                 acquired), not 4 serial acquire loads per cell */
#endif
#ifndef PAGODA_CELL_RELAXED
#define PAGODA_CELL_RELAXED 1 /* (FAST_LOAD 0) a lane's four cell loads relaxed + one CTA fence, not four serial
                                 acquires (measured +1-2 % on 3DES / MM / NOP) */
#endif
#ifndef PAGODA_FAST_PUB
#define PAGODA_FAST_PUB 1     /* a publisher checks 256 cells with relaxed loads all in flight, then one
                                 acquire fence (not 8 serial acquire loads per lane) */
#endif
#ifndef PAGODA_DIRECT_POST
#define PAGODA_DIRECT_POST 0  /* task MTBs always write completion records straight to the host window (one
                                 system-scope fence per batch) instead of the device queue + forwarders */
#endif
#ifndef PAGODA_DIRECT_IDLE_NS
#define PAGODA_DIRECT_IDLE_NS 50000   /* ... or when the group posted nothing for this long (lone tasks) */
#endif
#ifndef PAGODA_LOAD_AHEAD
#define PAGODA_LOAD_AHEAD 0   /* a holder that placed itself loads its claimed tickets before handing off (measured:
                                 MM 57.1 -> 54.8 M, the holder's own warp starts later; 3DES, mix neutral) */
#endif
#ifndef PAGODA_FREE_BEFORE_POST
#define PAGODA_FREE_BEFORE_POST 1  /* a task's last warp frees itself before posting the completion record */
#endif
#ifndef PAGODA_HOLDER_POSTS
#define PAGODA_HOLDER_POSTS 0 /* the scheduler token holder posts completion records (batched per round);
                                 the last warp of a task only marks it pending and frees itself */
#endif

namespace pagoda {


/* ------------------------------------------------------------------ PTX helpers */
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count)
{
    asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_arrive(uint64_t* bar)
{   /* .release.cta by default: the WarpTable slot written before is visible to the waiter */
    asm volatile("mbarrier.arrive.shared::cta.b64 _, [%0];" ::"r"(smem_u32(bar)) : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity)
{   /* try_wait suspends the warp in hardware (no issue slots burnt while idle) */
    uint32_t done = 0;
    const uint32_t a = smem_u32(bar);
    while (!done) {
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(a), "r"(parity), "n"(PAGODA_WAKE_HINT_NS)
            : "memory");
    }
}
/* An idle executor's wait for its dispatch mbarrier (exec_bar[warp], at the start of the MTB's
 * control block).  A warp suspended in try_wait is woken by mbarrier traffic anywhere in the CTA,
 * so idle warps run this loop millions of times per session; the loop therefore recomputes its
 * barrier address from %tid (two ALU ops) every trip instead of keeping it live across the task
 * body, where the 32-register build spilled it: a local-memory load per trip put idle warps on
 * the load/store pipe the busy warps' bodies need (ncu source counters). */
#ifndef PAGODA_WAIT_SLEEP_MAX
#define PAGODA_WAIT_SLEEP_MAX 0      /* 0: wait in mbarrier.try_wait (suspend); else test + nanosleep back-off (ns cap)
                                        (measured: no throughput difference; the suspension wakes sooner) */
#endif
__device__ __forceinline__ void exec_wait(uint32_t parity)
{
    extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
    uint32_t done = 0;
#if PAGODA_WAIT_SLEEP_MAX
    /* A warp suspended in try_wait is woken by ANY mbarrier traffic of the CTA (every dispatch of
     * every task), so idle warps re-check their barrier every few tens of ns: the check and the
     * re-suspend are two thirds of all instructions a 3DES session issues (ncu source counters,
     * DESIGN.md §8).  This variant tests without blocking, then sleeps (doubling from 64 ns up to
     * the cap).  Measured: the same throughput on every workload (the idle instructions use
     * issue slots the busy warps did not need), so the default stays the prompt suspension. */
    uint32_t ns = 64;
    for (;;) {
        uint32_t tid;
        asm volatile("mov.u32 %0, %%tid.x;" : "=r"(tid));
        const uint32_t a = smem_u32(pagoda_mk_smem) + ((tid >> 5) << 3);   /* &S.exec_bar[warp] */
        asm volatile("{ .reg .pred p; mbarrier.test_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                     : "=r"(done)
                     : "r"(a), "r"(parity)
                     : "memory");
        if (done) return;
        __nanosleep(ns);
        ns = min(ns * 2u, (uint32_t)PAGODA_WAIT_SLEEP_MAX);
    }
#else
    while (!done) {
        uint32_t tid;
        asm volatile("mov.u32 %0, %%tid.x;" : "=r"(tid));
        const uint32_t a = smem_u32(pagoda_mk_smem) + ((tid >> 5) << 3);   /* &S.exec_bar[warp] */
        asm volatile(
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(a), "r"(parity), "n"(PAGODA_WAKE_HINT_NS)
            : "memory");
    }
#endif
}
__device__ __forceinline__ void fence_acq_rel_gpu()
{
    asm volatile("fence.acq_rel.gpu;" ::: "memory");
}
__device__ __forceinline__ bool mbar_try_wait(uint64_t* bar, uint32_t parity, uint32_t hint_ns)
{
    uint32_t done;
    asm volatile(
        "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, %3; selp.u32 %0, 1, 0, p; }"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity), "r"(hint_ns)
        : "memory");
    return done != 0;
}
__device__ __forceinline__ uint64_t ld_acquire_gpu(const uint64_t* p)
{
    uint64_t v;
    asm volatile("ld.acquire.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_acquire_gpu32(const uint32_t* p)
{
    uint32_t v;
    asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_relaxed_gpu(const uint64_t* p)
{
    uint64_t v;
    asm volatile("ld.relaxed.gpu.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint64_t ld_acquire_sys(const volatile uint64_t* p)
{
    uint64_t v;
    asm volatile("ld.acquire.sys.global.u64 %0, [%1];" : "=l"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_acquire_sys32(const volatile uint32_t* p)
{
    uint32_t v;
    asm volatile("ld.acquire.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ uint32_t ld_relaxed_sys32(const volatile uint32_t* p)
{
    uint32_t v;
    asm volatile("ld.relaxed.sys.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_gpu(uint64_t* p, uint64_t v)
{
    asm volatile("st.release.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu(uint64_t* p, uint64_t v)
{
    asm volatile("st.relaxed.gpu.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_gpu32(uint32_t* p, uint32_t v)
{
    asm volatile("st.relaxed.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ uint32_t ld_relaxed_gpu32(const uint32_t* p)
{
    uint32_t v;
    asm volatile("ld.relaxed.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
    return v;
}
__device__ __forceinline__ void st_release_gpu32(uint32_t* p, uint32_t v)
{
    asm volatile("st.release.gpu.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void st_release_sys(volatile int64_t* p, int64_t v)
{
    asm volatile("st.release.sys.global.s64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys(volatile uint64_t* p, uint64_t v)
{
    asm volatile("st.relaxed.sys.global.u64 [%0], %1;" ::"l"(p), "l"(v) : "memory");
}
__device__ __forceinline__ void st_relaxed_sys32(volatile uint32_t* p, uint32_t v)
{
    asm volatile("st.relaxed.sys.global.u32 [%0], %1;" ::"l"(p), "r"(v) : "memory");
}
__device__ __forceinline__ void cp_async16(void* smem, const void* gmem)
{
    asm volatile("cp.async.cg.shared.global [%0], [%1], 16;" ::"r"(smem_u32(smem)), "l"(gmem) : "memory");
}
__device__ __forceinline__ void cp_async_wait_all()
{
    asm volatile("cp.async.commit_group;\n\tcp.async.wait_group 0;" ::: "memory");
}

/* ------------------------------------------------------------------ granule bitmap
 * Lane l of the scheduler warp owns granules [32l, 32l+32) (bit = 1: free).
 * Replaces the paper's buddy tree (§5.1) with a first-fit over a
 * bitmap: no power-of-two rounding, same scheduler-only (lock-free) ownership. */
__device__ __forceinline__ uint32_t bm_shr(uint32_t R, uint32_t s, uint32_t lane)
{   /* (multi-lane value R) >> s: position p gets bit p + s */
    const uint32_t q = s >> 5, r = s & 31u;
    uint32_t lo = __shfl_sync(0xffffffffu, R, (lane + q) & 31u);
    uint32_t hi = __shfl_sync(0xffffffffu, R, (lane + q + 1) & 31u);
    if (lane + q > 31u) lo = 0;
    if (lane + q + 1 > 31u) hi = 0;
    return r ? ((lo >> r) | (hi << (32u - r))) : lo;
}
/* lowest start of g consecutive free granules, or -1 */
__device__ __forceinline__ int bm_first_fit(uint32_t fg, uint32_t g, uint32_t lane)
{
    uint32_t R = fg, len = 1;
    while (len * 2u <= g) {
        R &= bm_shr(R, len, lane);
        len *= 2u;
    }
    if (g > len) R &= bm_shr(R, g - len, lane);
    const uint32_t b = __ballot_sync(0xffffffffu, R != 0);
    if (!b) return -1;
    const uint32_t L = __ffs(b) - 1;
    const uint32_t w = __shfl_sync(0xffffffffu, R, L);
    return (int)(L * 32u + __ffs(w) - 1);
}
/* The same for g <= 32 without shuffles: the lowest run of g free granules that lies inside one
 * lane's 32-granule word (runs across two words are left to bm_first_fit).  Shuffles travel the
 * shared-memory crossbar the task bodies keep busy; the holder's place step was the largest share
 * of its time under load (scripts/probe_prof.py). */
__device__ __forceinline__ int bm_first_fit_local(uint32_t fg, uint32_t g)
{
    uint32_t R = fg, len = 1;
    while (len * 2u <= g) {
        R &= R >> len;
        len *= 2u;
    }
    if (g > len) R &= R >> (g - len);
    const uint32_t b = __ballot_sync(0xffffffffu, R != 0);
    if (!b) return -1;
    const uint32_t L = __ffs(b) - 1;
    const uint32_t w = __shfl_sync(0xffffffffu, R, L);
    return (int)(L * 32u + __ffs(w) - 1);
}
#ifndef PAGODA_LOCAL_FIT
#define PAGODA_LOCAL_FIT 1
#endif
__device__ __forceinline__ int bm_fit(uint32_t fg, uint32_t g, uint32_t lane)
{
    if (PAGODA_LOCAL_FIT && g <= 32u) {
        const int o = bm_first_fit_local(fg, g);
        if (o >= 0) return o;
    }
    return bm_first_fit(fg, g, lane);
}
__device__ __forceinline__ uint32_t bm_range_bits(uint32_t off, uint32_t g, uint32_t lane)
{
    const uint32_t lo = max(off, lane * 32u), hi = min(off + g, lane * 32u + 32u);
    if (lo >= hi) return 0;
    const uint32_t n = hi - lo;
    return (n == 32u ? 0xffffffffu : ((1u << n) - 1u)) << (lo - lane * 32u);
}

/* scheduler counters: holder-private shared-memory words, added to DevCtl.ctr at exit */
enum { kScRounds = 0, kScProgress, kScTickets, kScClaimEmpty, kScLoadNotReady, kScPlaced, kScNoFit, kScHandoffs };
__device__ __forceinline__ void sc_add(SchedGroup& G, int i, uint32_t v)
{
    if ((threadIdx.x & 31u) == 0) G.sctr[i] += v;
}

/* profiling builds: ns per scheduler phase (holder-private) and per executor step */
#ifndef PAGODA_PROFILE
#define PAGODA_PROFILE 0
#endif
enum { kPfFold = 0, kPfLoad, kPfPlace, kPfClaim, kPfSleep, kPfBody, kPfFence, kPfPost };
__device__ __forceinline__ uint64_t pf_now() { return PAGODA_PROFILE ? globaltimer_ns() : 0; }
__device__ __forceinline__ void pf_add(SchedGroup& G, int i, uint64_t t0, bool shared_atomic)
{
    if (!PAGODA_PROFILE || (threadIdx.x & 31u) != 0) return;
    const unsigned long long d = globaltimer_ns() - t0;
    if (shared_atomic) atomicAdd(&G.sprof[i], d);
    else G.sprof[i] += d;
}

/* ------------------------------------------------------------------ life cycle stamps (PAGODA_LIFECYCLE) */
__device__ __forceinline__ uint64_t* life_slot(const MkParams& p, uint64_t id, int ev)
{
    return p.life + ((id & p.comp_mask) * 8u + (uint32_t)ev);
}
__device__ __forceinline__ void life_stamp(const MkParams& p, uint64_t id, int ev)
{
    if (p.life) *life_slot(p, id, ev) = globaltimer_ns();
}

/* ------------------------------------------------------------------ trace */
__device__ __forceinline__ void trace_ev(const MkParams& p, int mtb, uint32_t& seq, uint8_t kind, uint64_t task_id,
                                         uint16_t tb, uint32_t mask, uint16_t goff, uint16_t glen, uint8_t bar)
{
    if (p.trace_cap == 0) return;
    if ((threadIdx.x & 31u) == 0) {
        if (seq < p.trace_cap) {
            LedgerEvent e;
            e.seq = seq; e.mtb = (uint16_t)mtb; e.kind = kind; e.bar_id = bar; e.task_id = task_id;
            e.warp_mask = mask; e.tb = tb; e.gran_off = goff; e.gran_len = glen; e.pad = 0;
            e.pad2 = (uint32_t)globaltimer_ns();   /* low 32 bits of the event's %globaltimer (profiling) */
            p.trace[(size_t)mtb * p.trace_cap + seq] = e;
        }
        p.trace_count[mtb] = seq + 1;
    }
    seq++;
}

/* ------------------------------------------------------------------ completion records
 * A fence waits for every memory operation in flight on its SM, any warp's,
 * including posted PCIe writes to pinned host memory, which crawl while copy
 * engines keep the link busy (scripts/micro/membar_probe.cu; DESIGN.md
 * "PCIe isolation").  So SMs that run tasks never touch host memory: the last
 * warp of a task marks its slot in comp_pending; whichever warp holds the
 * MTB's poster flag releases the tasks' writes with one GPU-scope fence and
 * appends their ids to the device completion queue (one fetch-add per batch);
 * MTB 0's forwarder moves them to the host's completion window.  With a single
 * MTB there is no such split: the record goes to the host directly behind a
 * system-scope fence.  The task slot is returned (mb_tasks) only after its id
 * was read, so the id stays valid until then. */
__device__ __forceinline__ void post_completions(MtbShared& S, SchedGroup& G, const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    for (;;) {
        uint32_t got = 0;
        if (lane == 0) got = atomicExch(&G.poster, 1u) == 0u;
        if (!__shfl_sync(0xffffffffu, got, 0)) return;   /* the holder will see our bit */
        for (;;) {
            uint32_t m = 0;
            if (lane == 0) m = atomicExch(&G.comp_pending, 0u);
            m = __shfl_sync(0xffffffffu, m, 0);
            if (!m) break;
            const bool done = (m >> lane) & 1u;
            const uint64_t id = done ? S.tasks[lane].id : 0;
            bool mine = done;
            if (__any_sync(0xffffffffu, done && (S.tasks[lane].flags & kEntryGroup))) {
                /* entries of a spread task: count its finished TBs; the entry completing the last posts
                 * the task (release of this entry's writes before the count, acquire of the others' after) */
                fence_acq_rel_gpu();
                if (done && (S.tasks[lane].flags & kEntryGroup)) {
                    const TaskEntry& te = S.tasks[lane];
                    uint32_t* g = &p.grp[id & p.comp_mask];
                    const uint32_t ntb_all = te.reserved >> 16;
                    mine = atomicAdd(g, (uint32_t)te.n_tb) + te.n_tb == ntb_all;
                    if (mine) atomicExch(g, 0u);   /* every other entry of the task has added */
                }
                fence_acq_rel_gpu();
            }
            /* A lone task skips the forwarder hop: the group's last post is long ago, so its SM is quiet
             * and a system-scope fence is cheap.  Under load the queue path stays (a system fence on an
             * SM full of memory traffic waits for all of it: MM -12 % if every post went direct). */
            uint32_t direct = (p.n_mtb == 1 || PAGODA_DIRECT_POST) ? 1u : 0u;
            if (!direct && PAGODA_DIRECT_IDLE_NS) {
                if (lane == 0) {
                    const unsigned long long now = globaltimer_ns();
                    direct = now - G.last_post > (unsigned long long)PAGODA_DIRECT_IDLE_NS;
                    G.last_post = now;
                }
                direct = __shfl_sync(0xffffffffu, direct, 0);
            }
            if (direct) {
                asm volatile("fence.acq_rel.sys;" ::: "memory");
                if (mine) st_relaxed_sys(reinterpret_cast<volatile uint64_t*>(&p.comp[id & p.comp_mask]), id);
                if (mine) life_stamp(p, id, kLifeQueued);
                if (mine && p.n_mtb > 1) life_stamp(p, id, kLifeFwd);   /* in the host window already: no hop */
            } else {
                /* queue positions below dq_safe were cleared by the forwarders (their cursors, read
                 * by an acquire below when a position reaches the horizon) */
                const uint64_t safe = *(volatile unsigned long long*)&S.dq_safe;
                fence_acq_rel_gpu();   /* release: the tasks' writes (fenced by each of their warps) */
                const uint32_t pm = __ballot_sync(0xffffffffu, mine);
                unsigned long long base = 0;
                if (lane == 0 && pm) base = atomicAdd(reinterpret_cast<unsigned long long*>(&p.dctl->dq_tail),
                                                      (unsigned long long)__popc(pm));
                base = __shfl_sync(0xffffffffu, base, 0);
                const uint64_t slot = base + (uint64_t)__popc(pm & ((1u << lane) - 1u));
                if (__any_sync(0xffffffffu, mine && slot >= safe)) {   /* refresh the horizon */
                    uint64_t m = 0;
                    m = lane < p.n_fwd ? ld_acquire_gpu(&p.dctl->fwd_cur[lane]) : ~0ull;
                    for (uint32_t o = 1; o < kForwarders; o <<= 1) m = min(m, __shfl_xor_sync(0xffffffffu, m, o));
                    if (lane == 0) atomicMax(&S.dq_safe, (unsigned long long)(m + kDqEntries));
                }
                if (mine) {
                    uint64_t* q = &p.dq[slot & p.dq_mask];
                    if (slot >= safe)
                        while (*(volatile uint64_t*)q != 0) __nanosleep(64);   /* previous lap not forwarded yet */
                    st_relaxed_gpu(q, id + 1);
                    life_stamp(p, id, kLifeQueued);
                }
            }
            __syncwarp();
            if (lane == 0) {
                __threadfence_block();
                atomicOr(&G.mb_tasks, m);   /* the scheduler may now reuse those task slots */
            }
        }
        uint32_t again = 0;
        if (lane == 0) {
            atomicExch(&G.poster, 0u);
            __threadfence_block();   /* release the flag, then re-check: a bit set meanwhile by a */
            again = *(volatile uint32_t*)&G.comp_pending != 0u;   /* warp that found the flag taken */
        }
        if (!__shfl_sync(0xffffffffu, again, 0)) return;
    }
}

/* The poster behind a call: the 4-MTB/SM kernel (run_task<kCallCold>) takes it (its executor
 * spills less: MM 60.9 -> 62.9 M tasks/s); inlined elsewhere (mix as a call 12.9 -> 12.35 M). */
__device__ __noinline__ void post_completions_call(MtbShared& S, SchedGroup& G, const MkParams& p)
{
    post_completions(S, G, p);
}

/* MTB 0's forwarders (n_mtb > 1): completion queue -> the host's completion
 * window.  Forwarder f owns the queue chunks (kFwdChunk records) whose index
 * is f mod kForwarders and walks them in order.  Per sweep: the run of filled
 * records at its cursor (up to the chunk's end, 8 loads per lane in flight),
 * one system-scope fence (cumulative: orders the task writes the posters
 * released), then post the records and clear their queue slots.  The fence of
 * the NEXT sweep also orders those clears before the cursor's publication
 * (fwd_cur, the posters' wrap check).  Each exits once every MTB exited and
 * no record is left at or past its cursor; the last one out records where the
 * next session resumes. */
__device__ void comp_forwarder(MtbShared& S, const MkParams& p, uint32_t f)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t K = p.n_fwd, CH = kFwdChunk;
    uint64_t c = *(volatile uint64_t*)&p.dctl->dq_head;
    {   /* first position >= c in a chunk of mine */
        const uint64_t ch = c / CH, o = (f + K - ch % K) % K;
        if (o) c = (ch + o) * CH;
    }
    uint64_t published = ~0ull;
    uint32_t idle = 0;
    for (;;) {
        const uint32_t span = (uint32_t)((c / CH + 1) * CH - c);   /* records left in this chunk */
        uint64_t v[8];
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const uint32_t k = (uint32_t)i * 32u + lane;
            v[i] = k < span ? *(volatile uint64_t*)&p.dq[(c + k) & p.dq_mask] : 0;
        }
        uint32_t n = 0;
        bool gap = false;
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const uint32_t full = __ballot_sync(0xffffffffu, v[i] != 0);
            if (!gap) {
                if (full == 0xffffffffu) n += 32u;
                else {
                    n += (uint32_t)__ffs(~full) - 1u;
                    gap = true;
                }
            }
        }
        n = min(n, span);
        if (n == 0) {
            uint32_t done = 0;
            /* acquire of the exit count orders the tail read after it: every MTB's reservations
             * (made before its release-ordered exit increment) are then in the tail we read */
            if (lane == 0) done = ld_acquire_gpu32(&p.dctl->exited) >= p.n_exit &&
                                  ld_relaxed_gpu(&p.dctl->dq_tail) <= c;
            if (__shfl_sync(0xffffffffu, done, 0)) break;
            __nanosleep(idle < 16 ? 64 : min(512, PAGODA_IDLE_NS));
            idle++;
            continue;
        }
        idle = 0;
        asm volatile("fence.acq_rel.sys;" ::: "memory");
        if (lane == 0 && published != c) {   /* the previous sweeps' clears are ordered before this */
            st_relaxed_gpu(&p.dctl->fwd_cur[f], c);
            published = c;
        }
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const uint32_t k = (uint32_t)i * 32u + lane;
            if (k < n) {
                const uint64_t id = v[i] - 1;
                st_relaxed_sys(reinterpret_cast<volatile uint64_t*>(&p.comp[id & p.comp_mask]), id);
                life_stamp(p, id, kLifeFwd);
                st_relaxed_gpu(&p.dq[(c + k) & p.dq_mask], 0);
            }
        }
        __syncwarp();
        c += n;
        if (n == span) c += (K - 1) * CH;   /* chunk done: my next one */
    }
    if (lane == 0 && atomicAdd(&S.fwd_done, 1u) + 1u == (uint32_t)K) {
        /* every record below the final tail was forwarded: the next session resumes there */
        const uint64_t t = *(volatile uint64_t*)&p.dctl->dq_tail;
        *(volatile uint64_t*)&p.dctl->dq_head = t;
        for (uint32_t i = 0; i < 4; i++) *(volatile uint64_t*)&p.dctl->fwd_cur[i] = t;
    }
}

/* ------------------------------------------------------------------ task execution
 * Alg. 1 L29-43: run the body, then the deferred release: the last
 * warp of a TB returns its shmem granules and barrier ID through the mailbox
 * (markSMForDealloc), the last warp of the task posts its completion record,
 * every warp returns itself. */
template <bool kCallCold>
__device__ __forceinline__ void run_task(MtbShared& S, SchedGroup& G, char* smem_base, const MkParams& p, int mtb,
                                         int vmtb, int w, uint32_t resident)
{
    const uint32_t lane = threadIdx.x & 31u;
    const WarpSlot& s = S.wt[w];   /* read from shared memory when needed */
    const TaskEntry& t = S.tasks[s.task];
    uint64_t t0 = 0;
    if (p.trace_cap) t0 = globaltimer_ns();
    TaskEnv env{&p.dctl->error, resident};
    if (p.life && lane == 0)   /* the first warp to start stamps the body start */
        atomicCAS(reinterpret_cast<unsigned long long*>(life_slot(p, s.task_id, kLifeStart)), 0ull,
                  (unsigned long long)globaltimer_ns());
    uint64_t tp = pf_now();
    if (!run_body<kCallCold>(t.func_id, env, t.args) && lane == 0) atomicOr(&p.dctl->error, PAGODA_DEVERR_BAD_FUNC);
    __syncwarp();
    pf_add(G, kPfBody, tp, true);
    if (p.life && lane == 0)
        atomicMax(reinterpret_cast<unsigned long long*>(life_slot(p, s.task_id, kLifeEnd)),
                  (unsigned long long)globaltimer_ns());
    tp = pf_now();
    uint32_t last = 0;
    if (lane == 0) {
        /* this warp's global writes -> visible GPU-wide before anyone learns the warp is done
         * (release; the completion poster's system-scope fence then publishes them to the host) */
#if PAGODA_CTA_FENCE
        /* CTA-scope release: the completion poster (same MTB) acquires it through the shared-memory
         * counters below and its GPU-scope fence then releases every warp's writes (cumulativity) */
        asm volatile("fence.acq_rel.cta;" ::: "memory");
#else
        asm volatile("fence.acq_rel.gpu;" ::: "memory");
#endif
        if (p.trace_cap) {
            uint32_t* cnt = &p.exec_count[mtb * 32 + w];
            const uint32_t i = *cnt;
            if (i < p.trace_cap) {
                uint32_t smid;
                asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
                ExecRecord r{s.task_id, s.tb, (uint16_t)smid, (uint16_t)vmtb, (uint16_t)w, t0, globaltimer_ns()};
                p.exec_trace[((size_t)mtb * 32 + w) * p.trace_cap + i] = r;
            }
            *cnt = i + 1;
        }
        if (atomicSub(&S.tb_warps_left[s.tbslot], 1u) == 1u) atomicOr(&G.mb_tbs, 1u << s.tbslot);
        if (atomicSub(&S.task_warps_left[s.task], 1u) == 1u) {
            /* last warp of the task (Alg. 1 L41-42): its completion record is pending */
            life_stamp(p, s.task_id, kLifeDone);
            atomicOr(&G.comp_pending, 1u << s.task);
            __threadfence_block();   /* pending bit before the poster-flag attempt */
            last = 1;
        }
    }
    pf_add(G, kPfFence, tp, true);
    if (PAGODA_FREE_BEFORE_POST) {
        /* the warp is free for the next task before it posts: the post (a GPU fence and a queue
         * reservation, ~3 us under load) overlaps the next placement and wake-up instead of holding
         * the slot's warps.  Its WarpTable slot may be rewritten meanwhile; the post reads task
         * slots only (returned after it), and the holder does not exit while a post is running. */
        if (lane == 0) {
            __threadfence_block();
            atomicOr(&G.mb_warps, 1u << w);
            __threadfence_block();
        }
        __syncwarp();
    }
    tp = pf_now();
    if (!PAGODA_HOLDER_POSTS && __shfl_sync(0xffffffffu, last, 0)) {
        if constexpr (kCallCold) post_completions_call(S, G, p);
        else post_completions(S, G, p);
    }
    pf_add(G, kPfPost, tp, true);
    if (!PAGODA_FREE_BEFORE_POST) {
        if (lane == 0) {
            __threadfence_block();   /* TB / task frees are visible before the warp frees itself */
            atomicOr(&G.mb_warps, 1u << w);
            __threadfence_block();   /* ... and the warp's free bit before its attempt at the token */
        }
        __syncwarp();
    }
}

/* MTB 0's host poster (n_mtb > 1): the ingest warp's host-visible stores
 * (consumed count, device error word) are made here, so that the ingest warp's
 * own fences never wait for a posted PCIe write.  Exits after every MTB did. */
__device__ void host_poster(MtbShared& S, const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    if (lane != 0) return;
    uint64_t last = ~0ull;
    uint32_t last_err = 0;
    for (;;) {
        const uint32_t done = *(volatile uint32_t*)&S.ingest_done;
        const uint32_t exited = *(volatile uint32_t*)&p.dctl->exited;
        const uint64_t c = *(volatile uint64_t*)&S.ingest_copied;
        const uint32_t err = *(volatile uint32_t*)&p.dctl->error;
        if (c != last && !p.ce_ingest) {   /* (CE ingest: the copy stream writes consumed) */
            st_relaxed_sys(&p.hctl->consumed, c);
            last = c;
        }
        if (err != last_err) {
            st_relaxed_sys32(&p.hctl->error, err);
            last_err = err;
        }
        if (done && exited >= p.n_exit) break;
        __nanosleep(256);
    }
}

/* ------------------------------------------------------------------ ingest
 * Replaces the paper's one-cudaMemcpy-per-spawn with ready-field pipelining
 * (P:516-539): the host publishes a doorbell after writing entries; this warp
 * acquires it over PCIe, pulls the entries with asynchronous 16-byte copies
 * (many in flight, no registers held) into shared memory and publishes them
 * into the device ring, a bounded MPMC queue with one sequence word per cell:
 * the producer may fill the cell of position t once seq == t (its previous
 * occupant was consumed), then releases seq = t + 1. */
/* stage sizes: ingest_stage_entries() in mk_layout.cuh */

__device__ __forceinline__ void tma_load_1d(void* smem_dst, const void* gsrc, uint32_t bytes, uint64_t* bar)
{
    asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                     smem_u32(smem_dst)),
                 "l"(gsrc), "r"(bytes), "r"(smem_u32(bar))
                 : "memory");
}
__device__ __forceinline__ void tma_store_1d(void* gdst, const void* smem_src, uint32_t bytes)
{
    asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;" ::"l"(gdst), "r"(smem_u32(smem_src)),
                 "r"(bytes)
                 : "memory");
}

#ifndef PAGODA_INGEST_TIMERS
#define PAGODA_INGEST_TIMERS 1   /* ingest phase timers (PAGODA_CTR_INGEST_NS_*) */
#endif
__device__ __forceinline__ uint64_t ing_now() { return PAGODA_INGEST_TIMERS ? globaltimer_ns() : 0; }
struct IngestCtr {
    unsigned long long batches = 0, entries = 0, ns_db = 0, ns_copy = 0, ns_pub = 0, full = 0, ns_fence = 0,
                       ns_store = 0;
};

/* Publish one staged batch [s, s+n) into the device ring: wait until its cells
 * are free (seq == position: previous occupants loaded), acquire, bulk-store
 * the entries, order them before the cells' release (seq = position + 1). */
#ifndef PAGODA_EARLY_CHECK
#define PAGODA_EARLY_CHECK 0  /* (measured neutral) publishers check a stage's ring cells from its header, while its bytes cross PCIe */
#endif
#ifndef PAGODA_EARLY_EMPTY
#define PAGODA_EARLY_EMPTY 0  /* a stage is handed back to the loader once the bulk store has READ it, before the
                                 store completes and the cells are released (the stage's next fill overlaps them) */
#endif
/* Wait until the cells of positions [s, s+n) are free (seq == position: previous occupants loaded),
 * with relaxed loads (the caller's acquire fence completes the pattern).  False on abort. */
__device__ __forceinline__ bool ingest_check_cells(const MkParams& p, uint64_t s, uint32_t n, IngestCtr& c)
{
    const uint32_t lane = threadIdx.x & 31u;
    for (uint32_t base = 0; base < n;) {   /* 256 cells per round trip (8 loads per lane) */
        uint32_t sv[8];
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const uint32_t k = base + (uint32_t)i * 32u + lane;
            sv[i] = k < n ? ld_relaxed_gpu32(&p.dseq[(s + k) & p.ring_mask]) : (uint32_t)(s + k);
        }
        uint32_t bad = 0;
#pragma unroll
        for (int i = 0; i < 8; i++) bad |= __ballot_sync(0xffffffffu, sv[i] != (uint32_t)(s + base + (uint32_t)i * 32u + lane));
        if (bad) {
            c.full++;
            if (*(volatile uint32_t*)&p.dctl->stop == kStopAbort) return false;
            __nanosleep(128);
            continue;
        }
        base += 256u;
    }
    return true;
}

__device__ __forceinline__ bool ingest_publish(const MkParams& p, const char* src, uint64_t s, uint32_t n,
                                               IngestCtr& c, uint64_t* empty_bar = nullptr, bool checked = false)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t R = (uint64_t)p.ring_mask + 1;
    for (uint32_t base = checked ? n : 0u; base < n;) {   /* 256 cells per round trip (8 loads per lane) */
        uint32_t sv[8];
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const uint32_t k = base + (uint32_t)i * 32u + lane;
            /* the cell's previous reader is done: acquire (LDG.STRONG + L1 invalidate, no MEMBAR) per load,
             * or (FAST_PUB) relaxed loads all in flight at once, made an acquire by the fence below */
            sv[i] = k < n ? (PAGODA_FAST_PUB ? ld_relaxed_gpu32(&p.dseq[(s + k) & p.ring_mask])
                                             : ld_acquire_gpu32(&p.dseq[(s + k) & p.ring_mask]))
                          : (uint32_t)(s + k);
        }
        uint32_t bad = 0;
#pragma unroll
        for (int i = 0; i < 8; i++) bad |= __ballot_sync(0xffffffffu, sv[i] != (uint32_t)(s + base + (uint32_t)i * 32u + lane));
        if (bad) {   /* device ring full: wait for the schedulers */
            c.full++;
            if (*(volatile uint32_t*)&p.dctl->stop == kStopAbort) return false;
            __nanosleep(128);
            continue;
        }
        base += 256u;
    }
    if (PAGODA_FAST_PUB || checked) fence_acq_rel_gpu();   /* acquire pattern: relaxed reads of the cells, then this fence */
    const uint64_t t3 = ing_now();
    __syncwarp();          /* every lane's acquire precedes lane 0's bulk store */
    const uint64_t t4 = ing_now();
    if (lane == 0) {
        asm volatile("fence.proxy.async.global;" ::: "memory");   /* generic acquire -> async-proxy writes */
        asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
        const uint32_t e0 = (uint32_t)(s & p.ring_mask);
        const uint32_t n1 = min(n, (uint32_t)(R - e0));
        tma_store_1d(p.dring + e0, src, n1 * 64u);
        if (n1 < n) tma_store_1d(p.dring, src + n1 * 64u, (n - n1) * 64u);
        asm volatile("cp.async.bulk.commit_group;" ::: "memory");
        if (empty_bar) {   /* the stage's bytes have been read: the loader may refill it now */
            asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory");
            mbar_arrive(empty_bar);
        }
        asm volatile("cp.async.bulk.wait_group 0;" ::: "memory");
        asm volatile("fence.proxy.async.global;" ::: "memory");
    }
    __syncwarp();
    const uint64_t t5 = ing_now();
    fence_acq_rel_gpu();   /* the entry writes precede every lane's relaxed cell release */
    const uint64_t t6 = ing_now();
    c.ns_fence += (t4 - t3) + (t6 - t5);
    c.ns_store += t5 - t4;
    for (uint32_t i = lane; i < n; i += 32u) {
        const uint64_t t = s + i;
        st_relaxed_gpu32(&p.dseq[t & p.ring_mask], (uint32_t)(t + 1));
        if (p.life) life_stamp(p, reinterpret_cast<const TaskEntry*>(src)[i].id, kLifePub);
    }
    __syncwarp();
    /* hint for schedulers that work exists (publishers finish out of order: the max) */
    if (lane == 0) atomicMax(reinterpret_cast<unsigned long long*>(&p.dctl->tail), (unsigned long long)(s + n));
    c.batches++;
    c.entries += n;
    return true;
}

/* doorbell: lane 0 reads the host's published count and terminate word */
__device__ __forceinline__ void ingest_doorbell(const MkParams& p, uint64_t& pub, uint32_t& term, uint32_t& last_err,
                                                bool post_err, IngestCtr& c, uint64_t fetched)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t t0 = ing_now();
    uint32_t err = 0;
    if (lane == 0) {
        pub = ld_acquire_sys(&p.hctl->published);
        /* terminate matters only when nothing new was published: one PCIe round trip per poll otherwise */
        term = pub > fetched ? 0u : ld_relaxed_sys32(&p.hctl->terminate);
        if (term) {   /* the host publishes every entry of the session before it sets terminate: */
            term = ld_acquire_sys32(&p.hctl->terminate);   /* re-read the count after an acquire of it */
            pub = ld_acquire_sys(&p.hctl->published);       /* (so this count is final) */
        }
        err = *(volatile uint32_t*)&p.dctl->error;
        if (post_err && err != last_err) st_relaxed_sys32(&p.hctl->error, err);
    }
    pub = __shfl_sync(0xffffffffu, pub, 0);
    term = __shfl_sync(0xffffffffu, term, 0);
    last_err = __shfl_sync(0xffffffffu, err, 0);
    c.ns_db += ing_now() - t0;
}

/* issue the bulk copy of host ring entries [f, f+n) into a stage (lane 0) */
__device__ __forceinline__ void ingest_load(const MkParams& p, char* dst, uint64_t f, uint32_t n, uint64_t* bar)
{
    if ((threadIdx.x & 31u) != 0) return;
    const uint64_t R = (uint64_t)p.ring_mask + 1;
    asm volatile("fence.proxy.async.global;" ::: "memory");   /* the doorbell acquire orders these reads */
    const uint32_t e0 = (uint32_t)(f & p.ring_mask);
    const uint32_t n1 = min(n, (uint32_t)(R - e0));
    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(n * 64u) : "memory");
    tma_load_1d(dst, p.hring + e0, n1 * 64u, bar);
    if (n1 < n) tma_load_1d(dst + n1 * 64u, p.hring, (n - n1) * 64u, bar);
}

__device__ void ingest_flush(const MkParams& p, const IngestCtr& c)
{
    if ((threadIdx.x & 31u) != 0) return;
    if (c.batches) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_BATCHES], c.batches);
    if (c.entries) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_ENTRIES], c.entries);
    if (c.ns_db) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_NS_DOORBELL], c.ns_db);
    if (c.ns_copy) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_NS_COPY], c.ns_copy);
    if (c.ns_pub) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_NS_PUBLISH], c.ns_pub);
    if (c.full) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_RING_FULL], c.full);
    if (c.ns_fence) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_NS_FENCE], c.ns_fence);
    if (c.ns_store) atomicAdd(&p.dctl->ctr[PAGODA_CTR_INGEST_NS_STORE], c.ns_store);
}

/* Single-warp ingest (a context of one MTB, where MTB 0 also runs tasks): a
 * two-stage TMA pipeline, stage s pulled from the host ring while the other
 * is published; host-visible stores (consumed, error) made inline. */
__device__ void ingest(MtbShared& S, const MkParams& p, char* stage_buf, uint64_t* bars)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t SE = p.ingest_stage_entries;
    uint64_t copied = *(volatile uint64_t*)&p.dctl->tail;   /* published into the device ring (resumes) */
    uint64_t fetched = copied;                               /* loaded (or loading) into a stage */
    uint64_t pub = copied;                                   /* last doorbell value seen */
    uint64_t st_start[2] = {0, 0};
    uint32_t st_n[2] = {0, 0};
    uint32_t phase = 0, os = 0, ns = 0, inflight = 0, term = 0, last_err = 0;
    int idle = 0;
    IngestCtr c;
    for (;;) {
        if (fetched >= pub) {
            ingest_doorbell(p, pub, term, last_err, true, c, fetched);
            if (term == kStopAbort) {   /* host watchdog: abandon the queue, let idle MTBs exit */
                if (lane == 0) st_release_gpu32(&p.dctl->stop, kStopAbort);
                break;
            }
        }
        while (inflight < 2 && fetched < pub) {
            const uint32_t n = (uint32_t)min(pub - fetched, (uint64_t)SE);
            ingest_load(p, stage_buf + ns * (SE * 64u), fetched, n, &bars[ns]);
            st_start[ns] = fetched;
            st_n[ns] = n;
            fetched += n;
            ns ^= 1u;
            inflight++;
            idle = 0;
        }
        if (inflight) {
            const uint64_t t1 = ing_now();
            mbar_wait(&bars[os], (phase >> os) & 1u);
            phase ^= 1u << os;
            const uint64_t t2 = ing_now();
            c.ns_copy += t2 - t1;
            if (!ingest_publish(p, stage_buf + os * (SE * 64u), st_start[os], st_n[os], c)) break;
            copied = st_start[os] + st_n[os];
            if (lane == 0) st_relaxed_sys(&p.hctl->consumed, copied);   /* host may reuse those ring slots */
            c.ns_pub += ing_now() - t2;
            inflight--;
            os ^= 1u;
        } else if (term) {
            if (lane == 0) st_release_gpu32(&p.dctl->stop, 1u);
            break;
        } else if (++idle > 64) {
            __nanosleep(min(256, PAGODA_IDLE_NS));
        }
    }
    if (lane == 0) {
        *(volatile uint64_t*)&S.ingest_copied = copied;
        __threadfence_block();
        *(volatile uint32_t*)&S.ingest_done = 1u;
    }
    ingest_flush(p, c);
}

/* Multi-warp ingest (n_mtb > 1).  A fence waits for ALL of its warp's outstanding
 * memory operations, including a bulk read of the host ring still crossing a
 * busy PCIe link; so the warps that fence (the publishers) are not the warp
 * that reads host memory (the loader).  The loader fills kIngestStages stages
 * in ring order; stage k goes to buffer k mod kIngestStages and publisher
 * k mod kIngestPublishers, so each publisher owns every P-th stage, double-
 * buffered, and the publishers' per-batch latencies overlap.  Handshakes per
 * buffer: full[b] (bulk copy landed; an arrival without bytes and n = ~0 ends
 * a publisher's stream) and empty[b] (its publisher is done with it).
 * Publishers finish out of order; the contiguous published prefix (what the
 * host may reuse) advances over per-stage completion records. */
__device__ void ingest_loader(MtbShared& S, const MkParams& p, char* stage_buf)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t SE = p.ingest_stage_entries;
    uint64_t fetched = *(volatile uint64_t*)&p.dctl->tail;
    uint64_t pub = fetched;
    uint32_t term = 0, last_err = 0, k = 0, ends = 0;
    int idle = 0;
    IngestCtr c;
    for (;;) {
        if (fetched >= pub) {
            ingest_doorbell(p, pub, term, last_err, false, c, fetched);
            if (term == kStopAbort) {   /* host watchdog: the publishers see stop and leave too */
                if (lane == 0) st_release_gpu32(&p.dctl->stop, kStopAbort);
                break;
            }
        }
        const bool end = term && fetched >= pub;
        if (fetched < pub || end) {
            const uint32_t b = k % kIngestStages;
            if (k >= kIngestStages) mbar_wait(&S.ingest_empty[b], (k / kIngestStages - 1u) & 1u);   /* free again */
            k++;
            if (end) {   /* one end marker per publisher, in its next stage */
                if (lane == 0) {
                    S.ing_n[b] = ~0u;
                    __threadfence_block();
                    *(volatile uint32_t*)&S.ing_hdr[b] = k;   /* k was incremented above: stage k - 1 */
                    mbar_arrive(&S.ingest_bar[b]);
                }
                if (++ends == kIngestPublishers) break;
                continue;
            }
            const uint32_t n = (uint32_t)min(pub - fetched, (uint64_t)SE);
            if (lane == 0) {
                S.ing_start[b] = fetched;
                S.ing_n[b] = n;
                __threadfence_block();
                *(volatile uint32_t*)&S.ing_hdr[b] = k;   /* stage k - 1's header: its publisher checks the cells */
            }
            ingest_load(p, stage_buf + b * (SE * 64u), fetched, n, &S.ingest_bar[b]);
            fetched += n;
            idle = 0;
        } else if (++idle > 64) {
            __nanosleep(min(256, PAGODA_IDLE_NS));
        }
    }
    ingest_flush(p, c);
}

/* stage k was published (end position e): record it, then advance the
 * contiguous prefix as far as the records reach (one publisher at a time) */
__device__ __forceinline__ void ingest_finish(MtbShared& S, uint32_t k, uint64_t e)
{
    if ((threadIdx.x & 31u) != 0) return;
    const uint32_t slot = k % kIngestFinSlots;
    *(volatile uint64_t*)&S.ing_fin_end[slot] = e;
    __threadfence_block();
    *(volatile uint32_t*)&S.ing_fin[slot] = k + 1u;
    __threadfence_block();
    for (;;) {
        if (atomicCAS(&S.ing_lock, 0u, 1u) != 0u) return;   /* the holder re-checks after releasing */
        __threadfence_block();
        uint32_t q = *(volatile uint32_t*)&S.ing_prefix_k;
        uint64_t end = 0;
        bool moved = false;
        while (*(volatile uint32_t*)&S.ing_fin[q % kIngestFinSlots] == q + 1u) {
            end = *(volatile uint64_t*)&S.ing_fin_end[q % kIngestFinSlots];
            q++;
            moved = true;
        }
        if (moved) {
            *(volatile uint64_t*)&S.ingest_copied = end;   /* for the host poster */
            *(volatile uint32_t*)&S.ing_prefix_k = q;
        }
        __threadfence_block();
        atomicExch(&S.ing_lock, 0u);
        __threadfence_block();
        /* a record written while the lock was held may have been missed: look again */
        if (*(volatile uint32_t*)&S.ing_fin[q % kIngestFinSlots] != q + 1u) return;
    }
}

__device__ __noinline__ void ingest_publisher(MtbShared& S, const MkParams& p, char* stage_buf, uint32_t me)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t SE = p.ingest_stage_entries;
    bool aborted = false;
    IngestCtr c;
    for (uint32_t k = me;; k += kIngestPublishers) {   /* my stages: me, me + P, ... */
        const uint32_t b = k % kIngestStages;
        const uint64_t t1 = ing_now();
        bool checked = false;
        if (PAGODA_EARLY_CHECK) {
            /* the stage's header arrives before its bytes: check its cells while the host read is in
             * flight (the round trip leaves the publish chain); the acquire fence follows the load */
            while (*(volatile uint32_t*)&S.ing_hdr[b] != k + 1u) {
                if (*(volatile uint32_t*)&p.dctl->stop == kStopAbort) {
                    aborted = true;
                    break;
                }
                __nanosleep(32);
            }
            if (aborted) break;
            __syncwarp();
            __threadfence_block();   /* the header's fields after the header */
            const uint32_t n0 = *(volatile uint32_t*)&S.ing_n[b];
            if (n0 != ~0u) {
                if (!ingest_check_cells(p, *(volatile uint64_t*)&S.ing_start[b], n0, c)) {
                    aborted = true;
                    break;
                }
                checked = true;
            }
        }
        while (!mbar_try_wait(&S.ingest_bar[b], (k / kIngestStages) & 1u, 20000u)) {
            if (*(volatile uint32_t*)&p.dctl->stop == kStopAbort) {
                aborted = true;
                break;
            }
        }
        if (aborted) break;
        const uint64_t t2 = ing_now();
        const uint32_t n = *(volatile uint32_t*)&S.ing_n[b];
        if (n == ~0u) break;
        c.ns_copy += t2 - t1;
        const uint64_t s = *(volatile uint64_t*)&S.ing_start[b];
        if (!ingest_publish(p, stage_buf + b * (SE * 64u), s, n, c, PAGODA_EARLY_EMPTY ? &S.ingest_empty[b] : nullptr,
                            checked)) {
            aborted = true;
            break;
        }
        ingest_finish(S, k, s + n);
        if (!PAGODA_EARLY_EMPTY && lane == 0) mbar_arrive(&S.ingest_empty[b]);
        c.ns_pub += ing_now() - t2;
    }
    if (lane == 0) {
        /* the last publisher out: every stage was published (each saw its end marker after its
         * data stages), so the device ring's tail is final: drain and exit */
        if (atomicAdd(&S.ing_pubs_done, 1u) + 1u == kIngestPublishers) {
            if (!aborted && *(volatile uint32_t*)&p.dctl->stop != kStopAbort) st_release_gpu32(&p.dctl->stop, 1u);
            __threadfence_block();
            *(volatile uint32_t*)&S.ingest_done = 1u;
        }
    }
    ingest_flush(p, c);
}

/* PAGODA_CE_INGEST: MTB 0's scanner warp (in place of the ingest warps).  The host's copy stream
 * overwrites a device ring cell only once the ticket of the previous lap handed it back
 * (seq = position + R, stored by the scheduler after it copied the cell); this warp follows the
 * hand-backs in ring order and posts their contiguous prefix to the host (HostCtl.handed), 256
 * cells per L2 round trip.  With one MTB it also posts the device error word.  Exits once every
 * scheduler exited. */
__device__ void ce_scanner(const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t R = (uint64_t)p.ring_mask + 1;
    uint64_t P = p.ce_base, posted = ~0ull;
    uint32_t idle = 0, last_err = 0;
    for (;;) {
        uint32_t v[8];
#pragma unroll
        for (int i = 0; i < 8; i++) v[i] = ld_relaxed_gpu32(&p.dseq[(P + (uint64_t)i * 32u + lane) & p.ring_mask]);
        uint32_t n = 0;
        bool gap = false;
#pragma unroll
        for (int i = 0; i < 8; i++) {
            const uint32_t ok = __ballot_sync(0xffffffffu, v[i] == (uint32_t)(P + (uint64_t)i * 32u + lane + R));
            if (!gap) {
                if (ok == 0xffffffffu) n += 32u;
                else {
                    n += (uint32_t)__ffs(~ok) - 1u;
                    gap = true;
                }
            }
        }
        P += n;
        if (lane == 0) {
            if (P != posted && (n == 0 || P - posted >= 1024u || posted == ~0ull)) {
                st_relaxed_sys(reinterpret_cast<volatile uint64_t*>(&p.hctl->handed), P);
                posted = P;
            }
            if (p.n_mtb == 1) {
                const uint32_t err = *(volatile uint32_t*)&p.dctl->error;
                if (err != last_err) {
                    st_relaxed_sys32(&p.hctl->error, err);
                    last_err = err;
                }
            }
        }
        if (n) {
            idle = 0;
            continue;
        }
        uint32_t done = 0;
        if (lane == 0) done = ld_acquire_gpu32(&p.dctl->exited) >= p.n_exit;
        if (__shfl_sync(0xffffffffu, done, 0)) break;
        __nanosleep(idle < 16 ? 128 : min(1024, PAGODA_IDLE_NS));
        idle++;
    }
}

/* ------------------------------------------------------------------ scheduler
 * Alg. 1 L1-28 + Alg. 2, re-designed: one warp per MTB owns the
 * MTB's free masks (warps, TB records, task slots, barrier IDs: one word each;
 * granules: a 1024-bit lane-distributed bitmap).  It takes TICKETS (ring
 * positions) with one fetch-add on the device head, as many as its free warps
 * fit at the last task size seen, so no claim ever fails or retries; a ticket
 * is loaded into a task slot once its cell is published, and placed in FIFO
 * order as soon as the MTB has the resources. */
template <int kG>   /* kG: scheduling groups per MTB, a compile-time constant (the kernel is instantiated per count) */
struct Sched {
    static constexpr uint32_t rm = 32u / (uint32_t)kG - 1u;   /* the group's FIFO slice size - 1 */
    uint32_t free_w, free_task, free_tbs, free_bar, exec_mask;
    uint32_t fg;         /* this lane's 32 granule bits */
    uint32_t ph, pl, pt; /* FIFO: [ph,pl) loaded task slots, [pl,pt) tickets not yet loaded */
    uint32_t est_w;      /* warps of the last loaded task (0 = none yet) */
    uint32_t seq;        /* ledger clock */
    uint32_t holder_bit; /* the warp holding the scheduler token (this warp) */
    uint32_t g;          /* scheduling group (S.grp[g]) */
    int      vmtb;       /* ledger id of the group: mtb * kG + g */
};
/* FIFO position x of the group's slice of pend / pend_ticket */
template <int kG>
__device__ __forceinline__ uint32_t fq(const Sched<kG>& st, uint32_t x)
{
    return kG == 1 ? (x & 31u) : st.g * (Sched<kG>::rm + 1u) + (x & Sched<kG>::rm);
}

__device__ __forceinline__ uint32_t nth_set_bit(uint32_t mask, uint32_t n)
{   /* 0-based n-th set bit position (mask must have > n bits) */
    return __fns(mask, 0, (int)n + 1);
}

template <int kG>
__device__ bool sched_place(MtbShared& S, Sched<kG>& st, const MkParams& p, int mtb, uint32_t slot)
{
    const uint32_t lane = threadIdx.x & 31u;
    const TaskEntry& e = S.tasks[slot];
    /* granules from the request itself (the entry's u8 gran_tb field saturates above 255 granules,
     * while an MTB's arena can hold up to kMaxGranules) */
    const uint32_t wtb = e.warps_tb, ntb = e.n_tb, gtb = (e.shmem_bytes + PAGODA_GRANULE - 1u) / PAGODA_GRANULE;
    const bool need_bar = (e.flags & 1u) && wtb > 1;
    if ((uint32_t)__popc(st.free_w) < wtb * ntb || (uint32_t)__popc(st.free_tbs) < ntb ||
        (need_bar && (uint32_t)__popc(st.free_bar) < ntb))
        return false;
    int off0 = 0;   /* one TB: its first fit, found once (the feasibility check IS the allocation) */
    if (gtb) {   /* feasibility of all TBs' shared memory first (all-or-nothing per task) */
        if (ntb == 1) {
            off0 = bm_fit(st.fg, gtb, lane);
            if (off0 < 0) return false;
        } else {
            uint32_t fg2 = st.fg;
            for (uint32_t j = 0; j < ntb; j++) {
                const int off = bm_fit(fg2, gtb, lane);
                if (off < 0) return false;
                fg2 &= ~bm_range_bits((uint32_t)off, gtb, lane);
            }
        }
    }
    const uint64_t id = e.id;
    const uint16_t threads = e.threads_tb;
    /* a spread task's entry covers its TBs [tb0, tb0 + ntb) of ntb_all */
    const bool group = e.flags & kEntryGroup;
    const uint32_t tb0 = group ? (e.reserved & 0xFFFFu) : 0u, ntb_all = group ? (e.reserved >> 16) : ntb;
    if (lane == 0) S.task_warps_left[slot] = wtb * ntb;
    uint32_t all = 0;
    for (uint32_t j = 0; j < ntb; j++) {
        const uint32_t tbs = __ffs(st.free_tbs) - 1;
        st.free_tbs &= ~(1u << tbs);
        /* lowest free warps, the token holder last: it keeps scheduling unless it is needed */
        uint32_t m = 0, fw = st.free_w & ~st.holder_bit;
        for (uint32_t i = 0; i < wtb; i++) {
            if (!fw) fw = st.free_w & st.holder_bit;
            m |= fw & (0u - fw);
            fw &= fw - 1u;
        }
        st.free_w &= ~m;
        uint32_t bar = 0;
        if (need_bar) {
            bar = __ffs(st.free_bar) - 1;
            st.free_bar &= ~(1u << bar);
        }
        uint32_t off = 0;
        if (gtb) {
            off = ntb == 1 ? (uint32_t)off0 : (uint32_t)bm_fit(st.fg, gtb, lane);
            st.fg &= ~bm_range_bits(off, gtb, lane);
        }
        if (lane == 0) {
            S.tb_warps_left[tbs] = wtb;
            S.tb_goff[tbs] = (uint16_t)off;
            S.tb_glen[tbs] = (uint16_t)gtb;
            S.tb_bar[tbs] = (uint8_t)bar;
            S.tb_task[tbs] = id;
            S.tb_idx[tbs] = (uint16_t)(tb0 + j);
        }
        trace_ev(p, st.vmtb, st.seq, 1, id, (uint16_t)(tb0 + j), m, (uint16_t)off, (uint16_t)gtb, (uint8_t)bar);
        if ((m >> lane) & 1u) {   /* Alg. 2 L9-12: lane l fills warp l's WarpTable slot */
            WarpSlot ws;
            ws.smem_off = p.arena_offset + off * PAGODA_GRANULE;
            ws.smem_bytes = gtb * PAGODA_GRANULE;
            ws.tb = (uint16_t)(tb0 + j);
            ws.threads_tb = threads;
            ws.task = (uint8_t)slot;
            ws.warp_in_tb = (uint8_t)__popc(m & ((1u << lane) - 1u));
            ws.warps_tb = (uint8_t)wtb;
            ws.n_tb = (uint8_t)ntb;
            ws.bar_id = (uint8_t)bar;
            ws.tbslot = (uint8_t)tbs;
            ws.n_tb_all = (uint16_t)ntb_all;
            ws.task_id = id;
            S.wt[lane] = ws;
        }
        all |= m;
    }
    if (lane == 0 && !group) life_stamp(p, id, kLifePlace);
    __syncwarp();   /* counters written by lane 0 happen-before every lane's release-arrive */
    if ((all >> lane) & 1u) mbar_arrive(&S.exec_bar[lane]);   /* Alg. 2 L14: exec <- 1 */
    return true;
}

/* Batched placement ("__match_any_sync on (w, shmem, sync) groups identical tasks so
 * one pass places them"): the run of loaded tasks at the FIFO head that share the head's shape
 * (one thread block, same warps, granules and barrier need; a task spread over MTBs goes through
 * sched_place) is placed in ONE pass, as many as the MTB holds now: one free-mask update, lane i
 * keeps task i's bookkeeping, lane l writes warp l's WarpTable slot, one arrive per warp.  The
 * cost of placing k tasks is then about that of one (the holder's place step was the largest share
 * of its time: it runs among the body warps' shared-memory traffic).  Returns the number placed;
 * -1 if the head is not batchable (the caller uses sched_place). */
#ifndef PAGODA_BATCH_PLACE
#define PAGODA_BATCH_PLACE 0   /* measured: slower (most rounds place one task; the run logic costs more than it saves) */
#endif
template <int kG>
__device__ int sched_place_run(MtbShared& S, Sched<kG>& st, const MkParams& p, int mtb)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t navail = min(st.pl - st.ph, 32u);
    uint32_t key = 0xFFFFFFFFu, slot = 0;
    if (lane < navail) {
        slot = S.pend[fq(st, st.ph + lane)];
        const TaskEntry& e = S.tasks[slot];
        const uint32_t g = (e.shmem_bytes + PAGODA_GRANULE - 1u) / PAGODA_GRANULE;
        if (e.n_tb == 1 && !(e.flags & kEntryGroup))
            key = (uint32_t)e.warps_tb | (g << 6) | ((((e.flags & kEntrySync) != 0) && e.warps_tb > 1) ? (1u << 17) : 0u);
    }
    const uint32_t k0 = __shfl_sync(0xffffffffu, key, 0);
    if (k0 == 0xFFFFFFFFu) return -1;
    const uint32_t same = __ballot_sync(0xffffffffu, key == k0);
    uint32_t fit = same == 0xffffffffu ? 32u : (uint32_t)__ffs(~same) - 1u;   /* the run at the head */
    const uint32_t wtb = k0 & 63u, gtb = (k0 >> 6) & 2047u;
    const bool need_bar = (k0 >> 17) & 1u;
    fit = min(fit, (uint32_t)__popc(st.free_w) / wtb);
    fit = min(fit, (uint32_t)__popc(st.free_tbs));
    if (need_bar) fit = min(fit, (uint32_t)__popc(st.free_bar));
    /* granules: first fit task by task (register and shuffle work only); lane i keeps task i's offset */
    uint32_t off = 0;
    if (gtb) {
        for (uint32_t i = 0; i < fit; i++) {
            const int o = bm_first_fit(st.fg, gtb, lane);
            if (o < 0) {
                fit = i;
                break;
            }
            st.fg &= ~bm_range_bits((uint32_t)o, gtb, lane);
            if (lane == i) off = (uint32_t)o;
        }
    }
    if (fit == 0) return 0;
    /* warps: the lowest fit * wtb free ones, the token holder last (it keeps scheduling unless needed) */
    const uint32_t nw = fit * wtb;
    uint32_t sel = 0, fw = st.free_w & ~st.holder_bit;
    for (uint32_t i = 0; i < nw; i++) {
        if (!fw) fw = st.free_w & st.holder_bit;
        sel |= fw & (0u - fw);
        fw &= fw - 1u;
    }
    st.free_w &= ~sel;
    /* lane i < fit: task i's TB record, barrier, id */
    uint32_t tbs = 0, bar = 0;
    uint64_t id = 0;
    uint16_t threads = 0;
    if (lane < fit) {
        tbs = nth_set_bit(st.free_tbs, lane);
        if (need_bar) bar = nth_set_bit(st.free_bar, lane);
        const TaskEntry& e = S.tasks[slot];
        id = e.id;
        threads = e.threads_tb;
        S.task_warps_left[slot] = wtb;
        S.tb_warps_left[tbs] = wtb;
        S.tb_goff[tbs] = (uint16_t)off;
        S.tb_glen[tbs] = (uint16_t)gtb;
        S.tb_bar[tbs] = (uint8_t)bar;
        S.tb_task[tbs] = id;
        S.tb_idx[tbs] = 0;
        if (p.life) life_stamp(p, id, kLifePlace);
    }
    st.free_tbs &= ~__reduce_or_sync(0xffffffffu, lane < fit ? (1u << tbs) : 0u);
    if (need_bar) st.free_bar &= ~__reduce_or_sync(0xffffffffu, lane < fit ? (1u << bar) : 0u);
    /* lane l of the selected warps: task i = rank / wtb, warp wtb-rank within it */
    const uint32_t r = (uint32_t)__popc(sel & ((1u << lane) - 1u));
    const uint32_t ti = ((sel >> lane) & 1u) ? r / wtb : 0u;
    const uint32_t t_slot = __shfl_sync(0xffffffffu, slot, ti), t_tbs = __shfl_sync(0xffffffffu, tbs, ti);
    const uint32_t t_off = __shfl_sync(0xffffffffu, off, ti), t_bar = __shfl_sync(0xffffffffu, bar, ti);
    const uint32_t t_thr = __shfl_sync(0xffffffffu, (uint32_t)threads, ti);
    const uint64_t t_id = __shfl_sync(0xffffffffu, id, ti);
    if (p.trace_cap) {   /* the ledger: one ALLOC per task, in FIFO order */
        for (uint32_t i = 0; i < fit; i++) {
            const uint32_t mi = __ballot_sync(0xffffffffu, ((sel >> lane) & 1u) && ti == i);
            trace_ev(p, st.vmtb, st.seq, 1, __shfl_sync(0xffffffffu, id, i), 0, mi,
                     (uint16_t)__shfl_sync(0xffffffffu, off, i), (uint16_t)gtb,
                     (uint8_t)__shfl_sync(0xffffffffu, bar, i));
        }
    }
    if ((sel >> lane) & 1u) {
        WarpSlot ws;
        ws.smem_off = p.arena_offset + t_off * PAGODA_GRANULE;
        ws.smem_bytes = gtb * PAGODA_GRANULE;
        ws.tb = 0;
        ws.threads_tb = (uint16_t)t_thr;
        ws.task = (uint8_t)t_slot;
        ws.warp_in_tb = (uint8_t)(r - ti * wtb);
        ws.warps_tb = (uint8_t)wtb;
        ws.n_tb = 1;
        ws.bar_id = (uint8_t)t_bar;
        ws.tbslot = (uint8_t)t_tbs;
        ws.n_tb_all = 1;
        ws.task_id = t_id;
        S.wt[lane] = ws;
    }
    __syncwarp();   /* every lane's bookkeeping happens-before the release-arrives */
    if ((sel >> lane) & 1u) mbar_arrive(&S.exec_bar[lane]);
    return (int)fit;
}

/* Take tickets: as many tasks as the free warps fit at the last task size
 * (one ticket when the size is unknown), never more than the ring holds; one
 * at a time while the backlog is smaller than what all MTBs could take, so
 * consecutive (often similar-cost) tasks spread over MTBs. */
template <int kG>
__device__ int sched_claim(MtbShared& S, Sched<kG>& st, const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t queued = st.pt - st.ph;
    const uint32_t cap = st.rm + 1u - queued;
    uint32_t want;
    if (st.est_w == 0) want = queued == 0 ? 1u : 0u;
    else {   /* what fits now, plus one task of lookahead so the next is loaded when warps free */
        want = (uint32_t)__popc(st.free_w) / st.est_w + (uint32_t)PAGODA_LOOKAHEAD;
        want = want > queued ? want - queued : 0u;
        /* hysteresis: refill the queue in batches (one fetch-add and one load round per batch) */
        if (queued && want < (uint32_t)PAGODA_CLAIM_MIN) want = 0;
    }
    want = min(want, cap);
    if (p.max_tasks) {   /* pagoda_config.max_tasks: tasks held (task slots taken + tickets not yet loaded) */
        const uint32_t gslots = kG == 1 ? 0xffffffffu : (0xffffu << (16u * st.g));
        const uint32_t held = (uint32_t)__popc(gslots & ~st.free_task) + (st.pt - st.pl);
        want = min(want, p.max_tasks > held ? p.max_tasks - held : 0u);
    }
    if (want == 0) return 0;
    uint64_t head = 0, tail = 0;
    if (lane == 0) {
        head = ld_relaxed_gpu(&p.dctl->head);
        tail = ld_acquire_gpu(&p.dctl->tail);
    }
    head = __shfl_sync(0xffffffffu, head, 0);
    tail = __shfl_sync(0xffffffffu, tail, 0);
    if (head >= tail) {
        sc_add(S.grp[st.g], kScClaimEmpty, 1);
        return 0;
    }
    const uint64_t backlog = tail - head;
    if (p.spread_ns && backlog < (uint64_t)p.n_mtb * PAGODA_SMALL_MULT) {
        /* PAGODA_SPREAD, small backlog: a busier MTB claims later (its busy warps / 4 + 1 times
         * spread_ns after its last claim), so tasks go to the least-loaded MTBs first */
        const uint32_t busy = (uint32_t)__popc(st.exec_mask & ~st.free_w);
        const uint64_t now = globaltimer_ns();
        if (busy && now < S.grp[st.g].claim_after) return 0;
        if (lane == 0) S.grp[st.g].claim_after = now + (uint64_t)(busy + 4u) * p.spread_ns / 4u;
    }
#if PAGODA_CLAIM_FAIR
    /* at most a fair share of the backlog per claim: spreads consecutive tasks over MTBs when
     * the backlog is small, takes batches (one fetch-add and one load round) when it is not */
    want = min(want, max((uint32_t)PAGODA_CLAIM_SMALL, (uint32_t)min(backlog / (uint64_t)p.n_mtb, (uint64_t)32)));
#else
    if (backlog < (uint64_t)p.n_mtb * PAGODA_SMALL_MULT) want = min(want, (uint32_t)PAGODA_CLAIM_SMALL);
#endif
    const uint32_t k = (uint32_t)min((uint64_t)want, backlog);
    unsigned long long t0 = 0;
    if (lane == 0) t0 = atomicAdd(reinterpret_cast<unsigned long long*>(&p.dctl->head), (unsigned long long)k);
    t0 = __shfl_sync(0xffffffffu, t0, 0);
    if (lane < k) S.pend_ticket[fq(st, st.pt + lane)] = t0 + lane;
    sc_add(S.grp[st.g], kScTickets, k);
    st.pt += k;
    __syncwarp();
    return (int)k;
}

template <int kG>
__device__ int sched_copy(MtbShared& S, Sched<kG>& st, const MkParams& p, uint32_t r);

/* Load the published tickets at the front of the FIFO into free task slots,
 * then hand their cells back to the producer (seq = t + R). */
template <int kG>
__device__ int sched_load(MtbShared& S, Sched<kG>& st, const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t n = min(st.pt - st.pl, (uint32_t)__popc(st.free_task));
    if (n == 0) return 0;
    bool ready = false;
    if (p.ce_ingest) {   /* published = below the tail the copy stream wrote after the copy (acquire) */
        uint64_t tail = 0;
        if (lane == 0) tail = ld_acquire_gpu(&p.dctl->tail);
        tail = __shfl_sync(0xffffffffu, tail, 0);
        if (lane < n) ready = S.pend_ticket[fq(st, st.pl + lane)] < tail;
    } else if (lane < n) {
        const uint64_t t = S.pend_ticket[fq(st, st.pl + lane)];
        ready = ld_acquire_gpu32(&p.dseq[t & p.ring_mask]) == (uint32_t)(t + 1);
    }
    const uint32_t nr = __ballot_sync(0xffffffffu, !ready);
    const uint32_t r = nr ? (uint32_t)__ffs(nr) - 1u : 32u;   /* leading published tickets */
    if (r == 0) {
        sc_add(S.grp[st.g], kScLoadNotReady, 1);
        return 0;
    }
    return sched_copy(S, st, p, r);
}

/* Copy the first r tickets of the FIFO (published: their cells' sequence words
 * were acquired) into free task slots and hand the cells back. */
template <int kG>
__device__ int sched_copy(MtbShared& S, Sched<kG>& st, const MkParams& p, uint32_t r)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t t = lane < r ? S.pend_ticket[fq(st, st.pl + lane)] : 0;
#if PAGODA_FAST_LOAD
    /* 4 lanes per cell, one 16-byte relaxed load each: up to 8 cells per warp instruction, all in
     * flight together (one L2 round trip; the sequence words' acquires in sched_load ordered these
     * loads after them and invalidated L1).  The hand-back store of a cell must not be performed
     * before the cell's loads: the warp issues in order, and the shared-memory stores of the loaded
     * words (STS, which wait for the data) precede the hand-back in program order. */
    for (uint32_t c = lane; c < r * 4u; c += 32u) {
        const uint32_t i = c >> 2, q = c & 3u;
        const uint64_t ti = S.pend_ticket[fq(st, st.pl + i)];
        int4 v;
        asm volatile("ld.relaxed.gpu.global.v4.s32 {%0,%1,%2,%3}, [%4];"
                     : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w)
                     : "l"(reinterpret_cast<const int4*>(p.dring + (ti & p.ring_mask)) + q)
                     : "memory");
        reinterpret_cast<int4*>(&S.tasks[nth_set_bit(st.free_task, i)])[q] = v;
    }
    __syncwarp();
    uint32_t used = 0;
    if (lane < r) {
        const uint32_t slot = nth_set_bit(st.free_task, lane);
        S.pend[fq(st, st.pl + lane)] = (uint8_t)slot;
        st_relaxed_gpu32(&p.dseq[t & p.ring_mask], (uint32_t)(t + (uint64_t)p.ring_mask + 1));
        if (p.life && !(S.tasks[slot].flags & kEntryGroup)) {
            if (p.ce_ingest) life_stamp(p, S.tasks[slot].id, kLifePub);   /* (no device-side publication step) */
            life_stamp(p, S.tasks[slot].id, kLifeLoad);
        }
        used = 1u << slot;
    }
#elif PAGODA_FAST_LOAD == 0 && PAGODA_CELL_RELAXED
    /* lane i copies cell i with four relaxed 16-byte loads in flight together (the sequence word's
     * acquire already ordered them after the publication and invalidated L1), then a CTA-scope fence
     * before the hand-back: the loads have returned before the store issues */
    uint32_t used = 0;
    if (lane < r) {
        const uint32_t slot = nth_set_bit(st.free_task, lane);
        const int4* src = reinterpret_cast<const int4*>(p.dring + (t & p.ring_mask));
        int4* dst = reinterpret_cast<int4*>(&S.tasks[slot]);
        int4 v[4];
#pragma unroll
        for (int q = 0; q < 4; q++)
            asm volatile("ld.relaxed.gpu.global.v4.s32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(v[q].x), "=r"(v[q].y), "=r"(v[q].z), "=r"(v[q].w) : "l"(src + q) : "memory");
#pragma unroll
        for (int q = 0; q < 4; q++) dst[q] = v[q];
        asm volatile("fence.acq_rel.cta;" ::: "memory");
        S.pend[fq(st, st.pl + lane)] = (uint8_t)slot;
        st_relaxed_gpu32(&p.dseq[t & p.ring_mask], (uint32_t)(t + (uint64_t)p.ring_mask + 1));
        if (p.life && !(S.tasks[slot].flags & kEntryGroup)) {
            if (p.ce_ingest) life_stamp(p, S.tasks[slot].id, kLifePub);   /* (no device-side publication step) */
            life_stamp(p, S.tasks[slot].id, kLifeLoad);
        }
        used = 1u << slot;
    }
#elif PAGODA_CELL_ACQ
    /* lane i copies cell i whole with acquire loads (LDG.STRONG.GPU + L1 invalidate, no MEMBAR),
     * so its own hand-back store below is ordered after every read of the cell in program order.
     * (A st.release would be a MEMBAR.GPU, which waits for every memory operation in flight on the
     * SM.)  The four acquires are serial: four round trips. */
    uint32_t used = 0;
    if (lane < r) {
        const uint32_t slot = nth_set_bit(st.free_task, lane);
        const int4* src = reinterpret_cast<const int4*>(p.dring + (t & p.ring_mask));
        int4* dst = reinterpret_cast<int4*>(&S.tasks[slot]);
#pragma unroll
        for (int q = 0; q < 4; q++) {
            int4 v;
            asm volatile("ld.acquire.gpu.global.v4.s32 {%0,%1,%2,%3}, [%4];"
                         : "=r"(v.x), "=r"(v.y), "=r"(v.z), "=r"(v.w) : "l"(src + q) : "memory");
            dst[q] = v;
        }
        S.pend[fq(st, st.pl + lane)] = (uint8_t)slot;
        st_relaxed_gpu32(&p.dseq[t & p.ring_mask], (uint32_t)(t + (uint64_t)p.ring_mask + 1));
        if (p.life && !(S.tasks[slot].flags & kEntryGroup)) {
            if (p.ce_ingest) life_stamp(p, S.tasks[slot].id, kLifePub);   /* (no device-side publication step) */
            life_stamp(p, S.tasks[slot].id, kLifeLoad);
        }
        used = 1u << slot;
    }
#else
    for (uint32_t c = lane; c < r * 4u; c += 32u) {   /* 4 lanes per cell, coalesced */
        const uint32_t i = c >> 2;
        const uint64_t ti = S.pend_ticket[fq(st, st.pl + i)];
        const int4 v = __ldcg(reinterpret_cast<const int4*>(p.dring + (ti & p.ring_mask)) + (c & 3u));
        reinterpret_cast<int4*>(&S.tasks[nth_set_bit(st.free_task, i)])[c & 3u] = v;
    }
    __syncwarp();   /* all copies (loads) precede the release of each cell */
    uint32_t used = 0;
    if (lane < r) {
        const uint32_t slot = nth_set_bit(st.free_task, lane);
        S.pend[fq(st, st.pl + lane)] = (uint8_t)slot;
        st_release_gpu32(&p.dseq[t & p.ring_mask], (uint32_t)(t + (uint64_t)p.ring_mask + 1));
        used = 1u << slot;
    }
#endif
    used = __reduce_or_sync(0xffffffffu, used);
    st.free_task &= ~used;
    st.pl += r;
    __syncwarp();
    const TaskEntry& last = S.tasks[S.pend[fq(st, st.pl - 1)]];
    st.est_w = (uint32_t)last.warps_tb * last.n_tb;
    return (int)r;
}

#if PAGODA_FUSED_CLAIM
/* One L2 round trip for all of a round's questions to the device ring: lane 0
 * takes new tickets (fetch-add on the head), lanes 1-2 read the tail and the
 * head, lanes 3.. acquire the sequence words of up to 29 tickets claimed in
 * earlier rounds.  The claim size comes from the backlog seen last time (a
 * fair share of it per MTB), and an MTB that holds no tickets keeps ONE
 * standing reservation even when the ring is empty: the next task published
 * at that position is its own (consecutive tasks land on different MTBs).
 * Reserved positions past the final tail are void at stop (head = tail).
 * Returns how many tickets at the FIFO front are published (sched_copy). */
template <int kG>
__device__ int sched_claim_check(MtbShared& S, Sched<kG>& st, const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t queued = st.pt - st.ph;
    uint32_t want = 0;
    if (!S.no_tickets) {
        if (st.est_w == 0) want = queued == 0 ? 1u : 0u;
        else {
            want = (uint32_t)__popc(st.free_w) / st.est_w + (uint32_t)PAGODA_LOOKAHEAD;
            want = want > queued ? want - queued : 0u;
            if (queued && want < (uint32_t)PAGODA_CLAIM_MIN) want = 0;
        }
        const uint32_t est = S.grp[st.g].backlog_est;
        if (est == 0) want = min(want, st.pt == st.pl ? 1u : 0u);   /* a standing reservation */
        else want = min(want, max((uint32_t)PAGODA_CLAIM_SMALL, min(est / (uint32_t)p.n_mtb, 32u)));
        want = min(want, st.rm + 1u - queued);
    }
    const uint32_t n = min(st.pt - st.pl, min((uint32_t)__popc(st.free_task), 29u));
    uint64_t v = 0;
    bool ready = false;
    if (lane == 0) {
        if (want) v = atomicAdd(reinterpret_cast<unsigned long long*>(&p.dctl->head), (unsigned long long)want);
    } else if (lane == 1) {
        v = ld_acquire_gpu(&p.dctl->tail);
    } else if (lane == 2) {
        v = ld_relaxed_gpu(&p.dctl->head);
    } else if (lane - 3u < n) {
        const uint64_t t = S.pend_ticket[fq(st, st.pl + lane - 3u)];
        ready = ld_acquire_gpu32(&p.dseq[t & p.ring_mask]) == (uint32_t)(t + 1);
    }
    const uint64_t old = __shfl_sync(0xffffffffu, v, 0);
    const uint64_t tail = __shfl_sync(0xffffffffu, v, 1);
    uint64_t head = __shfl_sync(0xffffffffu, v, 2);
    const uint32_t rb = __ballot_sync(0xffffffffu, ready) >> 3;
    const uint32_t r = min((uint32_t)__ffs(~rb) - 1u, n);   /* leading published tickets */
    if (want) head = max(head, old + want);
    if (lane < want) S.pend_ticket[fq(st, st.pt + lane)] = old + lane;
    if (lane == 0) S.grp[st.g].backlog_est = (uint32_t)min(tail > head ? tail - head : 0ull, 0xffffffffull);
    sc_add(S.grp[st.g], kScTickets, want);
    if (want && old >= tail) sc_add(S.grp[st.g], kScClaimEmpty, 1);
    if (n && r == 0) sc_add(S.grp[st.g], kScLoadNotReady, 1);
    st.pt += want;
    __syncwarp();
    return (int)r;
}
#endif

/* ------------------------------------------------------------------ self-scheduling
 * The paper dedicates warp 0 of every MTB to scheduling.  Here the
 * scheduler is a TOKEN in shared memory instead: the warp holding it runs
 * scheduling rounds; a warp that finishes a task posts its frees and tries to
 * take the token; a holder that dispatches a task to itself hands the token to
 * another free warp (or releases it when none is free).  Invariant: either some
 * warp holds the token, or every worker is running a task (and the next one to
 * finish takes it).  So every warp of the MTB executes tasks: eight 4-warp tasks
 * per MTB instead of seven (SURVEY App. A "v2: self-scheduling"). */
template <int kG>
__device__ __forceinline__ void sst_save(MtbShared& S, const Sched<kG>& st)
{
    const uint32_t lane = threadIdx.x & 31u;
    SchedGroup& G = S.grp[st.g];
    G.fg[lane] = st.fg;
    if (lane == 0) {
        G.free_w = st.free_w;
        G.free_task = st.free_task;
        G.free_tbs = st.free_tbs;
        G.free_bar = st.free_bar;
        G.ph = st.ph;
        G.pl = st.pl;
        G.pt = st.pt;
        G.est_w = st.est_w;
        G.seq = st.seq;
    }
    __syncwarp();
}

/* the holder state of group g (the caller's warp now holds g's token) */
template <int kG>
__device__ __forceinline__ void sst_load(MtbShared& S, Sched<kG>& st, uint32_t exec_mask, uint32_t g, const MkParams& p,
                                         int mtb)
{
    __syncwarp();
    const SchedGroup& G = S.grp[g];
    st.fg = G.fg[threadIdx.x & 31u];
    st.free_w = G.free_w;
    st.free_task = G.free_task;
    st.free_tbs = G.free_tbs;
    st.free_bar = G.free_bar;
    st.ph = G.ph;
    st.pl = G.pl;
    st.pt = G.pt;
    st.est_w = G.est_w;
    st.seq = G.seq;
    st.exec_mask = exec_mask;
    st.holder_bit = 1u << (threadIdx.x >> 5);
    st.g = g;
    st.vmtb = mtb * kG + (int)g;
    (void)p;
}

__device__ __forceinline__ bool token_try(SchedGroup& G)
{
    uint32_t got = 0;
    if ((threadIdx.x & 31u) == 0) {
        got = atomicCAS(&G.token, 0u, 1u) == 0u;
        __threadfence_block();
    }
    return __shfl_sync(0xffffffffu, got, 0) != 0;
}

__device__ __forceinline__ void token_release(SchedGroup& G)
{
    __syncwarp();
    if ((threadIdx.x & 31u) == 0) {
        __threadfence_block();
        atomicExch(&G.token, 0u);
        __threadfence_block();
    }
    __syncwarp();
}

/* fold the mailboxes into the holder's state (deallocMarkedSM, Alg. 1 L22) */
template <int kG>
__device__ bool sched_fold(MtbShared& S, Sched<kG>& st, const MkParams& p, int mtb)
{
    const uint32_t lane = threadIdx.x & 31u;
    uint32_t mw = 0, mt = 0, mk = 0;
    SchedGroup& G = S.grp[st.g];
    if (lane == 0) {
        if (*(volatile uint32_t*)&G.mb_warps) mw = atomicExch(&G.mb_warps, 0u);
        __threadfence_block();
        if (*(volatile uint32_t*)&G.mb_tbs) mt = atomicExch(&G.mb_tbs, 0u);
        if (*(volatile uint32_t*)&G.mb_tasks) mk = atomicExch(&G.mb_tasks, 0u);
    }
    mw = __shfl_sync(0xffffffffu, mw, 0);
    mt = __shfl_sync(0xffffffffu, mt, 0);
    mk = __shfl_sync(0xffffffffu, mk, 0);
    if (!(mw | mt | mk)) return false;
    for (uint32_t b = mt; b; b &= b - 1u) {
        const uint32_t tbs = __ffs(b) - 1;
        const uint32_t goff = S.tb_goff[tbs], glen = S.tb_glen[tbs], bar = S.tb_bar[tbs];
        if (glen) st.fg |= bm_range_bits(goff, glen, lane);
        if (bar) st.free_bar |= 1u << bar;
        st.free_tbs |= 1u << tbs;
        if (p.trace_cap)
            trace_ev(p, st.vmtb, st.seq, 3, S.tb_task[tbs], S.tb_idx[tbs], 0, (uint16_t)goff, (uint16_t)glen, (uint8_t)bar);
    }
    if (p.trace_cap) {
        for (uint32_t b = mw; b; b &= b - 1u) {
            const uint32_t w = __ffs(b) - 1;
            trace_ev(p, st.vmtb, st.seq, 2, S.wt[w].task_id, S.wt[w].tb, 1u << w, 0, 0, 0);
        }
    }
    st.free_w |= mw;
    st.free_task |= mk;
    return true;
}

/* One scheduling round: fold, load published tickets, place in FIFO order
 * (Alg. 1 L14-28), take more tickets.  Sets exit when the session is over. */
template <int kG>
__device__ bool sched_round(MtbShared& S, Sched<kG>& st, const MkParams& p, int mtb, bool& exit)
{
    const uint32_t lane = threadIdx.x & 31u;
    uint64_t t0 = pf_now();
    bool progress = sched_fold(S, st, p, mtb);
    pf_add(S.grp[st.g], kPfFold, t0, true);
    /* completion records of the tasks whose last warp finished (a warp marks comp_pending before
     * it frees itself, so every task of a folded warp is in it): one fence and one queue
     * reservation for the whole batch, off the executors' path */
    if (PAGODA_HOLDER_POSTS && *(volatile uint32_t*)&S.grp[st.g].comp_pending) {
        t0 = pf_now();
        post_completions(S, S.grp[st.g], p);
        pf_add(S.grp[st.g], kPfPost, t0, true);
        progress = true;
    }
#if PAGODA_FUSED_CLAIM
    t0 = pf_now();
    {
        const uint32_t pt0 = st.pt;
        const int r = sched_claim_check(S, st, p);
        if (st.pt != pt0) progress = true;
        pf_add(S.grp[st.g], kPfClaim, t0, true);
        t0 = pf_now();
        if (r > 0 && sched_copy(S, st, p, (uint32_t)r) > 0) progress = true;
        pf_add(S.grp[st.g], kPfLoad, t0, true);
    }
#else
    if (PAGODA_CLAIM_FIRST) {
        t0 = pf_now();
        if (!S.no_tickets && sched_claim(S, st, p) > 0) progress = true;
        pf_add(S.grp[st.g], kPfClaim, t0, true);
    }
    t0 = pf_now();
    if (st.pl != st.pt && sched_load(S, st, p) > 0) progress = true;
    pf_add(S.grp[st.g], kPfLoad, t0, true);
#endif
    t0 = pf_now();
    while (st.ph != st.pl) {
        const int k = PAGODA_BATCH_PLACE ? sched_place_run(S, st, p, mtb) : -1;
        if (k > 0) {   /* a run of identical single-TB tasks placed in one pass */
            sc_add(S.grp[st.g], kScPlaced, (uint32_t)k);
            st.ph += (uint32_t)k;
            progress = true;
            continue;
        }
        if (k == 0 || !sched_place(S, st, p, mtb, S.pend[fq(st, st.ph)])) {
            sc_add(S.grp[st.g], kScNoFit, 1);
            break;
        }
        sc_add(S.grp[st.g], kScPlaced, 1);
        st.ph++;
        progress = true;
    }
    pf_add(S.grp[st.g], kPfPlace, t0, true);
    /* MTB 0 (the I/O MTB: ingest, host stores) and the MTB sharing its SM take no tickets
     * unless MTB 0 is the only MTB (validation then caps every task to its capacity) */
    if (!PAGODA_CLAIM_FIRST && !PAGODA_FUSED_CLAIM) {
        t0 = pf_now();
        if (!S.no_tickets && sched_claim(S, st, p) > 0) progress = true;
        pf_add(S.grp[st.g], kPfClaim, t0, true);
    }
    exit = false;
    sc_add(S.grp[st.g], kScRounds, 1);
    if (progress) sc_add(S.grp[st.g], kScProgress, 1);
    bool quiet = !progress && st.free_w == st.exec_mask && st.ph == st.pl;
    if (quiet) {   /* no completion pending, and (FREE_BEFORE_POST) none being posted: pending is read first,
                      a poster clears it only while holding the poster flag */
        uint32_t q = 0;
        if (lane == 0) {
            q = *(volatile uint32_t*)&S.grp[st.g].comp_pending == 0u;
            __threadfence_block();
            if (PAGODA_FREE_BEFORE_POST) q = q && *(volatile uint32_t*)&S.grp[st.g].poster == 0u;
        }
        quiet = __shfl_sync(0xffffffffu, q, 0) != 0;
    }
    if (quiet) {
        uint32_t stop = 0;
        if (lane == 0) stop = ld_acquire_gpu32(&p.dctl->stop);
        stop = __shfl_sync(0xffffffffu, stop, 0);
        if (stop == kStopAbort) exit = true;   /* host watchdog gave up */
        else if (stop) {
            uint64_t tail = 0, head = 0;
            if (lane == 0) {
                tail = ld_acquire_gpu(&p.dctl->tail);
                head = ld_relaxed_gpu(&p.dctl->head);
            }
            tail = __shfl_sync(0xffffffffu, tail, 0);
            head = __shfl_sync(0xffffffffu, head, 0);
            /* after stop the tail is final: tickets at or past it are void.  A round without progress
             * does not prove the ring drained: a claim cap (max_tasks) holds claims back while a
             * finished task's slot awaits its fold, so leave only once every ticket is handed out */
            exit = (st.pl == st.pt || S.pend_ticket[fq(st, st.pl)] >= tail) && (S.no_tickets || head >= tail);
        }
    }
    return progress;
}

/* The holder w has dispatched a task to itself: pass the token to another free
 * warp (it wakes with a SCHED slot), else release it — re-checking the mailbox
 * afterwards so a warp that freed itself meanwhile, and failed to take the
 * token, is not left without a scheduler. */
template <int kG>
__device__ void sched_handoff(MtbShared& S, Sched<kG>& st, const MkParams& p, int mtb)
{
    const uint32_t lane = threadIdx.x & 31u;
    for (;;) {
        sched_fold(S, st, p, mtb);
        if (st.free_w) {
            const uint32_t h = __ffs(st.free_w) - 1;
            sst_save(S, st);
            sc_add(S.grp[st.g], kScHandoffs, 1);
            if (lane == h) {
                S.wt[h].task = SLOT_SCHED;
                mbar_arrive(&S.exec_bar[h]);   /* release: the saved state is visible to h */
            }
            __syncwarp();
            return;
        }
        sst_save(S, st);
        SchedGroup& G = S.grp[st.g];
        token_release(G);
        uint32_t pending = 0;
        if (lane == 0) pending = *(volatile uint32_t*)&G.mb_warps;
        pending = __shfl_sync(0xffffffffu, pending, 0);
        if (!pending || !token_try(G)) return;
        sst_load(S, st, st.exec_mask, st.g, p, mtb);
    }
}

/* One holder phase: the warp owns the scheduler token and runs rounds until it
 * dispatched itself (hands the token on) or the session ends (returns true).
 * The scheduler state lives only here (loaded from / saved to shared memory),
 * so no register holds it while the warp runs task bodies. */
template <int kG>
__device__ __noinline__ bool holder_phase(MtbShared& S, const MkParams& p, int mtb, int w, uint32_t exec_mask,
                                          uint32_t g)
{
    const uint32_t lane = threadIdx.x & 31u;
    Sched<kG> st;
    sst_load(S, st, exec_mask, g, p, mtb);
    uint32_t backoff = 0;
    for (;;) {
        bool exit = false;
        const bool progress = sched_round(S, st, p, mtb, exit);
        if (exit) {   /* drain: release every other worker with a terminate slot */
            if (((exec_mask & ~(1u << w)) >> lane) & 1u) {
                S.wt[lane].task = SLOT_TERMINATE;
                mbar_arrive(&S.exec_bar[lane]);
            }
            if (lane == 0) {
                __threadfence();   /* this group's completion-queue reservations precede its exit count */
                atomicAdd(&p.dctl->exited, 1u);
                const SchedGroup& G = S.grp[g];
                for (int i = 0; i < 8; i++)
                    atomicAdd(&p.dctl->ctr[PAGODA_CTR_SCHED_ROUNDS + i], (unsigned long long)G.sctr[i]);
                if (PAGODA_PROFILE)   /* (executors still finishing their last task may add a little after) */
                    for (int i = 0; i < 8; i++) atomicAdd(&p.dctl->ctr[PAGODA_CTR_SCHED_NS_FOLD + i], G.sprof[i]);
            }
            return true;
        }
        if ((st.free_w >> w) & 1u) {   /* still free: keep scheduling */
            if (progress) backoff = 0;
            else {
                /* with work queued only shared-memory mailboxes are polled: stay responsive;
                 * otherwise the ring is polled in L2: back off */
                backoff = (st.ph != st.pt) ? 32u : (backoff ? min(backoff * 2u, (uint32_t)PAGODA_IDLE_NS) : 32u);
                const uint64_t t0 = pf_now();
                __nanosleep(backoff);
                pf_add(S.grp[st.g], kPfSleep, t0, true);
            }
            continue;
        }
        /* dispatched (by itself or before it took the token).  Load-ahead: the tickets this round
         * claimed are loaded now, before the token moves on, so the next holder (a warp freed by the
         * next finishing task, typically) finds a loaded task and places it at once instead of paying
         * two L2 round trips with the slot's warps idle */
        if (PAGODA_LOAD_AHEAD && st.pl != st.pt) sched_load(S, st, p);
        sched_handoff(S, st, p, mtb);
        return false;
    }
}

/* Every worker warp runs this loop (warps 0..exec_warps-1; MTB 0's last warp ingests); exec_mask is
 * the worker warps of its scheduling group g. */
template <int kG, bool kCallCold>
__device__ void worker(MtbShared& S, char* smem_base, const MkParams& p, int mtb, int w, uint32_t resident,
                       uint32_t exec_mask, bool holder, uint32_t g)
{
    uint32_t phase = 0;
    SchedGroup& G = S.grp[g];
    const int vmtb = mtb * kG + (int)g;
    for (;;) {
        if (holder) {
            if (holder_phase<kG>(S, p, mtb, w, exec_mask, g)) return;
            holder = false;
        }
        exec_wait(phase);   /* mbar_wait(&S.exec_bar[w], phase) without a live address register */
        phase ^= 1u;
        const uint8_t task = *(volatile uint8_t*)&S.wt[w].task;
        if (task == SLOT_TERMINATE) return;
        if (task == SLOT_SCHED) {
            holder = true;
            continue;
        }
        run_task<kCallCold>(S, G, smem_base, p, mtb, vmtb, w, resident);
        holder = token_try(G);
    }
}

/* ------------------------------------------------------------------ the kernel */
template <int kMinBlocks, int kThreads, int kG>
__global__ void __launch_bounds__(kThreads, kMinBlocks) master_kernel(MkParams p)
{
    constexpr int nw = kThreads / 32;   /* warps per MTB */
    extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
    MtbShared& S = *reinterpret_cast<MtbShared*>(pagoda_mk_smem);
    char* smem_base = reinterpret_cast<char*>(pagoda_mk_smem);
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, mtb = blockIdx.x;
    int arena_granules = p.arena_granules;
    char* ingest_stage = nullptr;
    const bool io = mtb == 0 && p.n_mtb > 1;   /* the I/O MTB: runs no tasks */
    if (io) {
        ingest_stage = smem_base + p.stage_offset;   /* everything after the control block */
        arena_granules = 0;
    } else if (mtb == 0) {   /* MTB 0 alone: it lends the top of its arena to the ingest warp */
        arena_granules -= (int)(2u * p.ingest_stage_entries * 64u / PAGODA_GRANULE);
        ingest_stage = smem_base + p.arena_offset + (size_t)arena_granules * PAGODA_GRANULE;
    }
    /* PCIe isolation: MTB 0 announces its SM; an MTB on the same SM runs no tasks either */
    uint32_t no_tickets = io ? 1u : 0u;
    if (p.n_mtb > 1 && threadIdx.x == 0) {
        uint32_t smid;
        asm volatile("mov.u32 %0, %%smid;" : "=r"(smid));
        if (mtb == 0) {
            st_release_gpu32(&p.dctl->io_smid, smid);
        } else {   /* co-resident with MTB 0 by the cooperative launch: it writes at once */
            uint32_t io_sm;
            while ((io_sm = ld_acquire_gpu32(&p.dctl->io_smid)) == kIoSmidNone) __nanosleep(32);
            if (io_sm == smid && p.io_sm_exclusive) no_tickets = 1u;
        }
    }
    uint32_t resident = 0;   /* shared-window address of the resident tables */
    if (p.resident_tdes_src && !io) {
        /* task-class resident tables (key-independent 3DES S-box/P tables), one copy per
         * lane, at the constant window address kResidentTdesAddr (bodies.cuh tdes_f):
         * word 4096 p + 64 v + 32 h + lane holds SP[j][v] for box j = byte p of x (h = 0:
         * boxes 0,6,4,2) or of y (h = 1: boxes 7,5,3,1), so any 32 lookups are conflict-free.
         * The dynamic segment starts after the CTA's reserved shared memory (window 1 KiB). */
        const uint32_t base = smem_u32(smem_base);
        if (base + kControlBytes <= kResidentTdesAddr && kResidentTdesAddr - base + kResidentTdesBytes <= p.arena_offset) {
            resident = kResidentTdesAddr;
            uint32_t* dst = reinterpret_cast<uint32_t*>(smem_base + (resident - base));
            for (uint32_t i = threadIdx.x; i < kResidentTdesBytes / 4; i += blockDim.x) {
                const uint32_t pr = i >> 12, v = (i >> 6) & 63u, h = (i >> 5) & 1u;
                const uint32_t j = h ? 7u - 2u * pr : (8u - 2u * pr) & 7u;
                const uint32_t w = __ldg(p.resident_tdes_src + j * 64u + v);
                dst[i] = PAGODA_TDES_ROT ? __funnelshift_l(w, w, 1) : w;   /* the rounds' rotated domain */
            }
        } else if (threadIdx.x == 0) {
            atomicOr(&p.dctl->error, PAGODA_DEVERR_LAYOUT);   /* bodies fall back to per-task tables */
        }
    }
    /* worker warps: the first exec_warps / n_grp warps of each group's range (MTB 0: minus the ingest warp) */
    const int ew = min(p.exec_warps, nw);
    const uint32_t n_grp = (uint32_t)kG, gw = (uint32_t)nw / n_grp, gs = 32u / n_grp;
    uint32_t exec_mask = 0;
    for (uint32_t g = 0; g < n_grp; g++) {
        const uint32_t per = min((uint32_t)ew / n_grp, gw);
        exec_mask |= (per >= 32u ? 0xffffffffu : ((1u << per) - 1u)) << (g * gw);
    }
    if (mtb == 0) exec_mask &= ~(1u << ingest_loader_warp(nw));
    if (io)   /* the I/O roles: loader (31), host poster (30), forwarder (28), publishers (29, 27, ...) */
    {
        exec_mask &= ~(1u << host_poster_warp(nw));
        for (uint32_t i = 0; i < p.n_fwd; i++) exec_mask &= ~(1u << forwarder_warp_i(i, nw));
        for (uint32_t i = 0; i < kIngestPublishers; i++) exec_mask &= ~(1u << ingest_publisher_warp(i, nw));
    }
    /* scheduling groups: group g owns warps [g nw/G, (g+1) nw/G), task slots and TB records
     * [32g/G, 32(g+1)/G), named barriers 1..7 / 8..15 (G = 2) or 1..15, and arena granules
     * [A g/G, A (g+1)/G) */
    const uint32_t my_g = (uint32_t)warp / gw;
    const uint32_t gmask_w = (gw >= 32u ? 0xffffffffu : ((1u << gw) - 1u)) << (my_g * gw);
    const uint32_t my_exec = exec_mask & gmask_w;
    const int first = __ffs(my_exec) - 1;
    if (warp == 0) {
        mbar_init(&S.exec_bar[lane], 1);
        mbar_init(&S.stage_bar[lane], 1);
        S.stage_ph[lane] = 0;
        if (lane < kIngestStages) {
            mbar_init(&S.ingest_bar[lane], 1);
            mbar_init(&S.ingest_empty[lane], 1);
            S.ing_hdr[lane] = 0;
        }
        for (uint32_t i = lane; i < kIngestFinSlots; i += 32u) S.ing_fin[i] = 0;
        /* initial scheduler state of each group, owned by its first worker (it starts with the token) */
        for (uint32_t g = 0; g < n_grp; g++) {
            SchedGroup& G = S.grp[g];
            const uint32_t g0 = (uint32_t)arena_granules * g / n_grp, g1 = (uint32_t)arena_granules * (g + 1) / n_grp;
            G.fg[lane] = bm_range_bits(g0, g1 - g0, lane);
            if (lane == 0) {
                const uint32_t gm = (gw >= 32u ? 0xffffffffu : ((1u << gw) - 1u)) << (g * gw);
                const uint32_t sm = (gs >= 32u ? 0xffffffffu : ((1u << gs) - 1u)) << (g * gs);
                G.mb_warps = G.mb_tbs = G.mb_tasks = 0;
                G.free_w = exec_mask & gm;
                G.free_task = sm;
                G.free_tbs = sm;
                /* named barriers 1..15; 0 belongs to the MTB */
                G.free_bar = n_grp == 1 ? 0xfffeu : (g == 0 ? 0x00feu : 0xff00u);
                G.ph = G.pl = G.pt = 0;
                G.est_w = 0;
                G.seq = 0;
                G.backlog_est = 0;
                G.claim_after = 0;
                G.comp_pending = 0;
                G.poster = 0;
                G.last_post = 0;
                /* a group without workers never runs a holder: it counts as exited now */
                G.token = (exec_mask & gm) ? 1u : 0u;
                if (!(exec_mask & gm)) atomicAdd(&p.dctl->exited, 1u);
                for (int i = 0; i < 8; i++) G.sctr[i] = 0;
                for (int i = 0; i < 8; i++) G.sprof[i] = 0;
            }
        }
        if (lane == 0) {
            S.fwd_done = 0;
            S.dev_error = &p.dctl->error;
            S.dq_safe = *(volatile uint64_t*)&p.dctl->dq_head + kDqEntries;
            S.no_tickets = no_tickets;
            /* where ingest resumes: the host poster must never post a smaller consumed count
             * (a spawn blocked on a ring slot would wait for it forever) */
            S.ingest_copied = *(volatile uint64_t*)&p.dctl->tail;
            S.ingest_done = p.ce_ingest ? 1u : 0u;   /* (CE ingest: no ingest warps) */
            S.ing_prefix_k = 0;
            S.ing_lock = 0;
            S.ing_pubs_done = 0;
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
    }
    __syncthreads();
    if (mtb == 0 && p.ce_ingest && warp == ingest_loader_warp(nw)) ce_scanner(p);
    else if (mtb == 0 && p.n_mtb == 1 && warp == ingest_loader_warp(nw)) ingest(S, p, ingest_stage, S.ingest_bar);
    else if (mtb == 0 && warp == ingest_loader_warp(nw)) ingest_loader(S, p, ingest_stage);
    else if (io && ingest_publisher_index(warp, nw) < kIngestPublishers) {
        if (!p.ce_ingest) ingest_publisher(S, p, ingest_stage, ingest_publisher_index(warp, nw));
    }
    else if (io && warp == host_poster_warp(nw)) host_poster(S, p);
    else if (io && forwarder_index(warp, nw) < p.n_fwd) comp_forwarder(S, p, forwarder_index(warp, nw));
    else if ((my_exec >> warp) & 1u)   /* 4 MTBs/SM (the MM presets): the bodies they do not run behind calls */
        worker<kG, kMinBlocks == 4>(S, smem_base, p, mtb, warp, resident, my_exec, warp == first, my_g);
}

template __global__ void master_kernel<1, 1024, 1>(MkParams);
template __global__ void master_kernel<2, 1024, 1>(MkParams);
template __global__ void master_kernel<4, 512, 1>(MkParams);   /* twice the MTBs (schedulers) per SM */
template __global__ void master_kernel<1, 1024, 2>(MkParams);   /* two scheduling groups per MTB */
template __global__ void master_kernel<2, 1024, 2>(MkParams);
template __global__ void master_kernel<4, 512, 2>(MkParams);

/* host side (runtime.cu): the registered 3DES key schedule of this module's MasterKernel */
cudaError_t set_tdes_const_keys(const void* keys384, uint64_t tables_ptr)
{
    cudaError_t e = cudaMemcpyToSymbol(c_tdes_keys, keys384, sizeof(c_tdes_keys));
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(c_tdes_tables, &tables_ptr, sizeof(tables_ptr));
    return e;
}

/* host side (runtime.cu): the registered DCT coefficient matrix of this module's MasterKernel */
cudaError_t set_dct_const_coef(const void* coef256, uint64_t coef_ptr)
{
    cudaError_t e = cudaMemcpyToSymbol(c_dct_coef, coef256, sizeof(c_dct_coef));
    if (e == cudaSuccess) e = cudaMemcpyToSymbol(c_dct_coef_ptr, &coef_ptr, sizeof(coef_ptr));
    return e;
}

/* host-side launcher (called by runtime.cu) */
cudaError_t launch_master(int mtbs_per_sm, int n_mtb, size_t smem_bytes, cudaStream_t stream, MkParams* params,
                          int* regs_out)
{
    const bool g2 = params->n_grp == 2;
    const void* fn = mtbs_per_sm == 4   ? (g2 ? reinterpret_cast<const void*>(&master_kernel<4, 512, 2>)
                                              : reinterpret_cast<const void*>(&master_kernel<4, 512, 1>))
                     : mtbs_per_sm == 2 ? (g2 ? reinterpret_cast<const void*>(&master_kernel<2, 1024, 2>)
                                              : reinterpret_cast<const void*>(&master_kernel<2, 1024, 1>))
                                        : (g2 ? reinterpret_cast<const void*>(&master_kernel<1, 1024, 2>)
                                              : reinterpret_cast<const void*>(&master_kernel<1, 1024, 1>));
    const int threads = mtbs_per_sm == 4 ? 512 : 1024;
    cudaError_t err = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_bytes);
    if (err != cudaSuccess) return err;
    cudaFuncAttributes attr;
    if (cudaFuncGetAttributes(&attr, fn) == cudaSuccess && regs_out) *regs_out = attr.numRegs;
    int per_sm = 0;
    err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, threads, smem_bytes);
    if (err != cudaSuccess) return err;
    if (per_sm < mtbs_per_sm) {
        fprintf(stderr, "pagoda: %d MTBs per SM requested, %d fit (%zu B of shared memory, %d threads, %d registers)\n",
                mtbs_per_sm, per_sm, smem_bytes, threads, regs_out ? *regs_out : -1);
        return cudaErrorCooperativeLaunchTooLarge;
    }
    void* args[] = {params};
    return cudaLaunchCooperativeKernel(fn, dim3(n_mtb), dim3(threads), args, smem_bytes, stream);
}

} // namespace pagoda
