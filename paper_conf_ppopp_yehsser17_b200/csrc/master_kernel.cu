/*
 * master_kernel.cu — the persistent MasterKernel (Fig. 1b).
 *
 * Grid: one cooperative launch of n_mtb = num_sms * mtbs_per_sm thread blocks
 * ("MTBs") of 1024 threads.  In every MTB warp 0 is the scheduler
 * and warps 1..31 are executors.  Warp 31 of MTB 0 is instead the
 * ingest warp that moves published TaskTable entries from the pinned host ring
 * into the device ring.
 *
 *   host ring --(ingest: LDGSTS over PCIe -> smem -> L2 device ring)--> device ring
 *   device ring --(scheduler: speculative copy + CAS claim)--> MTB task slots
 *   task slot --(place: warps / granules / barrier from bitmaps)--> WarpTable + mbarrier arrive
 *   executor warp --(body)--> mailboxes (deferred free) + completion record (D->H)
 *
 * Memory-model notes are inline; DESIGN.md "Ordering" has the full argument.
 */
#include <cuda_runtime.h>
#include <stdint.h>

#include "bodies.cuh"
#include "mk_layout.cuh"

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
            "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2, 1000000; selp.u32 %0, 1, 0, p; }"
            : "=r"(done)
            : "r"(a), "r"(parity)
            : "memory");
    }
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
__device__ __forceinline__ bool cas_acq_rel_gpu(uint64_t* p, uint64_t expect, uint64_t desired)
{
    uint64_t old;
    asm volatile("atom.acq_rel.gpu.global.cas.b64 %0, [%1], %2, %3;"
                 : "=l"(old)
                 : "l"(p), "l"(expect), "l"(desired)
                 : "memory");
    return old == expect;
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
__device__ __forceinline__ uint32_t bm_range_bits(uint32_t off, uint32_t g, uint32_t lane)
{
    const uint32_t lo = max(off, lane * 32u), hi = min(off + g, lane * 32u + 32u);
    if (lo >= hi) return 0;
    const uint32_t n = hi - lo;
    return (n == 32u ? 0xffffffffu : ((1u << n) - 1u)) << (lo - lane * 32u);
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
            e.warp_mask = mask; e.tb = tb; e.gran_off = goff; e.gran_len = glen; e.pad = 0; e.pad2 = 0;
            p.trace[(size_t)mtb * p.trace_cap + seq] = e;
        }
        p.trace_count[mtb] = seq + 1;
    }
    seq++;
}

/* ------------------------------------------------------------------ executor
 * Alg. 1 L29-43: wait for dispatch, run the body, then the
 * deferred release: the last warp of a TB returns its shmem granules and
 * barrier ID through the scheduler's mailbox (markSMForDealloc), the last warp
 * of the task posts its completion record, every warp returns itself. */
__device__ void executor(MtbShared& S, char* arena, const MkParams& p, int mtb, int w)
{
    const uint32_t lane = threadIdx.x & 31u;
    uint32_t phase = 0, stage_phase = 0;
    for (;;) {
        mbar_wait(&S.exec_bar[w], phase);
        phase ^= 1u;
        const WarpSlot s = S.wt[w];
        if (s.task == SLOT_TERMINATE) return;
        const TaskEntry& t = S.tasks[s.task];
        uint64_t t0 = 0;
        if (p.trace_cap) t0 = globaltimer_ns();
        TaskEnv env{s, arena, &S.stage_bar[w], &stage_phase, &p.dctl->error};
        if (!run_body(t.func_id, env, t.args) && lane == 0) atomicOr(&p.dctl->error, PAGODA_DEVERR_BAD_FUNC);
        __syncwarp();
        if (lane == 0) {
            /* this warp's global writes -> visible GPU-wide before anyone learns the warp is done */
            __threadfence();
            if (p.trace_cap) {
                uint32_t* cnt = &p.exec_count[mtb * 32 + w];
                const uint32_t i = *cnt;
                if (i < p.trace_cap) {
                    ExecRecord r{s.task_id, s.tb, (uint16_t)mtb, (uint16_t)w, t0, globaltimer_ns()};
                    p.exec_trace[((size_t)mtb * 32 + w) * p.trace_cap + i] = r;
                }
                *cnt = i + 1;
            }
            if (atomicSub(&S.tb_warps_left[s.tbslot], 1u) == 1u) atomicOr(&S.mb_tbs, 1u << s.tbslot);
            if (atomicSub(&S.task_warps_left[s.task], 1u) == 1u) {
                /* last warp of the task (Alg. 1 L41-42): the task's writes, ordered before the
                 * counter decrements of all its warps, become visible system-wide before the
                 * completion record the host polls (a posted PCIe write, no handshake). */
                st_release_sys(&p.comp[s.task_id & p.comp_mask], (int64_t)s.task_id);
                atomicOr(&S.mb_tasks, 1u << s.task);
            }
            __threadfence_block();   /* TB / task frees are visible before the warp frees itself */
            atomicOr(&S.mb_warps, 1u << w);
        }
        __syncwarp();
    }
}

/* ------------------------------------------------------------------ ingest
 * Replaces the paper's one-cudaMemcpy-per-spawn with ready-field pipelining
 * (P:516-539): the host publishes a doorbell after writing entries; this warp
 * acquires it over PCIe, pulls the entries with asynchronous 16-byte copies
 * (many in flight, no registers held) into shared memory, writes them to the
 * device ring and releases the device tail. */
constexpr int kIngestBatch = 256;                       /* entries per round (16 KiB staging) */
constexpr uint32_t kIngestStageBytes = kIngestBatch * 64;

__device__ void ingest(const MkParams& p, char* stage_buf)
{
    const uint32_t lane = threadIdx.x & 31u;
    const uint64_t R = (uint64_t)p.ring_mask + 1;
    uint64_t copied = 0;
    uint32_t last_err = 0;
    int idle = 0;
    for (;;) {
        uint64_t pub = 0, head = 0;
        uint32_t term = 0, err = 0;
        if (lane == 0) {
            pub = ld_acquire_sys(&p.hctl->published);
            term = ld_relaxed_sys32(&p.hctl->terminate);
            head = ld_acquire_gpu(&p.dctl->head);
            err = *(volatile uint32_t*)&p.dctl->error;
            if (err != last_err) st_relaxed_sys32(&p.hctl->error, err);
        }
        pub = __shfl_sync(0xffffffffu, pub, 0);
        term = __shfl_sync(0xffffffffu, term, 0);
        head = __shfl_sync(0xffffffffu, head, 0);
        last_err = __shfl_sync(0xffffffffu, err, 0);
        if (pub > copied) {
            uint64_t n = pub - copied;
            const uint64_t space = R - (copied - head);
            if (n > space) n = space;
            if (n > (uint64_t)kIngestBatch) n = kIngestBatch;
            if (n == 0) {              /* device ring full: wait for the schedulers */
                __nanosleep(200);
                continue;
            }
            const uint32_t chunks = (uint32_t)n * 4u;
            for (uint32_t c = lane; c < chunks; c += 32u) {
                const uint64_t e = (copied + (c >> 2)) & p.ring_mask;
                cp_async16(stage_buf + c * 16u, reinterpret_cast<const int4*>(p.hring + e) + (c & 3u));
            }
            cp_async_wait_all();
            __syncwarp();
            for (uint32_t c = lane; c < chunks; c += 32u) {
                const uint64_t e = (copied + (c >> 2)) & p.ring_mask;
                const int4 v = *reinterpret_cast<const int4*>(stage_buf + c * 16u);
                __stcg(reinterpret_cast<int4*>(p.dring + e) + (c & 3u), v);
            }
            __syncwarp();
            copied += n;
            if (lane == 0) {
                st_release_gpu(&p.dctl->tail, copied);   /* entries before the tail are complete */
                st_relaxed_sys(&p.hctl->consumed, copied); /* host may now reuse those ring slots */
            }
            idle = 0;
        } else if (term) {
            if (lane == 0) st_release_gpu32(&p.dctl->stop, 1u);
            return;
        } else if (++idle > 64) {
            __nanosleep(256);
        }
    }
}

/* ------------------------------------------------------------------ scheduler
 * Alg. 1 L1-28 + Alg. 2, re-designed: one warp per MTB owns the
 * MTB's free masks (warps, TB records, task slots, barrier IDs: one word each;
 * granules: a 1024-bit lane-distributed bitmap).  It claims entries from the
 * device ring only while it has free resources, in ring order, so tasks flow
 * to whichever MTB frees resources first. */
struct Sched {
    uint32_t free_w, free_task, free_tbs, free_bar, exec_mask;
    uint32_t fg;         /* this lane's 32 granule bits */
    uint32_t ph, pt;     /* pending FIFO of claimed, unplaced task slots */
    uint32_t seq;        /* ledger clock */
};

__device__ __forceinline__ uint32_t nth_set_bit(uint32_t mask, uint32_t n)
{   /* 0-based n-th set bit position (mask must have > n bits) */
    return __fns(mask, 0, (int)n + 1);
}

__device__ bool sched_place(MtbShared& S, Sched& st, const MkParams& p, int mtb, uint32_t slot)
{
    const uint32_t lane = threadIdx.x & 31u;
    const TaskEntry& e = S.tasks[slot];
    const uint32_t wtb = e.warps_tb, ntb = e.n_tb, gtb = e.gran_tb;
    const bool need_bar = (e.flags & 1u) && wtb > 1;
    if ((uint32_t)__popc(st.free_w) < wtb * ntb || (uint32_t)__popc(st.free_tbs) < ntb ||
        (need_bar && (uint32_t)__popc(st.free_bar) < ntb))
        return false;
    if (gtb) {   /* feasibility of all TBs' shared memory first (all-or-nothing per task) */
        uint32_t fg2 = st.fg;
        for (uint32_t j = 0; j < ntb; j++) {
            const int off = bm_first_fit(fg2, gtb, lane);
            if (off < 0) return false;
            fg2 &= ~bm_range_bits((uint32_t)off, gtb, lane);
        }
    }
    const uint64_t id = e.id;
    const uint16_t threads = e.threads_tb;
    if (lane == 0) S.task_warps_left[slot] = wtb * ntb;
    uint32_t all = 0;
    for (uint32_t j = 0; j < ntb; j++) {
        const uint32_t tbs = __ffs(st.free_tbs) - 1;
        st.free_tbs &= ~(1u << tbs);
        uint32_t m = 0, fw = st.free_w;
        for (uint32_t i = 0; i < wtb; i++) {
            m |= fw & (0u - fw);   /* lowest free warp */
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
            off = (uint32_t)bm_first_fit(st.fg, gtb, lane);
            st.fg &= ~bm_range_bits(off, gtb, lane);
        }
        if (lane == 0) {
            S.tb_warps_left[tbs] = wtb;
            S.tb_goff[tbs] = (uint16_t)off;
            S.tb_glen[tbs] = (uint16_t)gtb;
            S.tb_bar[tbs] = (uint8_t)bar;
            S.tb_task[tbs] = id;
            S.tb_idx[tbs] = (uint16_t)j;
        }
        trace_ev(p, mtb, st.seq, 1, id, (uint16_t)j, m, (uint16_t)off, (uint16_t)gtb, (uint8_t)bar);
        if ((m >> lane) & 1u) {   /* Alg. 2 L9-12: lane l fills warp l's WarpTable slot */
            WarpSlot ws;
            ws.smem_off = off * PAGODA_GRANULE;
            ws.smem_bytes = gtb * PAGODA_GRANULE;
            ws.tb = (uint16_t)j;
            ws.threads_tb = threads;
            ws.task = (uint8_t)slot;
            ws.warp_in_tb = (uint8_t)__popc(m & ((1u << lane) - 1u));
            ws.warps_tb = (uint8_t)wtb;
            ws.n_tb = (uint8_t)ntb;
            ws.bar_id = (uint8_t)bar;
            ws.tbslot = (uint8_t)tbs;
            ws.pad0 = 0;
            ws.task_id = id;
            S.wt[lane] = ws;
        }
        all |= m;
    }
    __syncwarp();   /* counters written by lane 0 happen-before every lane's release-arrive */
    if ((all >> lane) & 1u) mbar_arrive(&S.exec_bar[lane]);   /* Alg. 2 L14: exec <- 1 */
    return true;
}

/* Claim up to 32 entries at the device ring head that fit the free resources.
 * Entries are copied into free task slots BEFORE the CAS that claims them:
 * until the CAS succeeds no scheduler owns them, so the ingest warp cannot
 * have recycled their ring slots (it only reuses slots below the head). */
__device__ int sched_claim(MtbShared& S, Sched& st, const MkParams& p)
{
    const uint32_t lane = threadIdx.x & 31u;
    uint64_t head = 0, tail = 0;
    if (lane == 0) {
        head = ld_relaxed_gpu(&p.dctl->head);
        tail = ld_acquire_gpu(&p.dctl->tail);
    }
    head = __shfl_sync(0xffffffffu, head, 0);
    tail = __shfl_sync(0xffffffffu, tail, 0);
    if (head >= tail) return 0;
    uint32_t n = (uint32_t)min((uint64_t)32, tail - head);
    n = min(n, (uint32_t)__popc(st.free_task));
    n = min(n, 32u - (st.pt - st.ph));
    if (n == 0) return 0;
    /* speculative copy: 4 x 16 B per entry, L2 only (the slot may hold an older lap in L1) */
    for (uint32_t c = lane; c < n * 4u; c += 32u) {
        const uint32_t i = c >> 2;
        const TaskEntry* src = p.dring + ((head + i) & p.ring_mask);
        const int4 v = __ldcg(reinterpret_cast<const int4*>(src) + (c & 3u));
        reinterpret_cast<int4*>(&S.tasks[nth_set_bit(st.free_task, i)])[c & 3u] = v;
    }
    __syncwarp();
    /* needs of entry `lane`; inclusive prefix sums over the lanes */
    uint32_t nw = 0, nt = 0, nb = 0, ng = 0, my_slot = 0;
    if (lane < n) {
        my_slot = nth_set_bit(st.free_task, lane);
        const TaskEntry& e = S.tasks[my_slot];
        nw = (uint32_t)e.warps_tb * e.n_tb;
        nt = e.n_tb;
        nb = ((e.flags & 1u) && e.warps_tb > 1) ? e.n_tb : 0;
        ng = (uint32_t)e.gran_tb * e.n_tb;
    }
#pragma unroll
    for (int d = 1; d < 32; d <<= 1) {
        const uint32_t a = __shfl_up_sync(0xffffffffu, nw, d), b = __shfl_up_sync(0xffffffffu, nt, d);
        const uint32_t c = __shfl_up_sync(0xffffffffu, nb, d), g = __shfl_up_sync(0xffffffffu, ng, d);
        if (lane >= (uint32_t)d) { nw += a; nt += b; nb += c; ng += g; }
    }
    const uint32_t free_g = __reduce_add_sync(0xffffffffu, (uint32_t)__popc(st.fg));
    const bool fit = lane < n && nw <= (uint32_t)__popc(st.free_w) && nt <= (uint32_t)__popc(st.free_tbs) &&
                     nb <= (uint32_t)__popc(st.free_bar) && ng <= free_g;
    const uint32_t fb = __ballot_sync(0xffffffffu, fit);
    const uint32_t k = (fb == 0xffffffffu) ? 32u : (uint32_t)(__ffs(~fb) - 1);
    if (k == 0) return 0;
    bool ok = false;
    if (lane == 0) ok = cas_acq_rel_gpu(&p.dctl->head, head, head + k);
    ok = __shfl_sync(0xffffffffu, (int)ok, 0) != 0;
    if (!ok) return -1;
    if (lane < k) S.pend[(st.pt + lane) & 31u] = (uint8_t)my_slot;
    uint32_t used = 0;
    for (uint32_t i = 0; i < k; i++) used |= 1u << nth_set_bit(st.free_task, i);
    st.free_task &= ~used;
    st.pt += k;
    __syncwarp();
    return (int)k;
}

__device__ void scheduler(MtbShared& S, const MkParams& p, int mtb, int arena_granules)
{
    const uint32_t lane = threadIdx.x & 31u;
    Sched st;
    st.exec_mask = 0;
    for (int w = 1; w <= p.exec_warps && w < 32; w++)
        if (!(mtb == 0 && w == kIngestWarp)) st.exec_mask |= 1u << w;
    st.free_w = st.exec_mask;
    st.free_task = 0xffffffffu;
    st.free_tbs = 0xffffffffu;
    st.free_bar = 0xfffeu;        /* named barriers 1..15; 0 belongs to the MTB */
    st.fg = bm_range_bits(0, (uint32_t)arena_granules, lane);
    st.ph = st.pt = 0;
    st.seq = 0;
    uint32_t backoff = 0;
    for (;;) {
        bool progress = false;
        /* ---- fold the mailboxes (deallocMarkedSM, Alg. 1 L22) */
        uint32_t mw = 0, mt = 0, mk = 0;
        if (lane == 0) {
            if (*(volatile uint32_t*)&S.mb_warps) mw = atomicExch(&S.mb_warps, 0u);
            __threadfence_block();
            if (*(volatile uint32_t*)&S.mb_tbs) mt = atomicExch(&S.mb_tbs, 0u);
            if (*(volatile uint32_t*)&S.mb_tasks) mk = atomicExch(&S.mb_tasks, 0u);
        }
        mw = __shfl_sync(0xffffffffu, mw, 0);
        mt = __shfl_sync(0xffffffffu, mt, 0);
        mk = __shfl_sync(0xffffffffu, mk, 0);
        if (mw | mt | mk) {
            progress = true;
            for (uint32_t b = mt; b; b &= b - 1u) {
                const uint32_t tbs = __ffs(b) - 1;
                const uint32_t goff = S.tb_goff[tbs], glen = S.tb_glen[tbs], bar = S.tb_bar[tbs];
                if (glen) st.fg |= bm_range_bits(goff, glen, lane);
                if (bar) st.free_bar |= 1u << bar;
                st.free_tbs |= 1u << tbs;
                if (p.trace_cap)
                    trace_ev(p, mtb, st.seq, 3, S.tb_task[tbs], S.tb_idx[tbs], 0, (uint16_t)goff, (uint16_t)glen,
                             (uint8_t)bar);
            }
            if (p.trace_cap) {
                for (uint32_t b = mw; b; b &= b - 1u) {
                    const uint32_t w = __ffs(b) - 1;
                    trace_ev(p, mtb, st.seq, 2, S.wt[w].task_id, S.wt[w].tb, 1u << w, 0, 0, 0);
                }
            }
            st.free_w |= mw;
            st.free_task |= mk;
        }
        /* ---- place claimed tasks in FIFO order (Alg. 1 L14-28) */
        while (st.ph != st.pt) {
            if (!sched_place(S, st, p, mtb, S.pend[st.ph & 31u])) break;
            st.ph++;
            progress = true;
        }
        /* ---- claim more while resources are free */
        if (st.ph == st.pt && st.free_w && st.free_task) {
            const int k = sched_claim(S, st, p);
            if (k != 0) progress = true;   /* k < 0: lost a CAS race; retry at once */
        }
        if (progress) {
            backoff = 0;
            continue;
        }
        /* ---- idle */
        if (st.free_w == st.exec_mask && st.ph == st.pt) {
            uint32_t stop = 0;
            if (lane == 0) stop = ld_acquire_gpu32(&p.dctl->stop);
            stop = __shfl_sync(0xffffffffu, stop, 0);
            if (stop) {
                uint64_t head = 0, tail = 0;
                if (lane == 0) {
                    head = ld_relaxed_gpu(&p.dctl->head);
                    tail = ld_acquire_gpu(&p.dctl->tail);
                }
                if (__shfl_sync(0xffffffffu, (int)(head >= tail), 0)) break;
            }
        }
        backoff = backoff ? min(backoff * 2u, 1024u) : 32u;
        __nanosleep(backoff);
    }
    /* drain: release every executor warp with a terminate slot */
    if ((st.exec_mask >> lane) & 1u) {
        S.wt[lane].task = SLOT_TERMINATE;
        mbar_arrive(&S.exec_bar[lane]);
    }
    if (lane == 0) atomicAdd(&p.dctl->exited, 1u);
}

/* ------------------------------------------------------------------ the kernel */
template <int kMinBlocks>
__global__ void __launch_bounds__(1024, kMinBlocks) master_kernel(MkParams p)
{
    extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
    MtbShared& S = *reinterpret_cast<MtbShared*>(pagoda_mk_smem);
    char* arena = reinterpret_cast<char*>(pagoda_mk_smem) + kArenaOffset;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31, mtb = blockIdx.x;
    int arena_granules = p.arena_granules;
    char* ingest_stage = nullptr;
    if (mtb == 0) {   /* MTB 0 lends the top of its arena to the ingest warp */
        arena_granules -= (int)(kIngestStageBytes / PAGODA_GRANULE);
        ingest_stage = arena + (size_t)arena_granules * PAGODA_GRANULE;
    }
    if (warp == 0) {
        mbar_init(&S.exec_bar[lane], 1);
        mbar_init(&S.stage_bar[lane], 1);
        if (lane == 0) {
            S.mb_warps = S.mb_tbs = S.mb_tasks = 0;
            asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
        }
    }
    __syncthreads();
    if (warp == 0) scheduler(S, p, mtb, arena_granules);
    else if (mtb == 0 && warp == kIngestWarp) ingest(p, ingest_stage);
    else if (warp <= p.exec_warps) executor(S, arena, p, mtb, warp);
}

template __global__ void master_kernel<1>(MkParams);
template __global__ void master_kernel<2>(MkParams);

/* host-side launcher (called by runtime.cu) */
cudaError_t launch_master(int mtbs_per_sm, int n_mtb, size_t smem_bytes, cudaStream_t stream, MkParams* params,
                          int* regs_out)
{
    const void* fn = mtbs_per_sm == 2 ? reinterpret_cast<const void*>(&master_kernel<2>)
                                      : reinterpret_cast<const void*>(&master_kernel<1>);
    cudaError_t err = cudaFuncSetAttribute(fn, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem_bytes);
    if (err != cudaSuccess) return err;
    cudaFuncAttributes attr;
    if (cudaFuncGetAttributes(&attr, fn) == cudaSuccess && regs_out) *regs_out = attr.numRegs;
    int per_sm = 0;
    err = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, fn, 1024, smem_bytes);
    if (err != cudaSuccess) return err;
    if (per_sm < mtbs_per_sm) return cudaErrorCooperativeLaunchTooLarge;
    void* args[] = {params};
    return cudaLaunchCooperativeKernel(fn, dim3(n_mtb), dim3(1024), args, smem_bytes, stream);
}

} // namespace pagoda
