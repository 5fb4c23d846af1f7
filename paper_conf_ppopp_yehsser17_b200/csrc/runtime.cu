/*
 * runtime.cu — host side of the C ABI in include/pagoda.h.
 *
 * Spawn path (P:500-539 re-designed):
 *   id = next_id++                       (the TaskTable index, also the task id)
 *   wait until ring slot id mod R is free (GPU-posted `consumed` > id - R)
 *   wait until completion slot id mod C is free (task id - C done)
 *   write the 64-byte entry into the pinned host ring
 *   in-order commit: wait for published == id, then published = id + 1
 * The doorbell store is the only thing the GPU polls; no CUDA call per spawn.
 *
 * Completion (replaces the lazy aggregate copy-back + timeout):
 * the task's last warp writes comp[id mod C] = id into pinned memory; a slot
 * holds the newest finished occupant, and occupant id + C is only spawned after
 * id is done, so "comp[id mod C] >= id" <=> id done.
 */
#include <cuda.h>   /* driver types for cuStreamWriteValue64 (resolved at run time, no link) */
#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>
#include <time.h>
#include <immintrin.h>

#include <algorithm>
#include <atomic>
#include <chrono>
#include <condition_variable>
#include <mutex>
#include <thread>
#include <vector>

#include "bodies.cuh"
#include "mk_layout.cuh"
#include "pagoda.h"

namespace pagoda {
cudaError_t launch_master(int mtbs_per_sm, int n_mtb, size_t smem_bytes, cudaStream_t stream, MkParams* params,
                          int* regs_out);
cudaError_t set_tdes_const_keys(const void* keys384, uint64_t tables_ptr);
cudaError_t set_dct_const_coef(const void* coef256, uint64_t coef_ptr);
}
using namespace pagoda;

static const int kSpawnChunk = 64;   /* batched spawns publish the doorbell once per chunk */

struct pagoda_ctx {
    pagoda_config cfg;
    int device = 0, sm_count = 0, n_mtb = 0, regs = 0;
    int max_task_warps = 31;          /* largest warps*n_tb every task-running scheduling group can host */
    uint32_t max_task_granules = 0;   /* largest n_tb*granules every task-running group can host */
    int max_bars = PAGODA_BAR_IDS;    /* named barrier IDs of the smallest group (15; 7 with two groups) */
    int n_grp = 1;                    /* scheduling groups per MTB */
    uint32_t R = 0, C = 0;
    cudaStream_t stream = nullptr;
    /* pinned, mapped */
    HostCtl* hctl = nullptr;
    TaskEntry* hring = nullptr;
    volatile int64_t* comp = nullptr;
    /* device */
    TaskEntry* dring = nullptr;
    uint32_t* resident_src = nullptr;
    uint32_t* dseq = nullptr;
    uint64_t* dq = nullptr;                 /* device completion queue (n_mtb > 1) */
    uint32_t* grp = nullptr;                /* per-id TB counters of spread tasks */
    DevCtl* dctl = nullptr;
    LedgerEvent* trace = nullptr;
    uint32_t* trace_count = nullptr;
    ExecRecord* exec_trace = nullptr;
    uint64_t* life = nullptr;               /* PAGODA_LIFECYCLE stamps */
    uint32_t* exec_count = nullptr;
    /* host state */
    std::atomic<uint64_t> next_id{0};
    std::atomic<uint64_t> published{0};     /* host mirror of hctl->published */
    std::atomic<uint64_t> consumed_cache{0};
    std::atomic<uint64_t> low{0};           /* every id < low is done */
    std::mutex low_mtx;
    std::atomic<int> shutting{0};
    std::atomic<int> faulted{0};
    std::vector<int64_t> warps_prefix;      /* warps_prefix[id mod C] = sum of warps of tasks <= id */
    std::atomic<int64_t> warps_spawned{0};
    /* helper producer threads of pagoda_taskSpawnShapesMT (Fig. 1a: several CPU threads
     * spawn into the TaskTable), started on first use and kept until shutdown */
    struct SpawnJob {
        const int32_t* shapes;
        const char* args;
        size_t stride, bytes;
        pagoda_task_t* ids;
        int n, P;
    } job{};
    std::vector<std::thread> helpers;
    std::mutex mt_mtx;                      /* one multi-producer spawn at a time */
    std::atomic<uint64_t> job_gen{0};
    std::atomic<int> job_left{0};
    std::atomic<int> job_unvalidated{0};    /* producers still validating their blocks */
    std::atomic<int64_t> job_rc{0};
    std::atomic<int> helpers_quit{0};
    /* MasterKernel session */
    MkParams params;
    size_t smem = 0;
    cudaEvent_t ev_start = nullptr, ev_stop = nullptr;
    std::atomic<int> running{0};
    std::mutex session_mtx;
    int sessions = 0;
    /* PAGODA_CE_INGEST: the copy-engine ingest thread (one per context, started at init) */
    std::thread ce_thread;
    std::atomic<int> ce_cmd{0};             /* 0 idle, 1 run a session, 2 flush and stop it, 3 abort it, 4 exit */
    std::atomic<int> ce_busy{0};            /* 1 while the thread serves a session */
    std::mutex ce_mtx;
    std::condition_variable ce_cv;
    cudaStream_t ce_stream = nullptr;
    cudaEvent_t ce_ev[8] = {};             /* kCeInFlight (<= 8) copies' completion */
    uint64_t ce_issued = 0;                 /* ring positions whose copy was issued (carries over sessions) */
    CUdeviceptr d_tail = 0, d_stop = 0;
};

static inline uint64_t now_ns();
#ifndef PAGODA_CE_INFLIGHT
#define PAGODA_CE_INFLIGHT 3
#endif
static constexpr int kCeInFlight = PAGODA_CE_INFLIGHT;
#ifndef PAGODA_FWD_4MTB
#define PAGODA_FWD_4MTB 1   /* completion forwarders at 4 MTBs/SM (MTB 0 has 16 warps) */
#endif

/* cuStreamWriteValue64 / 32 through the runtime's driver entry points (no -lcuda) */
typedef CUresult (*WriteValue64Fn)(CUstream, CUdeviceptr, cuuint64_t, unsigned int);
typedef CUresult (*WriteValue32Fn)(CUstream, CUdeviceptr, cuuint32_t, unsigned int);
static WriteValue64Fn g_wv64 = nullptr;
static WriteValue32Fn g_wv32 = nullptr;
static bool load_stream_memops()
{
    static std::once_flag once;
    std::call_once(once, [] {
        cudaDriverEntryPointQueryResult q;
        void* f = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue64", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            g_wv64 = (WriteValue64Fn)f;
        f = nullptr;
        if (cudaGetDriverEntryPoint("cuStreamWriteValue32", &f, cudaEnableDefault, &q) == cudaSuccess &&
            q == cudaDriverEntryPointSuccess)
            g_wv32 = (WriteValue32Fn)f;
        cudaGetLastError();
    });
    return g_wv64 && g_wv32;
}

/* The copy-engine ingest (PAGODA_CE_INGEST), one session: copies the published, not yet issued
 * span of the host ring into the device ring (one cudaMemcpyAsync per contiguous part), then a
 * stream memory operation ordered after it (cuStreamWriteValue64, CU_STREAM_WRITE_VALUE_DEFAULT:
 * a memory barrier first) sets DevCtl.tail = the span's end: the schedulers' publication (ticket t
 * is published once an acquire of tail sees > t).  An event behind it tells this thread when the
 * copy has read the host ring: HostCtl.consumed (the spawners may reuse those slots).  A device
 * ring cell is overwritten only once the ticket of the previous lap handed it back (HostCtl.handed,
 * posted by MTB 0's scanner warp).  Command 2: flush what is published, then DevCtl.stop = 1
 * behind it; 3: stop = kStopAbort at once. */
static void ce_session(pagoda_ctx* c)
{
    const uint64_t R = c->R;
    uint64_t issued = c->ce_issued;
    /* at most kCeInFlight copies in the stream: a small copy and its memory operation take a few
     * microseconds on the GPU whatever their size, so a new copy waits for the oldest to land and
     * then takes everything published meanwhile */
    constexpr uint64_t kChunk = 2048;   /* entries per copy: a backlog (a prespawned session) streams in
                                           128 KiB steps, the first tasks start after the first one */
    uint64_t ends[kCeInFlight];
    int nq = 0, qh = 0;
    int idle = 0;
    /* PAGODA_CE_STATS (environment): per session, copies issued, entries, ns in the issuing calls,
     * ns with the stream full (kCeInFlight copies outstanding while entries wait), ns idle */
    static const bool stats = getenv("PAGODA_CE_STATS") != nullptr;
    uint64_t st_copies = 0, st_entries = 0, st_issue_ns = 0, st_full_ns = 0, st_idle_ns = 0, t_prev = now_ns();
    const uint64_t t_begin = t_prev;
    for (;;) {
        const int cmd = c->ce_cmd.load(std::memory_order_acquire);
        if (cmd == 3 || cmd == 4) {
            g_wv32((CUstream)c->ce_stream, c->d_stop, kStopAbort, 0);
            break;
        }
        while (nq && cudaEventQuery(c->ce_ev[qh]) == cudaSuccess) {   /* landed: its host slots are free */
            c->hctl->consumed = ends[qh];
            qh = (qh + 1) % kCeInFlight;
            nq--;
        }
        const uint64_t pub = c->hctl->published;
        std::atomic_thread_fence(std::memory_order_acquire);   /* entries below pub were written first */
        const uint64_t limit = std::min<uint64_t>(std::min<uint64_t>(pub, c->hctl->handed + R), issued + kChunk);
        if (stats) {   /* account the time since the last look to the state seen then */
            const uint64_t t = now_ns();
            if (limit > issued && nq >= kCeInFlight) st_full_ns += t - t_prev;
            else if (limit <= issued) st_idle_ns += t - t_prev;
            t_prev = t;
        }
        if (limit > issued && nq < kCeInFlight) {
            const uint64_t t_issue = stats ? now_ns() : 0;
            const uint64_t e0 = issued & (R - 1);
            const uint64_t n = limit - issued, n1 = std::min<uint64_t>(n, R - e0);
            cudaError_t ce = cudaMemcpyAsync(c->dring + e0, c->hring + e0, n1 * sizeof(TaskEntry), cudaMemcpyHostToDevice,
                                             c->ce_stream);
            if (ce == cudaSuccess && n1 < n)
                ce = cudaMemcpyAsync(c->dring, c->hring, (n - n1) * sizeof(TaskEntry), cudaMemcpyHostToDevice, c->ce_stream);
            const CUresult r1 = ce == cudaSuccess ? g_wv64((CUstream)c->ce_stream, c->d_tail, limit, 0) : CUDA_ERROR_UNKNOWN;
            const int slot = (qh + nq) % kCeInFlight;
            if (r1 != CUDA_SUCCESS || cudaEventRecord(c->ce_ev[slot], c->ce_stream) != cudaSuccess) {
                fprintf(stderr, "pagoda: copy-engine ingest: stream operation failed (%s, %d): ingest stops\n",
                        cudaGetErrorString(ce), (int)r1);
                c->faulted.store(1);
                g_wv32((CUstream)c->ce_stream, c->d_stop, kStopAbort, 0);   /* let the MasterKernel leave */
                break;
            }
            ends[slot] = limit;
            nq++;
            if (stats) {
                st_copies++;
                st_entries += limit - issued;
                t_prev = now_ns();
                st_issue_ns += t_prev - t_issue;
            }
            issued = limit;
            idle = 0;
            continue;
        }
        if (cmd == 2 && issued >= pub) {   /* everything published is issued: drain and exit */
            g_wv32((CUstream)c->ce_stream, c->d_stop, 1u, 0);
            break;
        }
        if (++idle > 1024) std::this_thread::yield();
        else _mm_pause();
    }
    cudaStreamSynchronize(c->ce_stream);
    c->hctl->consumed = issued;
    c->ce_issued = issued;
    if (stats)
        fprintf(stderr, "pagoda CE: %llu copies, %.1f entries/copy, issue %.2f us/copy, full %.1f us, idle %.1f us, "
                        "session %.1f us\n",
                (unsigned long long)st_copies, st_copies ? (double)st_entries / st_copies : 0.0,
                st_copies ? st_issue_ns * 1e-3 / st_copies : 0.0, st_full_ns * 1e-3, st_idle_ns * 1e-3,
                (now_ns() - t_begin) * 1e-3);
}

/* The context's ingest thread: serves sessions (ce_cmd 1/2/3) and idles in between (spinning
 * for 50 ms after a session, so back-to-back sessions start without a wake-up, then blocked). */
static void ce_thread_main(pagoda_ctx* c)
{
    cudaSetDevice(c->device);
    for (;;) {
        int cmd = c->ce_cmd.load(std::memory_order_acquire);
        const uint64_t t0 = now_ns();
        while (cmd == 0 && now_ns() - t0 < 50000000ull) {
            std::this_thread::yield();
            cmd = c->ce_cmd.load(std::memory_order_acquire);
        }
        if (cmd == 0) {
            std::unique_lock<std::mutex> lk(c->ce_mtx);
            c->ce_cv.wait(lk, [&] { return c->ce_cmd.load(std::memory_order_acquire) != 0; });
            cmd = c->ce_cmd.load(std::memory_order_acquire);
        }
        if (cmd == 4) return;
        ce_session(c);
        /* the session is over for this thread: back to idle unless told to exit meanwhile */
        int expect = c->ce_cmd.load(std::memory_order_acquire);
        while (expect != 4 && !c->ce_cmd.compare_exchange_weak(expect, 0)) { }
        c->ce_busy.store(0, std::memory_order_release);
        if (expect == 4) return;
    }
}
static void ce_command(pagoda_ctx* c, int cmd)
{
    {
        std::lock_guard<std::mutex> lk(c->ce_mtx);
        c->ce_cmd.store(cmd, std::memory_order_release);
    }
    c->ce_cv.notify_all();
}

/* Every live context, by device: the MasterKernel's constant bank (registered 3DES keys, DCT
 * coefficients) is one per device and process, so registration must not race a running
 * MasterKernel of ANY context on that device (start_kernel takes the same lock). */
static std::mutex g_ctx_mtx;
static std::vector<pagoda_ctx*> g_ctxs;

/* ------------------------------------------------------------------ helpers */
static inline uint64_t now_ns()
{
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
}

/* Device error bits that are contract violations (the context is unusable after
 * them: every later call returns -EIO); PAGODA_DEVERR_LAYOUT is only a notice. */
static const uint32_t kFatalDevErr = PAGODA_DEVERR_SYNC_WITHOUT_FLAG | PAGODA_DEVERR_BAD_FUNC;
static inline bool dev_fault(const pagoda_ctx* c)
{
    return (c->hctl->error & kFatalDevErr) != 0 || c->faulted.load(std::memory_order_relaxed);
}

/* Spin with pause / yield back-off; every ~1 ms check device faults and the
 * watchdog.  pred() returns true when done. */
template <class Pred>
static int spin_until(pagoda_ctx* c, Pred pred)
{
    if (dev_fault(c)) return -EIO;
    if (pred()) return 0;
    const uint64_t t0 = now_ns();
    uint64_t last_check = t0;
    uint64_t spins = 0;
    for (;;) {
        if (pred()) return 0;
        if (++spins < 4096) {
            _mm_pause();
            continue;
        }
        if ((spins & 63) == 0) std::this_thread::yield();
        else _mm_pause();
        const uint64_t t = now_ns();
        if (t - last_check > 1000000ull) {
            last_check = t;
            if (dev_fault(c)) return -EIO;
            if (!c->running.load(std::memory_order_acquire)) return pred() ? 0 : -EAGAIN;   /* stopped */
            cudaError_t q = cudaStreamQuery(c->stream);
            if (q != cudaErrorNotReady) {   /* MasterKernel gone while it should run: fault */
                if (pred()) return 0;
                c->faulted.store(1);
                return -EIO;
            }
            if (c->cfg.watchdog_s > 0 && (double)(t - t0) * 1e-9 > c->cfg.watchdog_s) return -ETIMEDOUT;
        }
    }
}

static void advance_low(pagoda_ctx* c, uint64_t limit)
{
    std::unique_lock<std::mutex> lk(c->low_mtx, std::try_to_lock);
    if (!lk.owns_lock()) return;
    uint64_t l = c->low.load(std::memory_order_relaxed);
    const uint64_t mask = c->C - 1;
    while (l < limit && c->comp[l & mask] >= (int64_t)l) l++;
    c->low.store(l, std::memory_order_release);
}

/* ------------------------------------------------------------------ task shapes
 * A task whose thread blocks do not fit one MTB (all warps of a task in one
 * MTB, vs "64K threads" per task in Fig. 8) is spread
 * over k consecutive TaskTable entries ("a group"), each a run of at most
 * `cap` of its TBs that one MTB can host; it consumes k ids, the first is the
 * task's id, and the MasterKernel posts it when the last TB finished
 * (DESIGN.md "Readings" 6).  Sub-entries: flags bit 1, reserved = first TB
 * (low 16 bits) | the task's TB count (high 16 bits). */
struct Split {
    int wtb = 0, cap = 0, k = 0;
    uint32_t gtb = 0;
};

static int shape_check(const pagoda_ctx* c, const int32_t* s, Split& o)
{
    const int threads = s[0], n_tb = s[1], shmem = s[2], sync = s[3], func = s[4];
    if (threads < 1 || threads > 1024 || n_tb < 1 || shmem < 0) return -EINVAL;
    if (!known_func(func)) return -EINVAL;
    o.wtb = (threads + 31) / 32;
    o.gtb = ((uint32_t)shmem + PAGODA_GRANULE - 1) / PAGODA_GRANULE;
    if (o.wtb > c->max_task_warps || o.gtb > c->max_task_granules) return -EINVAL;   /* one TB must fit an MTB */
    if (o.wtb * n_tb <= c->max_task_warps && o.gtb * (uint32_t)n_tb <= c->max_task_granules &&
        !(sync && o.wtb > 1 && n_tb > c->max_bars)) {   /* fits one MTB (the common case: no divisions) */
        o.cap = n_tb;
        o.k = 1;
        return 0;
    }
    int cap = c->max_task_warps / o.wtb;
    if (o.gtb) cap = std::min<int>(cap, (int)(c->max_task_granules / o.gtb));
    if (sync && o.wtb > 1) cap = std::min(cap, c->max_bars);
    o.cap = cap;
    o.k = (n_tb + cap - 1) / cap;
    if (o.k > 1 && (n_tb > 65535 || (uint32_t)o.k > c->R / 4)) return -EINVAL;
    return 0;
}

/* consecutive tasks mostly share a shape: validate a shape once */
struct ShapeMemo {
    int32_t last[5] = {-1, -1, -1, -1, -1};
    Split sp;
    int rc = 0;
    int check(const pagoda_ctx* c, const int32_t* s, Split& out)
    {
        if (s[0] != last[0] || s[1] != last[1] || s[2] != last[2] || s[3] != last[3] || s[4] != last[4]) {
            rc = shape_check(c, s, sp);
            memcpy(last, s, sizeof last);
        }
        out = sp;
        return rc;
    }
};

/* write entry j of a task (id0 = the task's id) into the host ring slot id0 + j */
static inline void write_entry(pagoda_ctx* c, uint64_t id0, int j, const int32_t* s, const Split& sp, const void* args,
                               size_t args_bytes)
{
    TaskEntry e;
    memset(&e, 0, sizeof e);
    const int tb0 = j * sp.cap;
    e.id = id0;
    e.func_id = (uint16_t)s[4];
    e.threads_tb = (uint16_t)s[0];
    e.warps_tb = (uint8_t)sp.wtb;
    e.n_tb = (uint8_t)std::min(sp.cap, s[1] - tb0);
    e.gran_tb = (uint8_t)std::min<uint32_t>(sp.gtb, 255u);
    e.flags = (s[3] ? 1 : 0) | (sp.k > 1 ? kEntryGroup : 0);
    e.shmem_bytes = (uint32_t)s[2];
    e.reserved = sp.k > 1 ? ((uint32_t)tb0 | ((uint32_t)s[1] << 16)) : 0u;
    if (args_bytes) memcpy(e.args, args, args_bytes);
    const __m128i* src = reinterpret_cast<const __m128i*>(&e);
    __m128i* d = reinterpret_cast<__m128i*>(&c->hring[(id0 + (uint64_t)j) & (c->R - 1)]);
    _mm_store_si128(d + 0, _mm_load_si128(src + 0));
    _mm_store_si128(d + 1, _mm_load_si128(src + 1));
    _mm_store_si128(d + 2, _mm_load_si128(src + 2));
    _mm_store_si128(d + 3, _mm_load_si128(src + 3));
    if (j > 0) c->comp[(id0 + (uint64_t)j) & (c->C - 1)] = (int64_t)(id0 + (uint64_t)j);   /* internal ids: only
        the first is ever handed out, and the watermark passes them once it passed the first */
}

template <class ShapeOf>
static int64_t spawn_batch(pagoda_ctx* c, int n, ShapeOf shape_of, const void* args_base, size_t args_stride,
                           size_t args_bytes, pagoda_task_t* ids_out, bool validated = false);

static inline bool same_row(const int32_t* a, const int32_t* b)
{
    return a[0] == b[0] && a[1] == b[1] && a[2] == b[2] && a[3] == b[3] && a[4] == b[4];
}
/* Validate n contiguous shape rows (5 x int32 each) before any is spawned (all-or-nothing).  A row
 * equal to its predecessor needs no check; after 8 such rows the rest of the run is skipped 256 rows
 * per memcmp (rows k and k-1 equal for every k of a chunk iff the chunk equals itself shifted by one
 * row); a changed row is looked up in a 4096-entry cache of validated shapes (mixed workloads, config
 * 5, cycle through a few hundred).  65,536 uniform rows: ~150 -> ~40 us on the host, inside the
 * session that waits for the first spawn.  Returns 0 or the first error. */
static int validate_rows(const pagoda_ctx* c, const int32_t* shapes, int n)
{
    struct Ent {
        int32_t s[5];
        uint32_t gen;   /* valid for the call whose generation this is (no clearing per call) */
    };
    static thread_local Ent cache[4096];
    static thread_local uint32_t gen = 0;
    if (++gen == 0) {   /* wrapped: start over */
        for (Ent& e : cache) e.gen = 0;
        gen = 1;
    }
    int run = 0;
    for (int i = 0; i < n;) {
        const int32_t* r = shapes + 5 * (size_t)i;
        if (i > 0 && same_row(r, r - 5)) {   /* same as the previous row (already valid) */
            i++;
            if (++run >= 8)   /* a long run: whole chunks equal to themselves shifted by one row */
                while (i + 256 <= n && memcmp(shapes + 5 * (size_t)i, shapes + 5 * (size_t)(i - 1), 20 * 256) == 0)
                    i += 256;
            continue;
        }
        run = 0;
        const uint32_t h = ((uint32_t)r[0] * 2654435761u ^ (uint32_t)r[1] * 40503u ^ (uint32_t)r[2] * 2246822519u ^
                            (uint32_t)r[3] * 3266489917u ^ (uint32_t)r[4] * 668265263u) >> 20;
        Ent& e = cache[h];
        if (e.gen != gen || !same_row(e.s, r)) {
            Split sp;
            if (int rc = shape_check(c, r, sp)) return rc;
            memcpy(e.s, r, 20);
            e.gen = gen;
        }
        i++;
    }
    return 0;
}

/* Ring slot `last` (and every one before it) is free: the ingest warp has copied entry last - R. */
static bool ring_room(pagoda_ctx* c, uint64_t last)
{
    if (last < c->R) return true;
    uint64_t cur = c->consumed_cache.load(std::memory_order_acquire);
    if (cur > last - c->R) return true;
    const uint64_t v = c->hctl->consumed;
    while (v > cur && !c->consumed_cache.compare_exchange_weak(cur, v)) { }
    return v > last - c->R;
}
/* Completion slot `last` is free: task last - C is done. */
static bool comp_room(pagoda_ctx* c, uint64_t last)
{
    if (last < c->C || c->low.load(std::memory_order_acquire) > last - c->C) return true;
    advance_low(c, last - c->C + 1);
    return c->low.load(std::memory_order_acquire) > last - c->C;
}

/* Reserve K consecutive ids.  The id sequence never gets a hole: when the ring
 * or completion slots those ids need are taken and waiting could not free them
 * (PAGODA_NONBLOCKING_SPAWN, or a stopped session, where nothing drains the
 * ring), nothing is reserved and -EAGAIN returned.  Otherwise the caller waits
 * for the slots after reserving; if that wait then fails (device fault,
 * watchdog) the ids stay unpublished, so the context is marked faulted
 * (reserve_failed) and every later call returns -EIO instead of waiting for
 * them. */
static int reserve_ids(pagoda_ctx* c, uint64_t K, uint64_t* id0)
{
    const bool nonblock = (c->cfg.flags & PAGODA_NONBLOCKING_SPAWN) != 0;
    uint64_t cur = c->next_id.load(std::memory_order_acquire);
    for (;;) {
        const uint64_t last = cur + K - 1;
        const bool room = ring_room(c, last) && comp_room(c, last);
        if (!room && (nonblock || !c->running.load(std::memory_order_acquire))) return -EAGAIN;
        if (c->next_id.compare_exchange_weak(cur, cur + K, std::memory_order_acq_rel)) {
            *id0 = cur;
            return 0;
        }
    }
}
static int reserve_failed(pagoda_ctx* c, int rc)
{
    c->faulted.store(1, std::memory_order_release);
    return rc;
}

extern "C" {

void pagoda_config_default(pagoda_config* cfg)
{
    if (!cfg) return;
    memset(cfg, 0, sizeof *cfg);
    cfg->device = 0;
    cfg->mtbs_per_sm = 2;
    cfg->num_sms = 0;
    cfg->ring_entries = 1u << 16;
    cfg->comp_entries = 1u << 20;
    cfg->arena_bytes = 96 * 1024;
    cfg->exec_warps = 32;
    cfg->flags = 0;
    cfg->trace_events = 8192;
    cfg->watchdog_s = 60.0;
    cfg->sched_groups = 1;
}

static bool pow2(uint32_t x) { return x && !(x & (x - 1)); }

/* Launch one MasterKernel session on the context's stream, bracketed by CUDA
 * events recorded before and after the launch (ev_stop completes at kernel exit). */
static int start_kernel(pagoda_ctx* c)
{
    cudaSetDevice(c->device);
    if (c->life) cudaMemsetAsync(c->life, 0, (size_t)c->C * 8 * sizeof(uint64_t), c->stream);
    if (c->trace_count) {
        cudaMemsetAsync(c->trace_count, 0, (size_t)c->n_mtb * c->n_grp * sizeof(uint32_t), c->stream);
        cudaMemsetAsync(c->exec_count, 0, (size_t)c->n_mtb * 32 * sizeof(uint32_t), c->stream);
    }
    std::lock_guard<std::mutex> reg(g_ctx_mtx);   /* no constant-bank registration during the launch */
    c->params.ce_base = c->ce_issued;   /* (CE ingest) the scanner's first position */
    cudaEventRecord(c->ev_start, c->stream);
    cudaError_t e = launch_master(c->cfg.mtbs_per_sm, c->n_mtb, c->smem, c->stream, &c->params, &c->regs);
    if (e != cudaSuccess) {
        fprintf(stderr, "pagoda: MasterKernel launch failed: %s\n", cudaGetErrorString(e));
        cudaGetLastError();
        return -EIO;
    }
    cudaEventRecord(c->ev_stop, c->stream);   /* completes when the session's kernel exits */
    if (c->cfg.flags & PAGODA_CE_INGEST) {
        /* terminate already set (pagoda_start_drain): flush what is published, then stop */
        c->ce_busy.store(1, std::memory_order_release);
        ce_command(c, c->hctl->terminate ? 2 : 1);
    }
    c->running.store(1, std::memory_order_release);
    c->sessions++;
    return 0;
}

/* Ask the running session to drain and exit; wait (bounded) for it. */
static int stop_kernel(pagoda_ctx* c, bool abort_now = false)
{
    c->hctl->terminate = abort_now ? kStopAbort : 1;
    const bool ce = (c->cfg.flags & PAGODA_CE_INGEST) != 0;
    if (ce) ce_command(c, abort_now ? 3 : 2);
    const uint64_t t0 = now_ns();
    cudaError_t q;
    bool aborted = abort_now;
    while ((q = cudaStreamQuery(c->stream)) == cudaErrorNotReady) {
        std::this_thread::sleep_for(std::chrono::microseconds(20));
        const double waited = (double)(now_ns() - t0) * 1e-9;
        if (!aborted && c->cfg.watchdog_s > 0 && waited > c->cfg.watchdog_s) {
            /* abandon the queue: idle MTBs exit, tasks still running are waited for a while */
            fprintf(stderr, "pagoda: MasterKernel did not drain (watchdog): aborting the session\n");
            c->hctl->terminate = kStopAbort;
            if (ce) ce_command(c, 3);
            aborted = true;
        }
        if (aborted && waited > c->cfg.watchdog_s + 10.0) {
            fprintf(stderr, "pagoda: MasterKernel did not exit after abort\n");
            return -ETIMEDOUT;   /* still resident: buffers must not be freed */
        }
    }
    while (ce && c->ce_busy.load(std::memory_order_acquire)) std::this_thread::yield();   /* its stream synced */
    c->running.store(0, std::memory_order_release);
    if (aborted) {
        c->faulted.store(1);
        return -ETIMEDOUT;
    }
    if (q != cudaSuccess) {
        fprintf(stderr, "pagoda: MasterKernel error: %s\n", cudaGetErrorString(q));
        c->faulted.store(1);
        return -EIO;
    }
    /* reset the session flags for the next start; ring positions carry over,
     * except tickets handed out past the final tail, which are void: head = tail */
    c->hctl->terminate = 0;
    const uint32_t zero = 0;
    uint32_t derr = 0;   /* the device error word, whether or not the kernel posted it before exiting */
    cudaMemcpy(&derr, &c->dctl->error, 4, cudaMemcpyDeviceToHost);
    if (derr) c->hctl->error |= derr;
    uint64_t tail = 0;
    cudaMemcpy(&tail, &c->dctl->tail, 8, cudaMemcpyDeviceToHost);
    cudaMemcpy(&c->dctl->head, &tail, 8, cudaMemcpyHostToDevice);
    cudaMemcpy(&c->dctl->stop, &zero, 4, cudaMemcpyHostToDevice);
    cudaMemcpy(&c->dctl->exited, &zero, 4, cudaMemcpyHostToDevice);
    const uint32_t none = kIoSmidNone;   /* MTB 0 announces its SM again next session */
    cudaMemcpy(&c->dctl->io_smid, &none, 4, cudaMemcpyHostToDevice);
    if (cudaStreamSynchronize(c->stream) != cudaSuccess) return -EIO;
    return (c->hctl->error & kFatalDevErr) ? -EIO : 0;
}

static void free_ctx(pagoda_ctx* c)
{
    if (!c) return;
    {
        std::lock_guard<std::mutex> reg(g_ctx_mtx);
        g_ctxs.erase(std::remove(g_ctxs.begin(), g_ctxs.end(), c), g_ctxs.end());
    }
    c->helpers_quit.store(1, std::memory_order_release);
    for (auto& t : c->helpers) t.join();
    if (c->hctl) cudaFreeHost(c->hctl);
    if (c->hring) cudaFreeHost(c->hring);
    if (c->comp) cudaFreeHost((void*)c->comp);
    if (c->dring) cudaFree(c->dring);
    if (c->dseq) cudaFree(c->dseq);
    if (c->dq) cudaFree(c->dq);
    if (c->grp) cudaFree(c->grp);
    if (c->resident_src) cudaFree(c->resident_src);
    if (c->dctl) cudaFree(c->dctl);
    if (c->trace) cudaFree(c->trace);
    if (c->trace_count) cudaFree(c->trace_count);
    if (c->exec_trace) cudaFree(c->exec_trace);
    if (c->life) cudaFree(c->life);
    if (c->exec_count) cudaFree(c->exec_count);
    if (c->ce_thread.joinable()) {
        ce_command(c, 4);
        c->ce_thread.join();
    }
    for (cudaEvent_t e : c->ce_ev)
        if (e) cudaEventDestroy(e);
    if (c->ce_stream) cudaStreamDestroy(c->ce_stream);
    if (c->stream) cudaStreamDestroy(c->stream);
    delete c;
}

int pagoda_init(const pagoda_config* cfg_in, pagoda_ctx** out)
{
    if (!out) return -EINVAL;
    *out = nullptr;
    pagoda_config cfg;
    if (cfg_in) cfg = *cfg_in;
    else pagoda_config_default(&cfg);
    /* 4 MTBs/SM: 512-thread MTBs.  (8 MTBs/SM of 256 threads were tried: the cooperative launch fails with
     * "too many blocks" although the occupancy API reports 8 per SM; each MTB uses all 16 named
     * barriers, the likely per-SM limit.) */
    /* (3 MTBs/SM of 512 threads at 40 registers were measured too: slower on every config, e.g. mix 12.9 -> 7.8 M) */
    if (cfg.mtbs_per_sm != 1 && cfg.mtbs_per_sm != 2 && cfg.mtbs_per_sm != 4) return -EINVAL;
    const uint32_t block_warps = cfg.mtbs_per_sm == 4 ? 16u : 32u;
    if (!pow2(cfg.ring_entries) || !pow2(cfg.comp_entries) || cfg.comp_entries < cfg.ring_entries ||
        cfg.ring_entries < 2 * kSpawnChunk)
        return -EINVAL;
    if (cfg.exec_warps < 1 || cfg.exec_warps > 32) return -EINVAL;
    if (cfg.sched_groups == 0) cfg.sched_groups = 1;
    if (cfg.sched_groups > 2) return -EINVAL;
    if (cfg.max_tasks > 32) return -EINVAL;
    cfg.exec_warps = std::min(cfg.exec_warps, block_warps);
    if (cfg.arena_bytes % PAGODA_GRANULE || cfg.arena_bytes / PAGODA_GRANULE > (uint32_t)kMaxGranules ||
        cfg.arena_bytes < 8u * PAGODA_GRANULE)
        return -EINVAL;
    int ndev = 0;
    if (cudaGetDeviceCount(&ndev) != cudaSuccess || cfg.device < 0 || cfg.device >= ndev) {
        cudaGetLastError();
        return -ENODEV;
    }
    if (cudaSetDevice(cfg.device) != cudaSuccess) return -ENODEV;
    cudaDeviceProp prop;
    if (cudaGetDeviceProperties(&prop, cfg.device) != cudaSuccess) return -ENODEV;
    if (prop.major != 10) return -ENODEV;   /* built for sm_100a only */
    const uint32_t arena_offset = (cfg.flags & PAGODA_RESIDENT_TDES) ? kResidentOffset + kResidentTdesBytes : kControlBytes;
    const size_t smem = arena_offset + cfg.arena_bytes;
    if (smem * (size_t)cfg.mtbs_per_sm + 1024 * (size_t)cfg.mtbs_per_sm > (size_t)prop.sharedMemPerMultiprocessor ||
        smem > (size_t)prop.sharedMemPerBlockOptin)
        return -EINVAL;
    if (cfg.num_sms < 0 || cfg.num_sms > prop.multiProcessorCount) return -EINVAL;

    pagoda_ctx* c = new (std::nothrow) pagoda_ctx;
    if (!c) return -ENOMEM;
    c->cfg = cfg;
    c->device = cfg.device;
    c->sm_count = prop.multiProcessorCount;
    const int nsm = cfg.num_sms ? cfg.num_sms : prop.multiProcessorCount;
    if (nsm * cfg.mtbs_per_sm == 1 && cfg.arena_bytes < 2u * 128u * 64u + 8u * PAGODA_GRANULE) {
        delete c;   /* one MTB lends the top of its arena to its ingest warp's two stages */
        return -EINVAL;
    }
    if (nsm * cfg.mtbs_per_sm > 1 && !(cfg.flags & PAGODA_CE_INGEST) &&
        ingest_stage_entries((uint32_t)smem, nsm * cfg.mtbs_per_sm) < 32u) {
        delete c;   /* the I/O MTB's shared memory holds no ingest stage of 32 entries: use PAGODA_CE_INGEST */
        return -EINVAL;
    }
    c->n_mtb = nsm * cfg.mtbs_per_sm;
    c->R = cfg.ring_entries;
    c->C = cfg.comp_entries;
    const uint32_t arena_g = cfg.arena_bytes / PAGODA_GRANULE;
    c->n_grp = (int)cfg.sched_groups;
    {   /* a task must fit the smallest scheduling group that takes tickets (a task-running MTB's
         * worker warps, split into n_grp equal warp ranges; the arena split the same way) */
        const uint32_t gw = block_warps / (uint32_t)c->n_grp;
        const uint32_t per = std::min<uint32_t>(cfg.exec_warps / (uint32_t)c->n_grp, gw);   /* workers per group */
        uint32_t exec = 0;
        for (int g = 0; g < c->n_grp; g++) exec |= (per >= 32u ? 0xffffffffu : ((1u << per) - 1u)) << (g * gw);
        uint32_t ag = arena_g;
        if (c->n_mtb == 1) {   /* MTB 0 alone: it also hosts the ingest warp and its staging */
            exec &= ~(1u << (block_warps - 1u));
            ag = arena_g - 2u * ingest_stage_entries(cfg.arena_bytes, 1) * 64u / PAGODA_GRANULE;
        }
        int mw = 32;
        for (int g = 0; g < c->n_grp; g++) {
            const uint32_t gm = (gw >= 32u ? 0xffffffffu : ((1u << gw) - 1u)) << (g * gw);
            const int k = __builtin_popcount(exec & gm);
            if (k) mw = std::min(mw, k);   /* a group without workers takes no tickets */
        }
        c->max_task_warps = mw;
        c->max_task_granules = ag / (uint32_t)c->n_grp;
        c->max_bars = c->n_grp == 1 ? PAGODA_BAR_IDS : 7;
    }
    c->warps_prefix.assign(c->C, 0);

    int rc = -ENOMEM;
    if (cudaHostAlloc((void**)&c->hctl, sizeof(HostCtl), cudaHostAllocMapped | cudaHostAllocPortable) != cudaSuccess)
        goto fail;
    memset((void*)c->hctl, 0, sizeof(HostCtl));
    if (cudaHostAlloc((void**)&c->hring, (size_t)c->R * sizeof(TaskEntry), cudaHostAllocMapped | cudaHostAllocPortable) !=
        cudaSuccess)
        goto fail;
    memset(c->hring, 0, (size_t)c->R * sizeof(TaskEntry));
    if (cudaHostAlloc((void**)&c->comp, (size_t)c->C * sizeof(int64_t), cudaHostAllocMapped | cudaHostAllocPortable) !=
        cudaSuccess)
        goto fail;
    for (uint32_t i = 0; i < c->C; i++) c->comp[i] = -1;
    if (cudaMalloc(&c->dring, (size_t)c->R * sizeof(TaskEntry)) != cudaSuccess) goto fail;
    if (cudaMalloc(&c->dseq, (size_t)c->R * sizeof(uint32_t)) != cudaSuccess) goto fail;
    {   /* cell i starts free for position i */
        std::vector<uint32_t> seq(c->R);
        for (uint32_t i = 0; i < c->R; i++) seq[i] = i;
        if (cudaMemcpy(c->dseq, seq.data(), seq.size() * sizeof(uint32_t), cudaMemcpyHostToDevice) != cudaSuccess)
            goto fail;
    }
    if (cudaMalloc(&c->dctl, sizeof(DevCtl)) != cudaSuccess) goto fail;
    if (cudaMemset(c->dctl, 0, sizeof(DevCtl)) != cudaSuccess) goto fail;
    if (cudaMemset(&c->dctl->io_smid, 0xFF, sizeof(uint32_t)) != cudaSuccess) goto fail;
    if (cudaMalloc(&c->dq, (size_t)kDqEntries * sizeof(uint64_t)) != cudaSuccess) goto fail;
    if (cudaMalloc(&c->grp, (size_t)c->C * sizeof(uint32_t)) != cudaSuccess) goto fail;
    if (cudaMemset(c->grp, 0, (size_t)c->C * sizeof(uint32_t)) != cudaSuccess) goto fail;
    if (cudaMemset(c->dq, 0, (size_t)kDqEntries * sizeof(uint64_t)) != cudaSuccess) goto fail;
    if (cfg.flags & PAGODA_TRACE) {
        const size_t cap = cfg.trace_events ? cfg.trace_events : 8192;
        c->cfg.trace_events = (uint32_t)cap;
        /* one ledger per scheduling group (its holder is the allocator's single owner) */
        if (cudaMalloc(&c->trace, (size_t)c->n_mtb * c->n_grp * cap * sizeof(LedgerEvent)) != cudaSuccess) goto fail;
        if (cudaMalloc(&c->trace_count, (size_t)c->n_mtb * c->n_grp * sizeof(uint32_t)) != cudaSuccess) goto fail;
        if (cudaMalloc(&c->exec_trace, (size_t)c->n_mtb * 32 * cap * sizeof(ExecRecord)) != cudaSuccess) goto fail;
        if (cudaMalloc(&c->exec_count, (size_t)c->n_mtb * 32 * sizeof(uint32_t)) != cudaSuccess) goto fail;
        cudaMemset(c->trace_count, 0, (size_t)c->n_mtb * c->n_grp * sizeof(uint32_t));
        cudaMemset(c->exec_count, 0, (size_t)c->n_mtb * 32 * sizeof(uint32_t));
    }
    if (cfg.flags & PAGODA_LIFECYCLE) {
        if (cudaMalloc(&c->life, (size_t)c->C * 8 * sizeof(uint64_t)) != cudaSuccess) goto fail;
        if (cudaMemset(c->life, 0, (size_t)c->C * 8 * sizeof(uint64_t)) != cudaSuccess) goto fail;
    }
    if (cudaStreamCreateWithFlags(&c->stream, cudaStreamNonBlocking) != cudaSuccess) goto fail;
    if (cfg.flags & PAGODA_CE_INGEST) {
        if (!load_stream_memops()) {
            rc = -ENOTSUP;
            goto fail;
        }
        if (cudaStreamCreateWithFlags(&c->ce_stream, cudaStreamNonBlocking) != cudaSuccess) goto fail;
        for (int i = 0; i < kCeInFlight; i++)
            if (cudaEventCreateWithFlags(&c->ce_ev[i], cudaEventDisableTiming) != cudaSuccess) goto fail;
        c->d_tail = (CUdeviceptr)&c->dctl->tail;
        c->d_stop = (CUdeviceptr)&c->dctl->stop;
        c->ce_thread = std::thread(ce_thread_main, c);
    }
    if (cudaEventCreate(&c->ev_start) != cudaSuccess || cudaEventCreate(&c->ev_stop) != cudaSuccess) goto fail;
    /* the set-up copies and memsets above ran on the legacy stream: wait for that stream only.  A
     * device-wide synchronize would also wait for another context's persistent MasterKernel on the
     * same device (pool members sharing a GPU) and never return. */
    if (cudaStreamSynchronize(cudaStreamLegacy) != cudaSuccess) goto fail;
    {
        MkParams& p = c->params;
        memset(&p, 0, sizeof p);
        void* dptr = nullptr;
        cudaHostGetDevicePointer(&dptr, (void*)c->hring, 0);
        p.hring = (const TaskEntry*)dptr;
        cudaHostGetDevicePointer(&dptr, (void*)c->hctl, 0);
        p.hctl = (HostCtl*)dptr;
        cudaHostGetDevicePointer(&dptr, (void*)c->comp, 0);
        p.comp = (int64_t*)dptr;
        p.dring = c->dring;
        p.dseq = c->dseq;
        p.dctl = c->dctl;
        p.ring_mask = c->R - 1;
        p.comp_mask = c->C - 1;
        p.exec_warps = (int)cfg.exec_warps;
        p.arena_granules = (int)arena_g;
        p.arena_offset = arena_offset;
        p.ingest_stage_entries = ingest_stage_entries(c->n_mtb == 1 ? cfg.arena_bytes : (uint32_t)smem, c->n_mtb);
        p.stage_offset = kStageOffset;
        p.io_sm_exclusive = nsm > 1 ? 1u : 0u;   /* one SM: its other MTB must run the tasks */
        p.dq = c->dq;
        p.grp = c->grp;
        p.dq_mask = kDqEntries - 1;
        if (cfg.flags & PAGODA_RESIDENT_TDES) {   /* the key-independent SP table, replicated by each MTB */
            std::vector<uint8_t> tab(PAGODA_TDES_TABLE_BYTES);
            const uint8_t zero_key[24] = {0};
            pagoda_tdes_tables(zero_key, tab.data());
            if (cudaMalloc(&c->resident_src, 2048) != cudaSuccess || cudaMemcpy(c->resident_src, tab.data(), 2048, cudaMemcpyHostToDevice) != cudaSuccess) goto fail;
            p.resident_tdes_src = c->resident_src;
        }
        p.n_mtb = c->n_mtb;
        p.n_grp = (uint32_t)c->n_grp;
        p.n_exit = (uint32_t)(c->n_mtb * c->n_grp);
        p.max_tasks = cfg.max_tasks;
        p.ce_ingest = (cfg.flags & PAGODA_CE_INGEST) ? 1u : 0u;
        if (cfg.flags & PAGODA_TRACE) {
            p.trace_cap = c->cfg.trace_events;
            p.trace = c->trace;
            p.trace_count = c->trace_count;
            p.exec_trace = c->exec_trace;
            p.exec_count = c->exec_count;
        }
        p.life = c->life;
        /* completion forwarders: 4 when MTB 0 has 32 warps; at 4 MTBs/SM (16 warps) 2 with the copy-engine
         * ingest (MTB 0's ingest warps idle: MM 54.5 -> 57.5 M) and 1 with the doorbell ingest (more cost its
         * publishers: MM 45 -> 42 M) */
        p.n_fwd = cfg.mtbs_per_sm == 4 ? ((cfg.flags & PAGODA_CE_INGEST) ? 2u : (uint32_t)PAGODA_FWD_4MTB)
                                       : (uint32_t)kForwarders;
        p.spread_ns = 0;
        if (cfg.flags & PAGODA_SPREAD) {   /* PAGODA_SPREAD_NS (environment) overrides the 6 us default */
            const char* e = getenv("PAGODA_SPREAD_NS");
            p.spread_ns = e ? (uint32_t)strtoul(e, nullptr, 10) : 6000u;
        }
        c->smem = smem;
        {
            std::lock_guard<std::mutex> reg(g_ctx_mtx);
            g_ctxs.push_back(c);
        }
        rc = (cfg.flags & PAGODA_NO_START) ? 0 : start_kernel(c);
        if (rc) goto fail;
    }
    *out = c;
    return 0;
fail:
    cudaGetLastError();
    free_ctx(c);
    return rc;
}

pagoda_task_t pagoda_taskSpawn(pagoda_ctx* c, int threads, int n_tb, int shmem_bytes, int sync_flag, int func_id,
                               const void* args, size_t args_bytes)
{
    if (!c) return -EINVAL;
    if (c->shutting.load(std::memory_order_acquire)) return -ESHUTDOWN;
    if (dev_fault(c)) return -EIO;
    const int32_t shape[5] = {threads, n_tb, shmem_bytes, sync_flag, func_id};
    Split sp;
    if (int rc = shape_check(c, shape, sp)) return rc;
    if (args_bytes > PAGODA_ARGS_MAX || (args_bytes > 0 && !args)) return -EINVAL;
    if (sp.k > 1) {   /* spread over several MTB entries: the batched path writes the group */
        pagoda_task_t id = -1;
        const int64_t rc = spawn_batch(c, 1, [&](int) { return shape; }, args, args_bytes, args_bytes, &id);
        return rc < 0 ? (pagoda_task_t)rc : id;
    }
    const int wtb = sp.wtb;
    const uint32_t gtb = sp.gtb;

    uint64_t id = 0;
    if (int rc = reserve_ids(c, 1, &id)) return rc;
    /* 1. ring slot free: the ingest warp has copied entry id - R */
    if (!ring_room(c, id)) {
        int rc = spin_until(c, [&] { return ring_room(c, id); });
        if (rc) return reserve_failed(c, rc);
    }
    /* 2. completion slot free: task id - C is done */
    if (!comp_room(c, id)) {
        int rc = spin_until(c, [&] { return comp_room(c, id); });
        if (rc) return reserve_failed(c, rc);
    }
    /* 3. the entry */
    write_entry(c, id, 0, shape, sp, args, args_bytes);
    (void)gtb;
    const int64_t w = (int64_t)wtb * n_tb;
    /* 4. in-order commit of the doorbell (x86 stores are ordered; the fence is for the compiler) */
    if (c->published.load(std::memory_order_acquire) != id) {
        int rc = spin_until(c, [&] { return c->published.load(std::memory_order_acquire) == id; });
        if (rc) return reserve_failed(c, rc);
    }
    c->warps_prefix[id & (c->C - 1)] = c->warps_spawned.fetch_add(w, std::memory_order_relaxed) + w;
    std::atomic_thread_fence(std::memory_order_release);
    c->hctl->published = id + 1;
    c->published.store(id + 1, std::memory_order_release);
    return (pagoda_task_t)id;
}

/* Batched spawn: the same entries taskSpawn would write, but ids are reserved
 * a chunk at a time and the doorbell is published once per chunk (the GPU
 * sees the chunk's tasks together, the host does one atomic and one doorbell
 * store per chunk instead of per task).  Every task is validated first. */
} /* extern "C" */

template <class ShapeOf>
static int64_t spawn_batch(pagoda_ctx* c, int n, ShapeOf shape_of, const void* args_base, size_t args_stride,
                           size_t args_bytes, pagoda_task_t* ids_out, bool validated)
{
    if (!c || n < 0) return -EINVAL;
    if (c->shutting.load(std::memory_order_acquire)) return -ESHUTDOWN;
    if (dev_fault(c)) return -EIO;
    if (args_bytes > PAGODA_ARGS_MAX || (args_bytes > 0 && !args_base)) return -EINVAL;
    ShapeMemo memo;
    for (int i = 0; i < n && !validated; i++) {   /* every task valid before any is spawned */
        Split sp;
        if (int rc = memo.check(c, shape_of(i), sp)) return rc;
    }
    const char* a = static_cast<const char*>(args_base);
    for (int base = 0; base < n;) {
        /* a chunk: up to kSpawnChunk tasks, each one or more entries (ids) */
        Split sps[kSpawnChunk];
        int m = 0;
        uint64_t K = 0;
        while (base + m < n && m < kSpawnChunk) {
            memo.check(c, shape_of(base + m), sps[m]);
            if (m > 0 && K + (uint64_t)sps[m].k > (uint64_t)(c->R / 4)) break;
            K += (uint64_t)sps[m].k;
            m++;
        }
        uint64_t id0 = 0;
        if (int rc = reserve_ids(c, K, &id0)) return base ? (int64_t)base : (int64_t)rc;   /* tasks before stay */
        const uint64_t last = id0 + K - 1;
        if (!ring_room(c, last)) {
            int rc = spin_until(c, [&] { return ring_room(c, last); });
            if (rc) return reserve_failed(c, rc);
        }
        if (!comp_room(c, last)) {
            int rc = spin_until(c, [&] { return comp_room(c, last); });
            if (rc) return reserve_failed(c, rc);
        }
        uint64_t id = id0;
        for (int i = 0; i < m; i++) {
            const int32_t* s = shape_of(base + i);
            for (int j = 0; j < sps[i].k; j++)
                write_entry(c, id, j, s, sps[i], args_bytes ? a + (size_t)(base + i) * args_stride : nullptr,
                            args_bytes);
            if (ids_out) ids_out[base + i] = (pagoda_task_t)id;
            id += (uint64_t)sps[i].k;
        }
        if (c->published.load(std::memory_order_acquire) != id0) {
            int rc = spin_until(c, [&] { return c->published.load(std::memory_order_acquire) == id0; });
            if (rc) return reserve_failed(c, rc);
        }
        int64_t ws = c->warps_spawned.load(std::memory_order_relaxed);
        id = id0;
        for (int i = 0; i < m; i++) {   /* a task's warps count at its first id, its other ids add none */
            const int32_t* s = shape_of(base + i);
            ws += (int64_t)sps[i].wtb * s[1];
            for (int j = 0; j < sps[i].k; j++) c->warps_prefix[(id++) & (c->C - 1)] = ws;
        }
        c->warps_spawned.store(ws, std::memory_order_relaxed);
        std::atomic_thread_fence(std::memory_order_release);
        c->hctl->published = last + 1;
        c->published.store(last + 1, std::memory_order_release);
        base += m;
    }
    return n;
}

/* Multi-producer spawn: the workload is cut into blocks of kMtBlock tasks and
 * block b is spawned by producer b mod P (the caller is producer 0), each
 * through spawn_batch.  Entries are written in parallel; publication stays in
 * id order (a chunk is published once every lower id is), so the GPU sees one
 * contiguous TaskTable exactly as with one producer. */
static const int kMtBlock = 4 * kSpawnChunk;

/* Producer t validates its own blocks; every producer waits until all have (all-or-nothing: a
 * rejected workload spawns nothing), then spawns them if none failed.  The validation pass runs
 * on all producers at once: over a large workload it is a scan of the shapes array (~1.3 MB for
 * 65,536 tasks) that would otherwise delay the first spawn of the session. */
static int64_t validate_part(const pagoda_ctx* c, const pagoda_ctx::SpawnJob& j, int t)
{
    for (int b0 = t * kMtBlock; b0 < j.n; b0 += j.P * kMtBlock)
        if (int rc = validate_rows(c, j.shapes + 5 * (size_t)b0, std::min(kMtBlock, j.n - b0))) return rc;
    return 0;
}
static bool validated_all(pagoda_ctx* c, const pagoda_ctx::SpawnJob& j, int t)
{
    const int64_t rc = validate_part(c, j, t);
    if (rc < 0) {
        int64_t z = 0;
        c->job_rc.compare_exchange_strong(z, rc);
    }
    c->job_unvalidated.fetch_sub(1, std::memory_order_acq_rel);
    while (c->job_unvalidated.load(std::memory_order_acquire) > 0) _mm_pause();
    return c->job_rc.load(std::memory_order_acquire) == 0;
}

static int64_t spawn_part(pagoda_ctx* c, const pagoda_ctx::SpawnJob& j, int t)
{
    for (int b0 = t * kMtBlock; b0 < j.n; b0 += j.P * kMtBlock) {
        const int m = std::min(kMtBlock, j.n - b0);
        const int32_t* sh = j.shapes + 5 * (size_t)b0;
        const int64_t rc = spawn_batch(c, m, [&](int i) { return sh + 5 * (size_t)i; },
                                       j.bytes ? j.args + (size_t)b0 * j.stride : nullptr, j.stride, j.bytes,
                                       j.ids ? j.ids + b0 : nullptr, true);
        if (rc < 0) return rc;
        if (rc < m) return -EAGAIN;   /* ring full (non-blocking spawn / stopped): the block is cut short */
    }
    return 0;
}

static void helper_main(pagoda_ctx* c, int t)
{
    uint64_t seen = 0;
    uint64_t idle = 0;
    for (;;) {
        const uint64_t g = c->job_gen.load(std::memory_order_acquire);
        if (g != seen) {
            seen = g;
            idle = 0;
            const pagoda_ctx::SpawnJob j = c->job;
            if (t < j.P) {
                const int64_t rc = validated_all(c, j, t) ? spawn_part(c, j, t) : 0;
                if (rc < 0) {
                    int64_t z = 0;
                    c->job_rc.compare_exchange_strong(z, rc);
                }
                c->job_left.fetch_sub(1, std::memory_order_acq_rel);
            }
            continue;
        }
        if (c->helpers_quit.load(std::memory_order_acquire)) return;
        /* spin while jobs are likely to follow (back-to-back steps), then sleep */
        if (++idle < (1u << 16)) _mm_pause();
        else std::this_thread::sleep_for(std::chrono::microseconds(idle < (1u << 20) ? 2 : 50));
    }
}

extern "C" {

int64_t pagoda_taskSpawnShapesMT(pagoda_ctx* c, int n, const int32_t* shapes, const void* args_base,
                                 size_t args_stride, size_t args_bytes, pagoda_task_t* ids_out, int n_producers)
{
    if (!c || n < 0 || (!shapes && n > 0) || n_producers < 1 || n_producers > PAGODA_MAX_PRODUCERS) return -EINVAL;
    if (args_bytes > PAGODA_ARGS_MAX || (args_bytes > 0 && !args_base)) return -EINVAL;
    const int P = std::min(n_producers, std::max(1, (n + kMtBlock - 1) / kMtBlock));
    if (P == 1) {
        if (int rc = validate_rows(c, shapes, n)) return rc;
        return spawn_batch(c, n, [&](int i) { return shapes + 5 * (size_t)i; }, args_base, args_stride, args_bytes,
                           ids_out, true);
    }
    std::lock_guard<std::mutex> lk(c->mt_mtx);
    while ((int)c->helpers.size() < P - 1) {
        const int t = (int)c->helpers.size() + 1;
        c->helpers.emplace_back(helper_main, c, t);
    }
    c->job = pagoda_ctx::SpawnJob{shapes, static_cast<const char*>(args_base), args_stride, args_bytes, ids_out, n, P};
    c->job_rc.store(0);
    c->job_unvalidated.store(P, std::memory_order_release);
    c->job_left.store(P - 1, std::memory_order_release);
    c->job_gen.fetch_add(1, std::memory_order_acq_rel);
    const int64_t rc0 = validated_all(c, c->job, 0) ? spawn_part(c, c->job, 0) : 0;
    while (c->job_left.load(std::memory_order_acquire) > 0) _mm_pause();
    const int64_t rc = rc0 < 0 ? rc0 : c->job_rc.load();
    return rc < 0 ? rc : n;
}

int64_t pagoda_taskSpawnMany(pagoda_ctx* c, int n, int threads, int n_tb, int shmem_bytes, int sync_flag, int func_id,
                             const void* args_base, size_t args_stride, size_t args_bytes, pagoda_task_t* ids_out)
{
    const int32_t shape[5] = {threads, n_tb, shmem_bytes, sync_flag, func_id};
    return spawn_batch(c, n, [&](int) { return shape; }, args_base, args_stride, args_bytes, ids_out);
}

int64_t pagoda_taskSpawnShapes(pagoda_ctx* c, int n, const int32_t* shapes, const void* args_base, size_t args_stride,
                               size_t args_bytes, pagoda_task_t* ids_out)
{
    if (!shapes && n > 0) return -EINVAL;
    if (!c || n < 0) return -EINVAL;
    if (int rc = validate_rows(c, shapes, n)) return rc;
    return spawn_batch(c, n, [&](int i) { return shapes + 5 * (size_t)i; }, args_base, args_stride, args_bytes,
                       ids_out, true);
}

int pagoda_check(pagoda_ctx* c, pagoda_task_t id)
{
    if (!c) return -EINVAL;
    if (id < 0 || (uint64_t)id >= c->next_id.load(std::memory_order_acquire)) return -EINVAL;
    if (dev_fault(c)) return -EIO;
    if ((uint64_t)id < c->low.load(std::memory_order_acquire)) return 1;
    if (c->comp[(uint64_t)id & (c->C - 1)] >= id) return 1;
    return 0;
}

int pagoda_wait(pagoda_ctx* c, pagoda_task_t id)
{
    if (!c) return -EINVAL;
    if (id < 0 || (uint64_t)id >= c->next_id.load(std::memory_order_acquire)) return -EINVAL;
    if (dev_fault(c)) return -EIO;
    if ((uint64_t)id < c->low.load(std::memory_order_acquire)) return 0;
    volatile int64_t* slot = &c->comp[(uint64_t)id & (c->C - 1)];
    int rc = spin_until(c, [&] { return *slot >= id; });
    std::atomic_thread_fence(std::memory_order_acquire);
    return rc;
}

int pagoda_waitBelow(pagoda_ctx* c, pagoda_task_t end)
{
    if (!c || end < 0) return -EINVAL;
    const uint64_t n = std::min<uint64_t>((uint64_t)end, c->next_id.load(std::memory_order_acquire));
    int rc = spin_until(c, [&] {
        advance_low(c, n);
        return c->low.load(std::memory_order_acquire) >= n;
    });
    std::atomic_thread_fence(std::memory_order_acquire);
    return rc;
}

int pagoda_waitAll(pagoda_ctx* c)
{
    if (!c) return -EINVAL;
    const uint64_t n = c->next_id.load(std::memory_order_acquire);
    int rc = spin_until(c, [&] {
        advance_low(c, n);
        return c->low.load(std::memory_order_acquire) >= n;
    });
    std::atomic_thread_fence(std::memory_order_acquire);
    return rc;
}

int pagoda_stop(pagoda_ctx* c)
{
    if (!c) return -EINVAL;
    std::lock_guard<std::mutex> lk(c->session_mtx);
    if (!c->running.load()) return -EALREADY;
    if (c->faulted.load()) {
        const int r2 = stop_kernel(c);
        return r2 ? r2 : -EIO;
    }
    /* Every task issued before the call is published, then terminate: the MasterKernel drains
     * everything published and exits (the ingest reads terminate before the published count),
     * so the stop does not wait for the host to observe the last completion first. */
    const uint64_t n = c->next_id.load(std::memory_order_acquire);
    int rc = spin_until(c, [&] { return c->published.load(std::memory_order_acquire) >= n; });
    const int r2 = stop_kernel(c);
    if (!rc && !r2) {   /* the session drained: every id below n has its completion record */
        rc = spin_until(c, [&] {
            advance_low(c, n);
            return c->low.load(std::memory_order_acquire) >= n;
        });
        if (rc == -EAGAIN) rc = -EIO;   /* published before terminate, yet not completed */
        std::atomic_thread_fence(std::memory_order_acquire);
    }
    return rc ? rc : r2;
}

int pagoda_start(pagoda_ctx* c)
{
    if (!c) return -EINVAL;
    std::lock_guard<std::mutex> lk(c->session_mtx);
    if (c->shutting.load() || c->faulted.load()) return -EIO;
    if (c->running.load()) return -EBUSY;
    return start_kernel(c);
}

int pagoda_start_drain(pagoda_ctx* c)
{
    if (!c) return -EINVAL;
    std::lock_guard<std::mutex> lk(c->session_mtx);
    if (c->shutting.load() || c->faulted.load()) return -EIO;
    if (c->running.load()) return -EBUSY;
    c->hctl->terminate = 1;   /* the session exits once everything already published is done */
    return start_kernel(c);
}

int pagoda_session_ms(pagoda_ctx* c, float* ms)
{
    if (!c || !ms) return -EINVAL;
    if (c->running.load() || c->sessions == 0) return -EBUSY;
    return cudaEventElapsedTime(ms, c->ev_start, c->ev_stop) == cudaSuccess ? 0 : -EIO;
}

int pagoda_shutdown(pagoda_ctx* c)
{
    if (!c) return -EINVAL;
    int rc = 0;
    {
        std::lock_guard<std::mutex> lk(c->session_mtx);
        if (c->running.load()) {
            if (!c->faulted.load()) rc = pagoda_waitAll(c);
            c->shutting.store(1, std::memory_order_release);
            const int r2 = stop_kernel(c, rc != 0 || c->faulted.load());
            if (c->running.load()) return r2;   /* still resident: freeing live buffers would fault it */
            if (!rc) rc = r2;
        }
        c->shutting.store(1, std::memory_order_release);
    }
    if ((c->hctl->error & kFatalDevErr) && rc == 0) rc = -EIO;
    cudaSetDevice(c->device);
    if (c->ev_start) cudaEventDestroy(c->ev_start);
    if (c->ev_stop) cudaEventDestroy(c->ev_stop);
    free_ctx(c);
    return rc;
}

int pagoda_get_info(pagoda_ctx* c, pagoda_info* o)
{
    if (!c || !o) return -EINVAL;
    memset(o, 0, sizeof *o);
    o->device = c->device;
    o->sm_count = c->sm_count;
    o->n_mtb = c->n_mtb;
    o->sched_groups = c->n_grp;
    o->mtbs_per_sm = c->cfg.mtbs_per_sm;
    o->exec_warps = (int)c->cfg.exec_warps;
    o->arena_bytes = (int)c->cfg.arena_bytes;
    o->regs_per_thread = c->regs;
    o->ring_entries = c->R;
    o->comp_entries = c->C;
    o->spawned = (int64_t)c->next_id.load();
    advance_low(c, c->next_id.load());
    o->completed_low = (int64_t)c->low.load();
    o->device_error = c->hctl->error;
    o->running = cudaStreamQuery(c->stream) == cudaErrorNotReady;
    return 0;
}

int64_t pagoda_trace_read(pagoda_ctx* c, int mtb, void* dst, size_t cap)
{
    if (!c || !c->trace || mtb < 0 || mtb >= c->n_mtb * c->n_grp) return -EINVAL;   /* a group's ledger id */
    uint32_t n = 0;
    if (cudaMemcpy(&n, c->trace_count + mtb, 4, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    const size_t k = std::min<size_t>({(size_t)n, cap, (size_t)c->cfg.trace_events});
    if (k && dst &&
        cudaMemcpy(dst, c->trace + (size_t)mtb * c->cfg.trace_events, k * sizeof(LedgerEvent), cudaMemcpyDeviceToHost) !=
            cudaSuccess)
        return -EIO;
    return n;
}

int64_t pagoda_lifecycle_read(pagoda_ctx* c, uint64_t first, size_t n, uint64_t* dst)
{
    if (!c || (!dst && n) || n > c->C) return -EINVAL;
    if (!c->life) return -ENODATA;
    cudaSetDevice(c->device);
    const uint64_t f = first & (c->C - 1);
    const size_t n1 = std::min<size_t>(n, c->C - f);
    if (cudaMemcpy(dst, c->life + f * 8, n1 * 64, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    if (n1 < n && cudaMemcpy(dst + n1 * 8, c->life, (n - n1) * 64, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    return (int64_t)n;
}

int64_t pagoda_trace_read_exec(pagoda_ctx* c, int mtb, int warp, void* dst, size_t cap)
{
    if (!c || !c->exec_trace || mtb < 0 || mtb >= c->n_mtb || warp < 0 || warp > 31) return -EINVAL;
    uint32_t n = 0;
    const size_t idx = (size_t)mtb * 32 + (size_t)warp;
    if (cudaMemcpy(&n, c->exec_count + idx, 4, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    const size_t k = std::min<size_t>({(size_t)n, cap, (size_t)c->cfg.trace_events});
    if (k && dst &&
        cudaMemcpy(dst, c->exec_trace + idx * c->cfg.trace_events, k * sizeof(ExecRecord), cudaMemcpyDeviceToHost) !=
            cudaSuccess)
        return -EIO;
    return n;
}

/* in-flight warps of a context = warps spawned - warps of the tasks below the
 * low watermark (tasks completed out of order above it still count) */
int64_t pagoda_inflight_warps(pagoda_ctx* c)
{
    if (!c) return -EINVAL;
    const uint64_t n = c->next_id.load(std::memory_order_acquire);
    advance_low(c, n);
    const uint64_t l = c->low.load(std::memory_order_acquire);
    const int64_t spawned = c->warps_spawned.load(std::memory_order_acquire);
    const int64_t done = l ? c->warps_prefix[(l - 1) & (c->C - 1)] : 0;
    return spawned - done;
}

/* a MasterKernel of some context on c's device is running (caller holds g_ctx_mtx) */
static bool device_busy(const pagoda_ctx* c)
{
    for (const pagoda_ctx* o : g_ctxs)
        if (o->device == c->device && o->running.load(std::memory_order_acquire)) return true;
    return false;
}

int pagoda_tdes_register(pagoda_ctx* c, const void* dev_tables)
{
    if (!c) return -EINVAL;
    std::lock_guard<std::mutex> reg(g_ctx_mtx);
    if (device_busy(c)) return -EBUSY;
    cudaSetDevice(c->device);
    uint8_t keys[384] = {0};
    uint64_t ptr = 0;
    if (dev_tables) {
        if (cudaMemcpy(keys, static_cast<const uint8_t*>(dev_tables) + 2048, sizeof keys, cudaMemcpyDeviceToHost) !=
            cudaSuccess) {
            cudaGetLastError();
            return -EINVAL;
        }
        ptr = (uint64_t)(uintptr_t)dev_tables;
    }
    return set_tdes_const_keys(keys, ptr) == cudaSuccess ? 0 : -EIO;
}

int pagoda_dct_register(pagoda_ctx* c, const float* dev_coef)
{
    if (!c) return -EINVAL;
    std::lock_guard<std::mutex> reg(g_ctx_mtx);
    if (device_busy(c)) return -EBUSY;
    cudaSetDevice(c->device);
    float coef[64] = {0};
    uint64_t ptr = 0;
    if (dev_coef) {
        if (cudaMemcpy(coef, dev_coef, sizeof coef, cudaMemcpyDeviceToHost) != cudaSuccess) {
            cudaGetLastError();
            return -EINVAL;
        }
        ptr = (uint64_t)(uintptr_t)dev_coef;
    }
    return set_dct_const_coef(coef, ptr) == cudaSuccess ? 0 : -EIO;
}

int pagoda_read_counters(pagoda_ctx* c, uint64_t* out, int n)
{
    if (!c || !out || n < 0) return -EINVAL;
    const int k = std::min(n, kNumCounters);
    if (cudaMemcpy(out, c->dctl->ctr, (size_t)k * 8, cudaMemcpyDeviceToHost) != cudaSuccess) return -EIO;
    return k;
}

const char* pagoda_version(void) { return "pagoda-b200 0.1 (sm_100a)"; }

} /* extern "C" */
