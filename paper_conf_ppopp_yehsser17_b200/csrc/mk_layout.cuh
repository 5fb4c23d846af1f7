/*
 * mk_layout.cuh — data layout shared by the host runtime (runtime.cu) and the
 * MasterKernel (master_kernel.cu).  DESIGN.md "Data layout" draws it.
 *
 * TaskTable entry (#TBs, #threads/TB, kernel, shmem/TB, sync flag,
 * inputs, ready, sched).  The ready/sched handshake is replaced by
 * doorbell ordering: an entry is visible to the GPU iff its index < the
 * published count, and its completion lives in the completion window.
 */
#ifndef PAGODA_MK_LAYOUT_CUH
#define PAGODA_MK_LAYOUT_CUH
#include <stdint.h>

#include "pagoda.h"
#include "pagoda_device.cuh"

namespace pagoda {

struct __align__(64) TaskEntry {
    uint64_t id;
    uint16_t func_id;
    uint16_t threads_tb;   /* requested threads per TB */
    uint8_t  warps_tb;     /* ceil(threads/32) */
    uint8_t  n_tb;
    uint8_t  gran_tb;      /* min(255, ceil(shmem/512)): informational; the MasterKernel derives granules from shmem_bytes */
    uint8_t  flags;        /* bit0 = sync, bit1 = one entry of a task spread over several MTBs (kEntryGroup) */
    uint32_t shmem_bytes;  /* requested bytes per TB */
    uint32_t reserved;     /* group entries: first TB (bits 0-15) | the task's TB count (bits 16-31) */
    uint8_t  args[PAGODA_ARGS_MAX];
};
static_assert(sizeof(TaskEntry) == 64, "TaskEntry is 64 bytes");
constexpr uint8_t kEntrySync = 1, kEntryGroup = 2;

/* pinned, mapped host memory: written by one side, read by the other over PCIe */
struct HostCtl {
    alignas(64) volatile uint64_t published;  /* host -> GPU doorbell: entries [0, published) written */
    volatile uint32_t terminate;              /* host -> GPU: drain and exit */
    alignas(64) volatile uint64_t consumed;   /* GPU -> host: entries copied to the device ring */
    alignas(64) volatile uint64_t handed;     /* GPU -> host (PAGODA_CE_INGEST): ring positions below this were
                                                 loaded by schedulers and handed back (their cells are free) */
    alignas(64) volatile uint32_t error;      /* GPU -> host: device error word (PAGODA_DEVERR_*) */
    volatile uint32_t ingest_alive;
    alignas(64) volatile uint64_t pad[8];
};

/* runtime counters, summed over the session (index = PAGODA_CTR_* in pagoda.h) */
constexpr int kNumCounters = 24;

/* device memory, L2-resident: the device ring's counters */
struct DevCtl {
    alignas(128) uint64_t tail;    /* entries published into the device ring (ingest warp; a hint) */
    alignas(128) uint64_t head;    /* tickets handed out to schedulers (fetch-add) */
    alignas(128) uint32_t stop;    /* set by ingest after terminate: schedulers drain and exit */
    alignas(128) uint32_t error;   /* device error word (executors atomicOr) */
    alignas(128) uint32_t exited;  /* MTBs that exited */
    alignas(128) unsigned long long ctr[kNumCounters];   /* runtime counters (pagoda_read_counters) */
    alignas(128) uint64_t dq_tail; /* completion queue: records reserved by task posters (fetch-add) */
    alignas(128) uint64_t dq_head; /* completion queue: records forwarded to the host (forwarders; resumes) */
    alignas(128) uint64_t fwd_cur[4]; /* each forwarder's cursor: its records below it are forwarded and cleared */
    alignas(128) uint32_t io_smid; /* the SM of MTB 0 (kIoSmidNone until MTB 0 starts) */
};
constexpr uint32_t kIoSmidNone = 0xFFFFFFFFu;

struct LedgerEvent {   /* 32 B; identical field order to the oracle's checker input */
    uint32_t seq;
    uint16_t mtb;
    uint8_t  kind;     /* 1 ALLOC, 2 FREE_WARPS, 3 FREE_TB */
    uint8_t  bar_id;
    uint64_t task_id;
    uint32_t warp_mask;
    uint16_t tb;
    uint16_t gran_off;
    uint16_t gran_len;
    uint16_t pad;
    uint32_t pad2;     /* low 32 bits of %globaltimer when the scheduler logged it (not checked) */
};
static_assert(sizeof(LedgerEvent) == 32, "LedgerEvent is 32 bytes");

struct ExecRecord {    /* 32 B */
    uint64_t task_id;
    uint16_t tb;
    uint16_t smid;     /* %smid: the SM the MTB runs on */
    uint16_t mtb;
    uint16_t warp;
    uint64_t t_start;
    uint64_t t_end;
};
static_assert(sizeof(ExecRecord) == 32, "ExecRecord is 32 bytes");

struct MkParams {
    const TaskEntry* hring;   /* pinned host ring (mapped) */
    HostCtl*         hctl;    /* pinned host control (mapped) */
    int64_t*         comp;    /* pinned completion window (mapped) */
    TaskEntry*       dring;   /* device ring */
    uint32_t*        dseq;    /* per-cell sequence numbers mod 2^32 (bounded MPMC queue): cell of position t holds
                                 t (free for the producer), t+1 (entry t published), t+R (entry t consumed) */
    DevCtl*          dctl;
    uint32_t ring_mask;
    uint32_t comp_mask;
    int      exec_warps;      /* executor warps per MTB (warps 1..exec_warps) */
    int      arena_granules;
    uint32_t arena_offset;    /* byte offset of the task arena in dynamic shared memory */
    uint32_t ingest_stage_entries;   /* entries per ingest stage (2 stages, multiple of 32) */
    const uint32_t* resident_tdes_src;   /* 2 KiB SP table in device memory, replicated per lane
                                            at kResidentOffset when non-null */
    int      n_mtb;
    uint64_t*        dq;      /* device completion queue (n_mtb > 1): id + 1 per record, 0 = empty */
    uint32_t*        grp;     /* [comp_mask + 1] TBs finished per spread task (group), by id; 0 between uses */
    uint32_t dq_mask;
    uint32_t stage_offset;    /* n_mtb > 1: MTB 0's ingest stages start at this dynamic-smem offset */
    uint32_t io_sm_exclusive; /* the MTB sharing MTB 0's SM runs no tasks (several SMs) */
    uint32_t trace_cap;       /* 0 = tracing off */
    LedgerEvent* trace;       /* [n_mtb][trace_cap] */
    uint32_t*    trace_count; /* [n_mtb] */
    ExecRecord*  exec_trace;  /* [n_mtb][32][trace_cap] */
    uint32_t*    exec_count;  /* [n_mtb][32] */
    uint64_t*    life;        /* PAGODA_LIFECYCLE: [comp_mask + 1][8] stamps (pagoda_lifecycle_read), or null */
    uint32_t     n_fwd;       /* completion forwarders in MTB 0 (1..kForwarders) */
    uint32_t     spread_ns;   /* PAGODA_SPREAD: spread-first claim delay per 4 busy warps (0 = off) */
    uint32_t     n_grp;       /* scheduling groups per MTB (1 or 2: pagoda_config.sched_groups) */
    uint32_t     n_exit;      /* holders that exit in a session: n_mtb * n_grp */
    uint32_t     max_tasks;   /* pagoda_config.max_tasks: cap on the tasks a group holds (0 = none) */
    uint64_t     ce_base;     /* PAGODA_CE_INGEST: the ring position the session starts at (everything below was
                                 loaded and handed back in earlier sessions) */
    uint32_t     ce_ingest;   /* PAGODA_CE_INGEST: the host copies entries and writes DevCtl.tail (no ingest warps,
                                 no per-cell publication words: a ticket t is published once tail > t) */
};
enum { kLifePub = 0, kLifeLoad, kLifePlace, kLifeStart, kLifeEnd, kLifeDone, kLifeQueued, kLifeFwd };

/* MTB 0's I/O roles (n_mtb > 1), by position from its last warp (nw = warps per MTB: 32, or 16
 * at 4 MTBs per SM): the loader (nw-1) feeds the device ring (alone it is the whole ingest when
 * n_mtb == 1), the host poster (nw-2) makes the ingest's host-visible stores, the completion
 * forwarders (nw-4, nw-8, ...) move completion records to the host, and kIngestPublishers publisher warps (nw-3,
 * nw-5, nw-6, ...) publish the loader's stages round-robin, each double-buffered
 * (kIngestStages = 2 x publishers), so their per-batch latencies (cell checks, the bulk store,
 * the release fence) overlap */
__host__ __device__ constexpr int ingest_loader_warp(int nw) { return nw - 1; }
__host__ __device__ constexpr int host_poster_warp(int nw) { return nw - 2; }
#ifndef PAGODA_INGEST_PUBLISHERS
#define PAGODA_INGEST_PUBLISHERS 2
#endif
constexpr uint32_t kIngestPublishers = PAGODA_INGEST_PUBLISHERS;
constexpr uint32_t kIngestStages = 2u * kIngestPublishers;
constexpr uint32_t kIngestFinSlots = 64;   /* >= kIngestStages: per-stage completion records */
static_assert(kIngestPublishers >= 1 && kIngestPublishers <= 4, "publisher warps nw-3, nw-5, nw-6, nw-7");
__host__ __device__ constexpr int ingest_publisher_warp(uint32_t i, int nw) { return i == 0 ? nw - 3 : nw - 4 - (int)i; }
__host__ __device__ constexpr uint32_t ingest_publisher_index(int warp, int nw)   /* kIngestPublishers+ if none */
{
    return warp == nw - 3 ? 0u : (warp >= nw - 7 && warp <= nw - 5) ? (uint32_t)(nw - 4 - warp) : 99u;
}
constexpr uint32_t kDqEntries = 1u << 16;  /* device completion queue */
/* completion forwarders (MTB 0, n_mtb > 1): forwarder f of MkParams::n_fwd (<= kForwarders) owns
 * the queue's chunks of kFwdChunk records whose index is f mod n_fwd (warps nw-4, nw-8, nw-9, nw-10) */
#ifndef PAGODA_FORWARDERS
#define PAGODA_FORWARDERS 4
#endif
constexpr uint32_t kForwarders = PAGODA_FORWARDERS;
constexpr uint32_t kFwdChunk = 256;
static_assert(kForwarders >= 1 && kForwarders <= 4, "forwarder warps nw-4, nw-8, nw-9, nw-10");
__host__ __device__ constexpr int forwarder_warp_i(uint32_t f, int nw) { return f == 0 ? nw - 4 : nw - 7 - (int)f; }
__host__ __device__ constexpr uint32_t forwarder_index(int warp, int nw)   /* kForwarders+ if none */
{
    return warp == nw - 4 ? 0u : (warp >= nw - 10 && warp <= nw - 8) ? (uint32_t)(nw - 7 - warp) : 99u;
}
/* ingest staging: 2 stages of MkParams::ingest_stage_entries entries (64 B each).  One MTB: lent
 * from the top of MTB 0's arena (128 entries).  Several: MTB 0 runs no tasks and gives its whole
 * shared memory after the control block (stage_offset) to them. */
constexpr uint32_t kIngestMaxStageEntries = 1024;
constexpr uint32_t kStageOffset = 7168;   /* > kControlBytes, 1 KiB aligned */
__host__ __device__ inline uint32_t ingest_stage_entries(uint32_t smem_bytes, int n_mtb)
{
    if (n_mtb == 1) return 128;   /* MTB 0 also runs tasks: keep most of its arena */
    uint32_t e = (smem_bytes - kStageOffset) / (kIngestStages * 64u) / 32u * 32u;
    return e > kIngestMaxStageEntries ? kIngestMaxStageEntries : e;
}
constexpr uint32_t kStopAbort = 2;       /* HostCtl.terminate / DevCtl.stop value: abandon work and exit */
constexpr int kMaxGranules = 1024;       /* lane-distributed bitmap: 32 lanes x 32 bits */

/* A scheduling group: a share of an MTB's warps, task slots, TB records, named barriers and arena
 * granules with its own scheduler token (self-scheduling).  An MTB has one group, or two
 * (pagoda_config.sched_groups = 2): two token holders place tasks in parallel in one MTB, e.g.
 * sharing the MTB-resident 3DES tables that a second MTB per SM could not hold. */
constexpr int kMaxSchedGroups = 2;
struct SchedGroup {
    /* holder state parked between token holders */
    uint32_t  fg[32];                /* granule bitmap, word l = granules [32l, 32l+32) (1 = free) */
    uint32_t  free_w, free_task, free_tbs, free_bar;
    uint32_t  ph, pl, pt, est_w, seq;
    uint32_t  token;                 /* 1 while some warp of the group holds its scheduler token */
    /* mailboxes (deferred frees): atomicOr by executors, folded by the holder */
    uint32_t  mb_warps, mb_tbs, mb_tasks;
    uint32_t  comp_pending;          /* task slots finished, completion record not yet posted */
    uint32_t  poster;                /* 1 while some warp posts the group's completion records */
    uint32_t  backlog_est;           /* ring backlog (tail - head) at the holder's last look (fused claims) */
    uint32_t  sctr[8];               /* scheduler counters (holder-only), flushed at exit */
    unsigned long long claim_after;  /* PAGODA_SPREAD_NS: no claim before this %globaltimer value */
    unsigned long long sprof[8];     /* PAGODA_PROFILE: ns per phase (PAGODA_CTR_SCHED_NS_FOLD + i) */
    unsigned long long last_post;    /* %globaltimer of the group's last completion post */
};

/* Per-MTB control block at the start of dynamic shared memory (P:456-458:
 * "the remaining shared memory ... stores scheduling data structures"). */
struct MtbShared {
    uint64_t  exec_bar[32];          /*    0: per-warp dispatch mbarriers (replaces the exec flag) */
    uint64_t  stage_bar[32];         /*  256: per-warp TMA staging mbarriers */
    WarpSlot  wt[32];                /*  512: WarpTable (Table 2) */
    TaskEntry tasks[32];             /* 1536: task slots (entries claimed by this MTB) */
    uint32_t  task_warps_left[32];   /* 3584: doneCtr (Alg. 1 L16, L41) */
    uint32_t  tb_warps_left[32];     /* 3712: per-TB counter (lastWarpInBlock, Alg. 1 L35) */
    uint16_t  tb_goff[32];           /* 3840 */
    uint16_t  tb_glen[32];           /* 3904 */
    uint8_t   tb_bar[32];            /* 3968 */
    uint8_t   pend[32];              /* 4000: FIFOs of claimed, not yet placed task slots (group g: its slice) */
    uint64_t  tb_task[32];           /* 4032: task id of each TB record (ledger) */
    uint16_t  tb_idx[32];            /* 4288: TB index j of each TB record (ledger) */
    uint64_t  pend_ticket[32];       /* 4352: claimed ring positions, FIFO (pend[] holds their slots once loaded) */
    uint32_t  stage_ph[32];          /* 4608: parity of each warp's staging mbarrier (TaskEnv::stage) */
    uint32_t* dev_error;             /* 4736: &DevCtl.error, for the paper-named free syncBlock() (kDevErrorPtrOffset) */
    uint32_t  ingest_done;           /* MTB 0: the ingest warps have exited */
    uint32_t  no_tickets;            /* this MTB runs no tasks (MTB 0 and the MTB sharing its SM) */
    uint64_t  ingest_copied;         /* MTB 0: entries published into the device ring, a prefix (host poster) */
    /* MTB 0 ingest, the rest of its control block */
    uint64_t  ingest_bar[kIngestStages];    /* stage s loaded (TMA complete_tx; n = ~0 without bytes: end) */
    uint64_t  ingest_empty[kIngestStages];  /* stage s free again (publisher -> loader) */
    uint64_t  ing_start[kIngestStages];     /* first ring position of the batch in stage s */
    uint32_t  ing_n[kIngestStages];         /* entries in stage s (~0: end of stream) */
    uint32_t  ing_hdr[kIngestStages];       /* k + 1 once stage k's start / n are written (before its load lands) */
    uint64_t  ing_fin_end[kIngestFinSlots]; /* stage k published: its end position ... */
    uint32_t  ing_fin[kIngestFinSlots];     /* ... and k + 1, in slot k mod kIngestFinSlots */
    uint32_t  ing_prefix_k;                 /* stages [0, k) all published (ingest_copied is their end) */
    uint32_t  ing_lock;                     /* serialises prefix advances */
    uint32_t  ing_pubs_done;                /* publishers that saw their end marker */
    uint32_t  fwd_done;              /* MTB 0: forwarders that exited */
    unsigned long long dq_safe;      /* completion-queue positions below this are known free (posters' cache) */
    SchedGroup grp[kMaxSchedGroups]; /* the MTB's scheduling groups (one unless PAGODA_config.sched_groups = 2) */
};
static_assert(offsetof(MtbShared, wt) == kWarpTableOffset, "WarpTable offset");
static_assert(offsetof(MtbShared, stage_bar) == kStageBarOffset, "staging mbarriers offset");
static_assert(offsetof(MtbShared, stage_ph) == kStagePhaseOffset, "staging parities offset");
static_assert(offsetof(MtbShared, dev_error) == kDevErrorPtrOffset, "device error pointer offset");
static_assert(kDevErrSyncWithoutFlag == PAGODA_DEVERR_SYNC_WITHOUT_FLAG, "error code");
static_assert(sizeof(MtbShared) <= kControlBytes && kControlBytes <= kResidentOffset, "control block fits");

} // namespace pagoda
#endif
