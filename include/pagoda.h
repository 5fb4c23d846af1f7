/*
 * pagoda.h — C ABI of the B200-native Pagoda runtime (host side).
 *
 * Pagoda (Yeh, Sabne, Sakdhnagool, Eigenmann, Rogers; PPoPP'17; cited P:<line> of
 * /root/reference/PAPER.md) virtualises GPU SMs for narrow tasks (< 500 threads,
 * P:18-20): a persistent MasterKernel pulls tasks that CPU
 * threads spawn into a TaskTable, allocates executor warps, shared
 * memory and named barriers to them at warp granularity (Alg. 1/2 P:738-880,
 * §5), runs their bodies and signals completion.
 *
 * Calls follow Table 1: taskSpawn / wait / check / waitAll on the
 * host.  The bare paper names would collide with POSIX wait(2), so the C ABI
 * prefixes them with `pagoda_`.
 *
 * Conventions for every function below
 *   - thread-safe: any number of host threads may spawn / wait concurrently;
 *   - errors are negative errno values, never exceptions; 0 (or a valid id) on success;
 *   - pointers named `args` are HOST pointers, copied before the call returns;
 *     device pointers carried INSIDE args are caller-owned and must stay valid
 *     until wait/check reports the task done;
 *   - the context owns every pinned-host and device buffer it allocated.
 */
#ifndef PAGODA_H
#define PAGODA_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

typedef struct pagoda_ctx pagoda_ctx;   /* opaque: rings, MasterKernel stream, counters */
typedef int64_t pagoda_task_t;          /* >= 0: task id; < 0: -errno */

/* ---- limits fixed by the design ---------------- */
#define PAGODA_ARGS_MAX      40   /* bytes of inline task arguments per TaskTable entry */
#define PAGODA_GRANULE       512  /* shared-memory allocation granule */
#define PAGODA_MAX_EXEC_WARPS 32  /* worker warps per MTB: every warp executes; the paper's dedicated
                                     scheduler warp is a token passed between them */
#define PAGODA_BAR_IDS       15   /* named barriers 1..15 per MTB; 0 is the MTB's own */

/* config flags */
#define PAGODA_TRACE         0x1u /* record the per-MTB scheduler ledger (tests; slows scheduling) */
#define PAGODA_NO_START      0x2u /* pagoda_init allocates but does not launch; call pagoda_start(_drain) */
#define PAGODA_RESIDENT_TDES 0x4u /* keep 64 KiB of lane-replicated 3DES S-box tables resident in every MTB
                                     (conflict-free lookups; the arena starts after them) */
#define PAGODA_SPREAD        0x10u /* spread-first claims: while the ring backlog is small, an MTB running
                                      tasks claims the next one later the more warps it has busy (6 us per
                                      4 warps), so few, uneven tasks (config 1) go to the idlest MTBs */
#define PAGODA_LIFECYCLE     0x8u /* stamp every task's life cycle on the GPU clock (profiling; 64 B per
                                     completion slot): see pagoda_lifecycle_read */
#define PAGODA_CE_INGEST     0x40u /* copy-engine ingest: a host thread of the context copies newly published
                                     TaskTable entries into the device ring with cudaMemcpyAsync and
                                     publishes the device ring's tail with a stream memory operation
                                     (cuStreamWriteValue64, ordered after the copy), instead of MTB 0's
                                     warps pulling entries over PCIe; MTB 0 keeps a scanner warp that
                                     reports which ring cells the schedulers have handed back */
#define PAGODA_NONBLOCKING_SPAWN 0x20u /* taskSpawn returns -EAGAIN instead of waiting when the TaskTable
                                     ring slot or completion slot a new task needs is still taken
                                     (the paper's CPU waits for a free entry) */

typedef struct {
    int      device;        /* CUDA device ordinal (default 0) */
    int      mtbs_per_sm;   /* MasterKernel thread blocks (MTBs) per SM: 1 or 2 (1024 threads each; default 2,
                               P:453-455) or 4 (512 threads each: twice the schedulers per SM; arena <= 48 KiB) */
    int      num_sms;       /* SMs to occupy, 0 = all (148 on B200) */
    uint32_t ring_entries;  /* TaskTable ring entries, host and device, power of 2 (default 65536) */
    uint32_t comp_entries;  /* completion window, power of 2 >= ring_entries (default 1<<20) */
    uint32_t arena_bytes;   /* shared-memory arena per MTB, multiple of 512 (default 96 KiB at 2 MTB/SM); the
                               rest of the SM's 228 KiB is L1 (the executors' register spills live there).
                               Without PAGODA_CE_INGEST, MTB 0's shared memory must hold 4 ingest stages
                               of >= 32 entries (-EINVAL otherwise) */
    uint32_t exec_warps;    /* worker warps per MTB, 1..32, capped at the MTB's warps (32 at 1-2 MTBs/SM,
                               16 at 4 MTBs/SM; default 32 = all; fewer = debug config).  One thread
                               block may use at most this many warps (pagoda_info.exec_warps); a
                               single-MTB context keeps one warp for its ingest */
    uint32_t flags;         /* PAGODA_TRACE */
    uint32_t trace_events;  /* ledger capacity per MTB when PAGODA_TRACE (default 8192) */
    double   watchdog_s;    /* wait/waitAll/shutdown give up with -ETIMEDOUT after this many
                               seconds without progress (default 60; <= 0 disables) */
    uint32_t sched_groups;  /* scheduling groups per MTB: 1 (default) or 2.  With 2, an MTB's warps,
                               task slots, TB records, arena and named barriers (1..7 / 8..15) are split
                               in halves (exec_warps counts both: exec_warps / 2 workers per half),
                               each with its own scheduler token, so two holders place
                               tasks in parallel (e.g. sharing the MTB-resident 3DES tables); a thread
                               block must then fit half an MTB and a task has at most 7 syncing TBs
                               per entry.  The ledger (PAGODA_TRACE) is kept per group: ids
                               mtb * sched_groups + g in pagoda_trace_read / executor records. */
    uint32_t max_tasks;     /* tasks one scheduling group holds at once (claimed, loaded, running or
                               posting), 0..32; 0 (default) = as many as its free warps fit plus one
                               of lookahead.  A small cap leaves the rest in the shared ring for
                               whichever MTB frees first: uneven task costs (config 1) then spread
                               over MTBs by completion instead of by claim order */
} pagoda_config;

/* Fill *cfg with the defaults above. */
void pagoda_config_default(pagoda_config* cfg);

/* Start Pagoda on cfg->device: allocate the pinned TaskTable ring, doorbell and
 * completion window, the device ring, and launch the persistent MasterKernel
 * (cooperative launch: all MTBs co-resident).  cfg NULL = defaults.
 * While the MasterKernel runs it holds every warp of the SMs it occupies, so
 * other kernels on that device wait until pagoda_shutdown (copies still run).
 * Returns 0 and *out, or -ENODEV (no such device / not sm_100), -ENOMEM, -EINVAL
 * (bad config), -EIO (launch failed). */
int pagoda_init(const pagoda_config* cfg, pagoda_ctx** out);

/* waitAll, then stop the MasterKernel, free everything and *out is invalid.
 * Freeing device memory synchronizes the whole device, so another context's
 * MasterKernel still running on the same GPU must be stopped first (the pool
 * does this for its members).  Returns 0, -EIO (device fault seen),
 * -ETIMEDOUT (watchdog; resources leaked). */
int pagoda_shutdown(pagoda_ctx* ctx);

/* taskSpawn (Table 1, §3): spawn one task of n_threadblocks
 * thread blocks of `threads` threads (rounded up to whole warps), each block
 * with `shmem_bytes` of shared memory (getSMPtr) and, if sync_flag, a named
 * barrier (syncBlock).  func_id selects a compiled-in task body
 * (pagoda_tasks.h); args/args_bytes (<= 40) are copied into the entry.
 * Non-blocking: returns once the entry is published (it blocks, with back-off,
 * only while the TaskTable ring or completion window is full, as the paper's
 * CPU does when no entry is free; with PAGODA_NONBLOCKING_SPAWN it
 * returns -EAGAIN instead).  Ids never skip a number because of an error: a
 * spawn that cannot get its slots without waiting in vain reserves no id.
 * A task whose thread blocks all fit one MTB (warps, shared memory, 15
 * barrier IDs) runs inside one MTB.  A larger task (e.g. the
 * "64K threads" of Fig. 8) is spread TB by TB over k MTB-sized
 * TaskTable entries; it consumes k ids (the returned one is the first; ids
 * stay strictly increasing but skip k - 1) and completes when its last TB does.
 * Returns the task id (>= 0, strictly increasing per context) or
 *   -EINVAL  threads < 1 or > 1024, n_threadblocks < 1 or (spread) > 65535,
 *            ceil(threads/32) > exec_warps (the worker warps of one MTB: 32 by
 *            default, 16 at 4 MTBs per SM, 31 in a single-MTB context; see
 *            pagoda_info.exec_warps), round_up(shmem, 512) > arena (one TB
 *            must fit an MTB), k > ring_entries / 4, unknown func_id,
 *            args_bytes > 40 or args NULL with args_bytes > 0;
 *   -EAGAIN  the ring / completion slot is taken and the spawn may not wait:
 *            PAGODA_NONBLOCKING_SPAWN, or the session is stopped (nothing
 *            drains the ring until pagoda_start); nothing was spawned;
 *   -ETIMEDOUT  the watchdog expired while waiting for a slot (the context is
 *            then faulted: later calls return -EIO);
 *   -ESHUTDOWN after pagoda_shutdown began;  -EIO after a device fault
 *            (PAGODA_DEVERR_SYNC_WITHOUT_FLAG / _BAD_FUNC) or a failed spawn. */
pagoda_task_t pagoda_taskSpawn(pagoda_ctx* ctx, int threads, int n_threadblocks, int shmem_bytes,
                               int sync_flag, int func_id, const void* args, size_t args_bytes);

/* wait (Table 1): block until task `id` is done.  After it returns 0
 * the task's device writes are visible to later host copies and to every task
 * spawned afterwards.  Returns 0, -EINVAL (id never issued), -EIO (a device
 * fault was seen: every call from then on returns it), -ETIMEDOUT. */
int pagoda_wait(pagoda_ctx* ctx, pagoda_task_t id);

/* check (Table 1): non-blocking; 1 if done, 0 if pending, -EINVAL
 * (id never issued), -EIO (device fault seen). */
int pagoda_check(pagoda_ctx* ctx, pagoda_task_t id);

/* waitAll (Table 1): block until every task whose id was issued before
 * the call is done.  Returns 0, -EIO, -ETIMEDOUT. */
int pagoda_waitAll(pagoda_ctx* ctx);

/* Block until every task with id < end is done (ids issued later are not
 * waited for).  For callers that pipeline copies per spawn batch.  Returns 0,
 * -EINVAL, -EIO, -ETIMEDOUT, -EAGAIN (session stopped). */
int pagoda_waitBelow(pagoda_ctx* ctx, pagoda_task_t end);

/* Convenience for C and Python callers: spawn n tasks of one shape, task i's
 * args at args_base + i*args_stride (args_bytes each); each is a separate
 * pagoda_taskSpawn.  ids_out (nullable) receives the ids.  Returns the number
 * spawned (n) or the first error (tasks before it stay spawned). */
int64_t pagoda_taskSpawnMany(pagoda_ctx* ctx, int n, int threads, int n_threadblocks, int shmem_bytes,
                             int sync_flag, int func_id, const void* args_base, size_t args_stride,
                             size_t args_bytes, pagoda_task_t* ids_out);

/* Same with a per-task shape: shapes[i] = {threads, n_threadblocks, shmem_bytes,
 * sync_flag, func_id} (5 int32 per task).  Both batched forms return n, or,
 * when the ring fills and the call may not wait (PAGODA_NONBLOCKING_SPAWN or
 * a stopped session), the number of leading tasks spawned (0 < count < n; with
 * none spawned -EAGAIN), or the first error. */
int64_t pagoda_taskSpawnShapes(pagoda_ctx* ctx, int n, const int32_t* shapes, const void* args_base,
                               size_t args_stride, size_t args_bytes, pagoda_task_t* ids_out);

/* The same from n_producers host threads (Fig. 1a: several CPU
 * threads spawn into one TaskTable): the calling thread and n_producers - 1
 * helper threads the context starts on first use (kept until shutdown) each
 * spawn every n_producers-th block of 256 consecutive tasks.  Every task is
 * validated before any is spawned (-EINVAL spawns nothing).  ids_out[i] is task
 * i's id; ids are not in workload order across blocks.  One multi-producer call
 * runs at a time per context (others wait); plain taskSpawn calls may run
 * concurrently.  1 <= n_producers <= PAGODA_MAX_PRODUCERS.  Returns n or the
 * first error (tasks of other blocks may have been spawned by then). */
#define PAGODA_MAX_PRODUCERS 8
int64_t pagoda_taskSpawnShapesMT(pagoda_ctx* ctx, int n, const int32_t* shapes, const void* args_base,
                                 size_t args_stride, size_t args_bytes, pagoda_task_t* ids_out, int n_producers);

/* ---- MasterKernel sessions ------------------------------------------------
 * pagoda_init starts a session.  pagoda_stop waits for every issued task,
 * asks the MasterKernel to drain and exit, and waits for it (the ring, the
 * completion window and the ids carry over); pagoda_start launches a new
 * session.  While stopped, other kernels can use the GPU; spawns are accepted
 * and run at the next start; wait/waitAll on unfinished tasks return -EAGAIN.
 * Returns 0, -EALREADY (stop: not running), -EBUSY (start: running), -EIO,
 * -ETIMEDOUT. */
int pagoda_stop(pagoda_ctx* ctx);
int pagoda_start(pagoda_ctx* ctx);
/* Start a self-terminating session: it runs every task already spawned (while
 * stopped; at most ring_entries of them) and exits without a host signal.
 * For tools that serialise kernel launches (Nsight Compute).  Follow with
 * pagoda_stop to collect it. */
int pagoda_start_drain(pagoda_ctx* ctx);
/* Device time of the last finished session: CUDA events recorded on the
 * MasterKernel's stream just before its launch and just after it (so the
 * second completes when the kernel exits).  -EBUSY while a session runs. */
int pagoda_session_ms(pagoda_ctx* ctx, float* ms);

/* ---- measurement helpers (CLOCK_MONOTONIC ns) -------------------------------
 * Spawn n tasks as pagoda_taskSpawnShapes does, recording spawn_ns[i] just
 * before task i's spawn call, while a poller thread records done_ns[i] when
 * check() first reports it done.  Returns n or the first error. */
int64_t pagoda_run_timed(pagoda_ctx* ctx, int n, const int32_t* shapes, const void* args_base,
                         size_t args_stride, size_t args_bytes, int64_t* spawn_ns, int64_t* done_ns);
/* Open loop (SURVEY §8(d) C4 latency variant): task i is spawned at t0 + arrival_ns[i] (t0 = the
 * call; arrival_ns non-decreasing, e.g. Poisson arrivals at a fraction of the measured capacity),
 * whether or not earlier tasks completed; arrive_ns[i] = t0 + arrival_ns[i] (the scheduled arrival,
 * CLOCK_MONOTONIC) and done_ns[i] as in pagoda_run_timed, so done - arrive includes any wait of
 * the spawning thread.  Returns n, -EINVAL (decreasing arrivals) or the first error. */
int64_t pagoda_run_open_loop(pagoda_ctx* ctx, int n, const int32_t* shapes, const void* args_base,
                             size_t args_stride, size_t args_bytes, const int64_t* arrival_ns, int64_t* arrive_ns,
                             int64_t* done_ns);
/* Closed loop, one task in flight: lat_ns[i] = spawn -> wait() return of task i. */
int pagoda_latency_loop(pagoda_ctx* ctx, int n, int threads, int n_threadblocks, int shmem_bytes,
                        int sync_flag, int func_id, const void* args, size_t args_bytes, int64_t* lat_ns);

/* PCIe round-trip floor: one GPU warp echoes a pinned-host
 * counter n times (host writes i, the GPU polls with ld.acquire.sys and writes
 * back i, the host polls); rtt_ns[i] = host write -> echo seen.  Must run
 * while no MasterKernel holds the device.  Returns 0, -EINVAL, -ENODEV,
 * -ENOMEM, -EIO, -ETIMEDOUT. */
int pagoda_pingpong(int device, int n, int64_t* rtt_ns);

/* Roofline denominators the paper's hardware never had to name ("the LDS and
 * INT32 peaks are not published: microbenchmark them on the box").  which = 0: shared-memory
 * lookups of the 3DES pattern (lane-replicated table, one bank per lane); which = 1: INT32
 * lop3.b32.  Two 1024-thread blocks per SM, 8 independent chains per thread; each block times
 * itself in SM cycles.  *per_sm_clk = lanes (ops) per SM per clock; *ops_per_s (nullable) =
 * whole-kernel ops/s by CUDA events at the clock it ran at.  Run while no MasterKernel holds
 * the device.  Returns 0, -EINVAL, -ENODEV, -ENOMEM, -EIO. */
int pagoda_measure_pipe_peak(int device, int which, double* per_sm_clk, double* ops_per_s);

/* Runtime counters accumulated on the device since the context was created
 * (read while stopped or running; ns are %globaltimer nanoseconds). */
enum {
    PAGODA_CTR_INGEST_BATCHES = 0, PAGODA_CTR_INGEST_ENTRIES, PAGODA_CTR_INGEST_NS_DOORBELL,
    PAGODA_CTR_INGEST_NS_COPY, PAGODA_CTR_INGEST_NS_PUBLISH, PAGODA_CTR_INGEST_RING_FULL,
    PAGODA_CTR_SCHED_ROUNDS, PAGODA_CTR_SCHED_PROGRESS, PAGODA_CTR_TICKETS, PAGODA_CTR_CLAIM_EMPTY,
    PAGODA_CTR_LOAD_NOT_READY, PAGODA_CTR_PLACED, PAGODA_CTR_PLACE_NOFIT, PAGODA_CTR_HANDOFFS,
    PAGODA_CTR_INGEST_NS_FENCE,   /* ns of the ingest publish phase spent in its fences */
    PAGODA_CTR_INGEST_NS_STORE,   /* ns spent in the bulk store into the device ring */
    /* profiling builds only (-DPAGODA_PROFILE=1), else 0: scheduler-holder and executor time split */
    PAGODA_CTR_SCHED_NS_FOLD, PAGODA_CTR_SCHED_NS_LOAD, PAGODA_CTR_SCHED_NS_PLACE, PAGODA_CTR_SCHED_NS_CLAIM,
    PAGODA_CTR_SCHED_NS_SLEEP, PAGODA_CTR_EXEC_NS_BODY, PAGODA_CTR_EXEC_NS_FENCE, PAGODA_CTR_EXEC_NS_POST,
    PAGODA_CTR_COUNT = 24
};
/* Copy min(n, PAGODA_CTR_COUNT) counters into out[]; returns the number copied or < 0. */
int pagoda_read_counters(pagoda_ctx* ctx, uint64_t* out, int n);

/* Runtime facts and counters. */
typedef struct {
    int      device, sm_count, n_mtb, mtbs_per_sm, exec_warps, arena_bytes, regs_per_thread;
    uint32_t ring_entries, comp_entries;
    int64_t  spawned;       /* ids issued */
    int64_t  completed_low; /* every id below this is known done */
    uint32_t device_error;  /* 0 or a PAGODA_DEVERR_* code */
    int      running;       /* MasterKernel still resident */
    int      sched_groups;  /* scheduling groups per MTB (pagoda_config.sched_groups) */
} pagoda_info;
int pagoda_get_info(pagoda_ctx* ctx, pagoda_info* out);

/* Device errors (SURVEY §8(b) "Device errors"): the MasterKernel ORs a code into the device
 * error word, which reaches the host within microseconds; from then on every host call on
 * the context (spawn, wait, check, waitAll, stop, shutdown) returns -EIO.  LAYOUT is a notice
 * only (the tasks still run correctly). */
#define PAGODA_DEVERR_SYNC_WITHOUT_FLAG 1u  /* syncBlock() in a multi-warp TB spawned with sync=0 (P:976-983:
                                               only sync tasks get a barrier ID) */
#define PAGODA_DEVERR_BAD_FUNC          2u  /* entry with unknown func_id reached an executor */
#define PAGODA_DEVERR_LAYOUT            4u  /* resident tables did not fit the shared-memory layout (fell back) */

/* Ledger (PAGODA_TRACE): copy up to cap 32-byte events of MTB `mtb` into dst
 * (host memory), after pagoda_shutdown's drain or while idle.  Layout: see
 * DESIGN.md "Trace ledger".  Returns the number of events recorded (may be > cap
 * if the buffer overflowed: then only cap were kept) or -EINVAL. */
int64_t pagoda_trace_read(pagoda_ctx* ctx, int mtb, void* dst, size_t cap);

/* Executor intervals (PAGODA_TRACE): per executor warp a list of
 * {u64 task_id; u16 tb; u16 smid; u16 mtb; u16 warp; u64 t_start_ns; u64 t_end_ns} (32 B).
 * Copies up to cap records of (mtb, warp) into dst; returns the count. */
int64_t pagoda_trace_read_exec(pagoda_ctx* ctx, int mtb, int warp, void* dst, size_t cap);

/* Task life cycle (PAGODA_LIFECYCLE): for task ids [first, first + n) copy 8 u64
 * %globaltimer stamps each (ns; 0 = not seen) into dst (host memory), in order:
 * [0] published into the device ring (ingest), [1] loaded into an MTB's task
 * slot (claim + load done), [2] placed (warps/granules/barrier assigned,
 * executors released), [3] first warp starts the body, [4] last warp ends the
 * body, [5] last warp's completion fence done, [6] completion record queued
 * (device queue, or the host window with one MTB), [7] record forwarded to
 * the host window.  Slots are indexed id mod comp_entries and zeroed at each
 * pagoda_start.  Returns n, -EINVAL or -ENODATA (flag not set). */
int64_t pagoda_lifecycle_read(pagoda_ctx* ctx, uint64_t first, size_t n, uint64_t* dst);

/* Host-side preparation of the 3DES task's device tables:
 * writes PAGODA_TDES_TABLE_BYTES bytes to dst (HOST memory) for the EDE3 key
 * K1|K2|K3 (24 bytes, FIPS 46-3 byte order).  Copy them to device memory and
 * pass the device pointer in pagoda_tdes_args.tables.  Returns 0. */
#define PAGODA_TDES_TABLE_BYTES (2048 + 384 + 16384 + 16384)
int pagoda_tdes_tables(const uint8_t key24[24], void* dst);

/* Register a 3DES key schedule as resident task-class data (with
 * PAGODA_RESIDENT_TDES): 3DES tasks whose `tables` pointer equals dev_tables
 * (device memory written by pagoda_tdes_tables) take their 48 round keys from
 * the MasterKernel's constant bank instead of staging them through shared
 * memory.  One schedule per device and process (the MasterKernel's constant
 * bank is shared by every context on the device); NULL unregisters.  Call while
 * NO context on the device is running (NO_START or after pagoda_stop):
 * -EBUSY otherwise.  Returns 0, -EINVAL (unreadable pointer), -EBUSY, -EIO. */
int pagoda_tdes_register(pagoda_ctx* ctx, const void* dev_tables);

/* Register a DCT coefficient matrix (pagoda_dct_args.coef: 64 fp32 C[u][x], device memory) as
 * resident task-class data: DCT tasks whose coef pointer equals dev_coef read the second
 * pass's coefficients from the MasterKernel's constant bank (same values, same arithmetic:
 * outputs are bit-identical).  The matrix is copied at registration; later writes to dev_coef
 * are not seen.  One matrix per device and process; NULL unregisters.  Call while no context on
 * the device is running: -EBUSY otherwise.  Returns 0, -EINVAL (unreadable pointer), -EBUSY, -EIO.
 * Table 5 / DESIGN.md "DCT". */
int pagoda_dct_register(pagoda_ctx* ctx, const float* dev_coef);

/* Naive baseline (the paper's CUDA-HyperQ): launch
 * each task as its own kernel <<<n_tb, threads, shmem>>> of the same body on
 * streams[i % n_streams] (n_streams <= 32), from the calling thread, then
 * synchronise.  shapes/args as in pagoda_taskSpawnShapes (args are the same
 * device-pointer blocks).  Returns 0 or -EIO.  If elapsed_ns is non-NULL it
 * receives first-launch -> all-done host time. */
int pagoda_naive_run(int device, int n, const int32_t* shapes, const void* args_base, size_t args_stride,
                     size_t args_bytes, int n_streams, int64_t* elapsed_ns);

/* Static-fusion baseline (NEXT-2; "static task fusion combines
 * multiple tasks into a monolithic large task"): ONE kernel launch of n thread
 * blocks of threads_per_task threads (multiple of 32, the paper uses 256);
 * block i runs task i's body with its shared-memory request (the launch
 * reserves the largest).  Every task must have n_threadblocks == 1.  The task
 * table (func id, shmem, args) is copied to the device inside the timed
 * region.  elapsed_ns (nullable): host time from that copy to completion;
 * kernel_ms (nullable): CUDA-event time of the kernel alone.
 * Returns 0, -EINVAL, -ENOMEM, -EIO. */
int pagoda_fused_run(int device, int n, const int32_t* shapes, const void* args_base, size_t args_stride,
                     size_t args_bytes, int threads_per_task, int64_t* elapsed_ns, float* kernel_ms);

/* ---- multi-GPU pool: one context (MasterKernel) per GPU, tasks least-loaded-first.
 * Tasks are independent: no collective, host-side only.  Each member has its own
 * spawner thread, bound to the CPUs of its GPU's NUMA node; that thread creates the member's
 * context, so the pinned rings are allocated on that node. */
typedef struct pagoda_pool pagoda_pool;
/* One member per entry of devices[0..n_dev) with cfg (device field ignored; several entries may
 * name the same device, each then running a MasterKernel of cfg->num_sms SMs, e.g. 2 x 74 on
 * one B200).  cfg may carry PAGODA_NO_START (start members with pagoda_start(pagoda_pool_ctx)). */
int pagoda_pool_init(int n_dev, const int* devices, const pagoda_config* cfg, pagoda_pool** out);
/* Index of the device with the fewest in-flight warps (spawned, not yet seen
 * completed); ties go to the lowest index.  warps_hint is added to the chosen
 * device's in-flight count (the caller then spawns there). */
int pagoda_pool_pick(pagoda_pool* pool, int warps_hint);
pagoda_ctx* pagoda_pool_ctx(pagoda_pool* pool, int index);
int pagoda_pool_size(pagoda_pool* pool);
/* Spawn on the least-loaded context; *index_out (nullable) gets the chosen index.
 * args_per_dev[i] (args_bytes each) are the args to use if device i is chosen. */
pagoda_task_t pagoda_pool_spawn(pagoda_pool* pool, int threads, int n_threadblocks, int shmem_bytes,
                                int sync_flag, int func_id, const void* const* args_per_dev,
                                size_t args_bytes, int* index_out);
/* Batched form: the n tasks (shapes as in pagoda_taskSpawnShapes) are cut into
 * runs of `chunk` consecutive tasks; every member's spawner thread claims the
 * next run only while its GPU is among the least loaded (in-flight warps within
 * two runs' warps of the smallest member's: pagoda_pool_may_claim), and spawns
 * it on its own context; so runs go least-loaded-first and the members' rings
 * are written in parallel.  args_base_per_dev[i] + k * args_stride are task k's
 * args if it lands on member i (device pointers of that device).  ids_out /
 * dev_out (nullable) receive each task's id and member index.  Returns n once
 * every task is spawned, or the first error. */
int64_t pagoda_pool_spawn_shapes(pagoda_pool* pool, int n, const int32_t* shapes, const void* const* args_base_per_dev,
                                 size_t args_stride, size_t args_bytes, int chunk, pagoda_task_t* ids_out,
                                 int32_t* dev_out);
int pagoda_pool_waitAll(pagoda_pool* pool);
int pagoda_pool_shutdown(pagoda_pool* pool);
/* NUMA node member i's spawner thread is bound to (-1: unknown / not bound). */
int pagoda_pool_numa_node(pagoda_pool* pool, int index);
/* Member i's share of the last batched spawn: tasks it spawned, ns inside its spawn calls
 * (the host cost: tasks / spawn_ns is that thread's spawn rate), ns it held back because
 * another member was less loaded.  Returns 0 or -EINVAL. */
int pagoda_pool_stats(pagoda_pool* pool, int index, int64_t* tasks, int64_t* spawn_ns, int64_t* hold_ns);

/* In-flight warps of one context: warps of spawned tasks minus those of the
 * tasks below its completion watermark (the pool's load measure). */
int64_t pagoda_inflight_warps(pagoda_ctx* ctx);
/* The picker rule alone (host-only, testable without a GPU): index of the
 * smallest of loads[0..n), ties to the lowest index; -EINVAL if n < 1. */
int pagoda_pick_least_loaded(const int64_t* loads, int n);
/* The spawner's claim rule alone (host-only): 1 if loads[me] <= min(loads) + slack, else 0;
 * -EINVAL on bad arguments. */
int pagoda_pool_may_claim(const int64_t* loads, int n, int me, int64_t slack);

/* Library version string. */
const char* pagoda_version(void);

#ifdef __cplusplus
}
#endif
#endif
