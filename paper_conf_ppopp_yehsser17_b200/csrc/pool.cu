/*
 * pool.cu — the multi-GPU pool (BASELINE.json north star: "one
 * MasterKernel per GPU and a host spawner distributing tasks least-loaded-first").
 *
 * Tasks are independent, so there is no collective: the pool is
 * host-side only.  Each member is one context (one MasterKernel) plus ONE
 * spawner thread of its own, bound to the CPUs of the GPU's NUMA node; the
 * thread also creates the context, so its pinned TaskTable ring, doorbell and
 * completion window are first-touched on that node.  A batched spawn
 * (pagoda_pool_spawn_shapes) is cut into chunks; every spawner claims the next
 * chunk only while its GPU is among the least loaded (in-flight warps <= the
 * smallest member's + one chunk's warps), so chunks go least-loaded-first and
 * the spawners write their rings in parallel (one host thread per GPU: the
 * single spawn loop of one thread tops out near 65 M entries/s).
 *
 * Several members may share one device (each with num_sms SMs: two half-GPU
 * MasterKernels co-reside), which exercises the pool on a one-GPU machine.
 */
#include <cuda_runtime.h>
#include <errno.h>
#include <pthread.h>
#include <sched.h>
#include <stdint.h>
#include <stdio.h>
#include <string.h>
#include <time.h>
#include <immintrin.h>

#include <algorithm>
#include <atomic>
#include <climits>
#include <condition_variable>
#include <mutex>
#include <thread>
#include <vector>

#include "pagoda.h"

extern "C" int64_t pagoda_inflight_warps(pagoda_ctx* c);

static inline uint64_t pool_now_ns()
{
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
}

/* NUMA node of a CUDA device from sysfs (-1 if unknown) */
static int device_numa_node(int dev)
{
    char bus[32] = {0};
    if (cudaDeviceGetPCIBusId(bus, sizeof bus, dev) != cudaSuccess) {
        cudaGetLastError();
        return -1;
    }
    for (char* c = bus; *c; c++)
        if (*c >= 'A' && *c <= 'F') *c = (char)(*c - 'A' + 'a');
    char path[128];
    snprintf(path, sizeof path, "/sys/bus/pci/devices/%s/numa_node", bus);
    FILE* f = fopen(path, "r");
    if (!f) return -1;
    int node = -1;
    if (fscanf(f, "%d", &node) != 1) node = -1;
    fclose(f);
    return node;
}

/* bind the calling thread to the CPUs of NUMA node `node` ("0-55,112-167" lists); false if not possible */
static bool bind_to_node(int node)
{
    if (node < 0) return false;
    char path[96];
    snprintf(path, sizeof path, "/sys/devices/system/node/node%d/cpulist", node);
    FILE* f = fopen(path, "r");
    if (!f) return false;
    char buf[4096] = {0};
    const bool got = fgets(buf, sizeof buf, f) != nullptr;
    fclose(f);
    if (!got) return false;
    cpu_set_t set;
    CPU_ZERO(&set);
    int n = 0;
    for (char* s = buf; *s && *s != '\n';) {
        char* e = nullptr;
        long a = strtol(s, &e, 10);
        if (e == s) break;
        long b = a;
        if (*e == '-') {
            s = e + 1;
            b = strtol(s, &e, 10);
        }
        for (long c = a; c <= b && c < CPU_SETSIZE; c++, n++) CPU_SET((int)c, &set);
        s = (*e == ',') ? e + 1 : e;
    }
    return n > 0 && pthread_setaffinity_np(pthread_self(), sizeof set, &set) == 0;
}

/* pure picker: index of the smallest load, ties to the lowest index */
extern "C" int pagoda_pick_least_loaded(const int64_t* loads, int n)
{
    if (!loads || n < 1) return -EINVAL;
    int best = 0;
    for (int i = 1; i < n; i++)
        if (loads[i] < loads[best]) best = i;
    return best;
}

/* Claim rule of a spawner (host-only, unit-tested): member `me` may take the
 * next chunk iff its load is within `slack` warps of the least-loaded member's. */
extern "C" int pagoda_pool_may_claim(const int64_t* loads, int n, int me, int64_t slack)
{
    if (!loads || n < 1 || me < 0 || me >= n || slack < 0) return -EINVAL;
    int64_t lo = loads[0];
    for (int i = 1; i < n; i++) lo = std::min(lo, loads[i]);
    return loads[me] <= lo + slack ? 1 : 0;
}

struct PoolJob {
    const int32_t* shapes = nullptr;
    const void* const* args = nullptr;
    size_t stride = 0, bytes = 0;
    int n = 0, chunk = 0;
    int64_t slack = 0;
    pagoda_task_t* ids = nullptr;
    int32_t* dev = nullptr;
};

struct PoolMember {
    pagoda_ctx* ctx = nullptr;
    int device = 0, numa = -1, bound = 0;
    std::thread th;
    /* stats of the last batched spawn (pagoda_pool_stats) */
    std::atomic<int64_t> tasks{0}, spawn_ns{0}, hold_ns{0};
};

struct pagoda_pool {
    std::vector<PoolMember*> m;
    std::vector<int64_t> pending;   /* pagoda_pool_pick: warps picked but not yet spawned */
    std::mutex pick_mtx;
    /* batched-spawn job handed to the spawner threads */
    std::mutex job_mtx;             /* one batched spawn at a time */
    std::mutex cv_mtx;
    std::condition_variable cv;
    uint64_t gen = 0;               /* job generation (guarded by cv_mtx) */
    bool quit = false;
    PoolJob job;
    std::atomic<int64_t> next{0};
    std::atomic<int> left{0};
    std::atomic<int64_t> rc{0};
    std::atomic<int> init_left{0};
};

static int64_t member_load(pagoda_pool* p, int i) { return pagoda_inflight_warps(p->m[i]->ctx); }

/* one spawner's share of a batched spawn */
static void run_job(pagoda_pool* p, int me)
{
    const PoolJob& j = p->job;
    PoolMember& M = *p->m[me];
    const int k = (int)p->m.size();
    std::vector<int64_t> loads(k);
    const uint64_t t_start = pool_now_ns();
    int64_t spawned = 0, hold = 0, spawn = 0;
    for (;;) {
        if (p->next.load(std::memory_order_relaxed) >= j.n || p->rc.load(std::memory_order_relaxed) < 0) break;
        /* least-loaded first: claim only while within one chunk of the smallest load */
        if (k > 1) {
            for (int i = 0; i < k; i++) loads[i] = member_load(p, i);
            if (!pagoda_pool_may_claim(loads.data(), k, me, j.slack)) {
                const uint64_t t0 = pool_now_ns();
                for (int s = 0; s < 64; s++) _mm_pause();
                hold += (int64_t)(pool_now_ns() - t0);
                continue;
            }
        }
        const int64_t c = p->next.fetch_add(j.chunk, std::memory_order_acq_rel);
        if (c >= j.n) break;
        const int m = (int)std::min<int64_t>(j.chunk, j.n - c);
        const char* a = j.args ? static_cast<const char*>(j.args[me]) : nullptr;
        const uint64_t t0 = pool_now_ns();
        const int64_t rc = pagoda_taskSpawnShapes(M.ctx, m, j.shapes + 5 * (size_t)c,
                                                  a ? a + (size_t)c * j.stride : nullptr, j.stride, j.bytes,
                                                  j.ids ? j.ids + c : nullptr);
        spawn += (int64_t)(pool_now_ns() - t0);
        if (rc != m) {
            int64_t z = 0;
            p->rc.compare_exchange_strong(z, rc < 0 ? rc : -EAGAIN);
            break;
        }
        if (j.dev)
            for (int i = 0; i < m; i++) j.dev[c + i] = me;
        spawned += m;
    }
    (void)t_start;
    M.tasks.store(spawned);
    M.spawn_ns.store(spawn);
    M.hold_ns.store(hold);
}

static void spawner_main(pagoda_pool* p, int me, pagoda_config cfg)
{
    PoolMember& M = *p->m[me];
    cudaSetDevice(M.device);
    M.numa = device_numa_node(M.device);
    M.bound = bind_to_node(M.numa) ? 1 : 0;
    /* the context is created on this (node-bound) thread: its pinned rings are first-touched here */
    cfg.device = M.device;
    pagoda_ctx* c = nullptr;
    const int rc = pagoda_init(&cfg, &c);
    M.ctx = c;
    if (rc) {
        int64_t z = 0;
        p->rc.compare_exchange_strong(z, rc);
    }
    p->init_left.fetch_sub(1, std::memory_order_acq_rel);
    uint64_t seen = 0;
    for (;;) {
        {
            std::unique_lock<std::mutex> lk(p->cv_mtx);
            p->cv.wait(lk, [&] { return p->quit || p->gen != seen; });
            if (p->quit) return;
            seen = p->gen;
        }
        if (M.ctx) run_job(p, me);
        p->left.fetch_sub(1, std::memory_order_acq_rel);
    }
}

static void stop_spawners(pagoda_pool* p)
{
    {
        std::lock_guard<std::mutex> lk(p->cv_mtx);
        p->quit = true;
    }
    p->cv.notify_all();
    for (auto* m : p->m)
        if (m->th.joinable()) m->th.join();
}

extern "C" int pagoda_pool_init(int n_dev, const int* devices, const pagoda_config* cfg, pagoda_pool** out)
{
    if (!out || n_dev < 1 || !devices) return -EINVAL;
    *out = nullptr;
    pagoda_config c;
    if (cfg) c = *cfg;
    else pagoda_config_default(&c);
    pagoda_pool* p = new pagoda_pool;
    p->init_left.store(n_dev);
    for (int i = 0; i < n_dev; i++) {
        PoolMember* m = new PoolMember;
        m->device = devices[i];
        p->m.push_back(m);
    }
    for (int i = 0; i < n_dev; i++) p->m[i]->th = std::thread(spawner_main, p, i, c);
    while (p->init_left.load(std::memory_order_acquire) > 0) std::this_thread::yield();
    const int rc = (int)p->rc.load();
    if (rc) {
        stop_spawners(p);
        for (auto* m : p->m) {
            if (m->ctx) pagoda_shutdown(m->ctx);
            delete m;
        }
        delete p;
        return rc;
    }
    p->pending.assign(n_dev, 0);
    *out = p;
    return 0;
}

extern "C" int pagoda_pool_size(pagoda_pool* p) { return p ? (int)p->m.size() : -EINVAL; }

extern "C" pagoda_ctx* pagoda_pool_ctx(pagoda_pool* p, int i)
{
    return (p && i >= 0 && i < (int)p->m.size()) ? p->m[i]->ctx : nullptr;
}

extern "C" int pagoda_pool_numa_node(pagoda_pool* p, int i)
{
    if (!p || i < 0 || i >= (int)p->m.size()) return -EINVAL;
    return p->m[i]->bound ? p->m[i]->numa : -1;
}

extern "C" int pagoda_pool_stats(pagoda_pool* p, int i, int64_t* tasks, int64_t* spawn_ns, int64_t* hold_ns)
{
    if (!p || i < 0 || i >= (int)p->m.size()) return -EINVAL;
    if (tasks) *tasks = p->m[i]->tasks.load();
    if (spawn_ns) *spawn_ns = p->m[i]->spawn_ns.load();
    if (hold_ns) *hold_ns = p->m[i]->hold_ns.load();
    return 0;
}

extern "C" int pagoda_pool_pick(pagoda_pool* p, int warps_hint)
{
    if (!p) return -EINVAL;
    std::lock_guard<std::mutex> lk(p->pick_mtx);
    std::vector<int64_t> load(p->m.size());
    for (size_t i = 0; i < p->m.size(); i++) load[i] = member_load(p, (int)i) + p->pending[i];
    const int best = pagoda_pick_least_loaded(load.data(), (int)load.size());
    p->pending[best] += warps_hint;
    return best;
}

extern "C" pagoda_task_t pagoda_pool_spawn(pagoda_pool* p, int threads, int n_tb, int shmem_bytes, int sync_flag,
                                           int func_id, const void* const* args_per_dev, size_t args_bytes,
                                           int* index_out)
{
    if (!p) return -EINVAL;
    const int w = ((threads + 31) / 32) * n_tb;
    const int i = pagoda_pool_pick(p, w);
    if (i < 0) return i;
    pagoda_task_t id = pagoda_taskSpawn(p->m[i]->ctx, threads, n_tb, shmem_bytes, sync_flag, func_id,
                                        args_per_dev ? args_per_dev[i] : nullptr, args_bytes);
    {
        std::lock_guard<std::mutex> lk(p->pick_mtx);
        p->pending[i] -= w;   /* now counted by the context itself (or failed) */
    }
    if (index_out) *index_out = i;
    return id;
}

/* Batched least-loaded spawning on every member's own spawner thread (see the
 * file comment).  Returns n, or the first error (chunks claimed before it stay
 * spawned). */
extern "C" int64_t pagoda_pool_spawn_shapes(pagoda_pool* p, int n, const int32_t* shapes,
                                            const void* const* args_base_per_dev, size_t args_stride,
                                            size_t args_bytes, int chunk, pagoda_task_t* ids_out, int32_t* dev_out)
{
    if (!p || n < 0 || (n > 0 && !shapes) || chunk < 1) return -EINVAL;
    if (n == 0) return 0;
    std::lock_guard<std::mutex> jl(p->job_mtx);
    int64_t warps = 0;
    for (int i = 0; i < n; i++) warps += (int64_t)((shapes[5 * (size_t)i] + 31) / 32) * shapes[5 * (size_t)i + 1];
    PoolJob j;
    j.shapes = shapes;
    j.args = args_base_per_dev;
    j.stride = args_stride;
    j.bytes = args_bytes;
    j.n = n;
    j.chunk = chunk;
    j.slack = std::max<int64_t>(1, 2 * (warps * chunk + n - 1) / n);   /* two chunks' worth of warps */
    j.ids = ids_out;
    j.dev = dev_out;
    p->job = j;
    p->next.store(0);
    p->rc.store(0);
    p->left.store((int)p->m.size(), std::memory_order_release);
    {
        std::lock_guard<std::mutex> lk(p->cv_mtx);
        p->gen++;
    }
    p->cv.notify_all();
    while (p->left.load(std::memory_order_acquire) > 0) _mm_pause();
    const int64_t rc = p->rc.load();
    return rc < 0 ? rc : n;
}

extern "C" int pagoda_pool_waitAll(pagoda_pool* p)
{
    if (!p) return -EINVAL;
    int rc = 0;
    for (auto* m : p->m) {
        int r = pagoda_waitAll(m->ctx);
        if (r && !rc) rc = r;
    }
    return rc;
}

extern "C" int pagoda_pool_shutdown(pagoda_pool* p)
{
    if (!p) return -EINVAL;
    stop_spawners(p);
    int rc = 0;
    /* every member's MasterKernel exits BEFORE any member frees memory: cudaFree synchronizes the
     * whole device, so freeing one member while another (sharing the GPU) still runs would never
     * return */
    for (auto* m : p->m) {
        int r = pagoda_waitAll(m->ctx);
        if (r && !rc) rc = r;
    }
    for (auto* m : p->m) {
        int r = pagoda_stop(m->ctx);
        if (r && r != -EALREADY && !rc) rc = r;
    }
    for (auto* m : p->m) {
        int r = pagoda_shutdown(m->ctx);
        if (r && !rc) rc = r;
        delete m;
    }
    delete p;
    return rc;
}
