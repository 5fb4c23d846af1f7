/*
 * measure.cu — measurement helpers over the public API (pagoda.h
 * "Measurement"): a timed spawn run that records per-task spawn and done
 * times (the metric's p50 spawn-to-done latency under load), and the isolated
 * closed-loop latency of one task at a time.  Host clock: CLOCK_MONOTONIC.
 */
#include <errno.h>
#include <stdint.h>
#include <string.h>
#include <time.h>
#include <immintrin.h>

#include <atomic>
#include <thread>
#include <vector>

#include "pagoda.h"

static inline int64_t mono_ns()
{
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (int64_t)ts.tv_sec * 1000000000ll + (int64_t)ts.tv_nsec;
}

extern "C" int64_t pagoda_run_timed(pagoda_ctx* c, int n, const int32_t* shapes, const void* args_base,
                                    size_t args_stride, size_t args_bytes, int64_t* spawn_ns, int64_t* done_ns)
{
    if (!c || n < 0 || !shapes || !spawn_ns || !done_ns) return -EINVAL;
    memset(done_ns, 0, sizeof(int64_t) * (size_t)n);
    std::vector<pagoda_task_t> ids((size_t)n, -1);
    std::atomic<int> spawned{0};
    std::atomic<int> err{0};
    /* poller: stamps each task the first time check() reports it done */
    std::thread poller([&] {
        int lo = 0;
        while (lo < n && !err.load(std::memory_order_relaxed)) {
            const int hi = spawned.load(std::memory_order_acquire);
            const int end = hi < lo + 8192 ? hi : lo + 8192;
            for (int i = lo; i < end; i++) {
                if (done_ns[i]) continue;
                const int r = pagoda_check(c, ids[i]);
                if (r == 1) done_ns[i] = mono_ns();
                else if (r < 0) { err.store(r); return; }
            }
            while (lo < hi && done_ns[lo]) lo++;
            if (lo == end) _mm_pause();
        }
    });
    const char* a = static_cast<const char*>(args_base);
    for (int i = 0; i < n; i++) {
        const int32_t* s = shapes + 5 * (size_t)i;
        spawn_ns[i] = mono_ns();
        const pagoda_task_t id =
            pagoda_taskSpawn(c, s[0], s[1], s[2], s[3], s[4], a ? a + (size_t)i * args_stride : nullptr, args_bytes);
        if (id < 0) {
            err.store((int)id);
            break;
        }
        ids[i] = id;
        spawned.store(i + 1, std::memory_order_release);
    }
    poller.join();
    if (err.load()) return err.load();
    return n;
}

extern "C" int pagoda_latency_loop(pagoda_ctx* c, int n, int threads, int n_tb, int shmem_bytes, int sync_flag,
                                   int func_id, const void* args, size_t args_bytes, int64_t* lat_ns)
{
    if (!c || n < 0 || !lat_ns) return -EINVAL;
    for (int i = 0; i < n; i++) {
        const int64_t t0 = mono_ns();
        const pagoda_task_t id = pagoda_taskSpawn(c, threads, n_tb, shmem_bytes, sync_flag, func_id, args, args_bytes);
        if (id < 0) return (int)id;
        const int r = pagoda_wait(c, id);
        if (r) return r;
        lat_ns[i] = mono_ns() - t0;
    }
    return 0;
}
