/*
 * naive.cu — two host-side pieces that sit beside the MasterKernel:
 *
 * 1. The naive baseline: every task is its own kernel launch
 *    <<<n_tb, warps*32, shmem>>> of the SAME body (NativeEnv), issued
 *    round-robin on up to 32 streams — the paper's CUDA-HyperQ comparison
 *    (set CUDA_DEVICE_MAX_CONNECTIONS=32 before the CUDA
 *    context is created).
 * 2. The static-fusion baseline (NEXT-2): every task fused into
 *    ONE kernel launch, one thread block of a fixed thread count per task
 *    (the paper uses 256), the task's shape and args read from a device table.
 * 3. The multi-GPU pool: one context per GPU and a
 *    least-loaded picker (fewest in-flight warps, ties to the lowest index).
 */
#include <cuda_runtime.h>
#include <errno.h>
#include <stdint.h>
#include <string.h>
#include <time.h>

#include <algorithm>
#include <climits>
#include <mutex>
#include <vector>

#include "bodies.cuh"
#include "pagoda.h"

using namespace pagoda;

struct alignas(8) ArgBlock {
    unsigned char b[PAGODA_ARGS_MAX];
};

__global__ void naive_task_kernel(int func_id, int threads_tb, uint32_t smem_bytes, ArgBlock a)
{
    NativeEnv env{threads_tb, smem_bytes};
    run_body(func_id, env, a.b);
}

static uint64_t mono_ns()
{
    timespec ts;
    clock_gettime(CLOCK_MONOTONIC, &ts);
    return (uint64_t)ts.tv_sec * 1000000000ull + (uint64_t)ts.tv_nsec;
}

extern "C" int pagoda_naive_run(int device, int n, const int32_t* shapes, const void* args_base, size_t args_stride,
                                size_t args_bytes, int n_streams, int64_t* elapsed_ns)
{
    if (n < 0 || !shapes || n_streams < 1 || n_streams > 32 || args_bytes > PAGODA_ARGS_MAX) return -EINVAL;
    if (cudaSetDevice(device) != cudaSuccess) return -ENODEV;
    int max_smem = 0;
    for (int i = 0; i < n; i++) max_smem = std::max(max_smem, (int)shapes[5 * (size_t)i + 2]);
    int rounded = ((max_smem + PAGODA_GRANULE - 1) / PAGODA_GRANULE) * PAGODA_GRANULE;
    if (cudaFuncSetAttribute(naive_task_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, std::max(rounded, 0)) !=
        cudaSuccess)
        return -EINVAL;
    std::vector<cudaStream_t> st(n_streams);
    for (auto& s : st)
        if (cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking) != cudaSuccess) return -EIO;
    if (cudaDeviceSynchronize() != cudaSuccess) return -EIO;
    const char* a = static_cast<const char*>(args_base);
    const uint64_t t0 = mono_ns();
    for (int i = 0; i < n; i++) {
        const int32_t* s = shapes + 5 * (size_t)i;
        ArgBlock ab;
        memset(&ab, 0, sizeof ab);
        if (a && args_bytes) memcpy(ab.b, a + (size_t)i * args_stride, args_bytes);
        const int warps = (s[0] + 31) / 32;
        const uint32_t g = ((uint32_t)s[2] + PAGODA_GRANULE - 1) / PAGODA_GRANULE * PAGODA_GRANULE;
        naive_task_kernel<<<s[1], warps * 32, g, st[i % n_streams]>>>(s[4], s[0], g, ab);
    }
    cudaError_t e = cudaDeviceSynchronize();
    const uint64_t t1 = mono_ns();
    for (auto& s : st) cudaStreamDestroy(s);
    if (elapsed_ns) *elapsed_ns = (int64_t)(t1 - t0);
    return e == cudaSuccess ? 0 : -EIO;
}

/* ------------------------------------------------------------------ static fusion */
struct FusedTask {
    int32_t func_id;
    uint32_t smem_bytes;   /* the task's request rounded to the granule */
    ArgBlock a;
};

__global__ void fused_tasks_kernel(const FusedTask* __restrict__ tasks)
{
    const FusedTask& t = tasks[blockIdx.x];
    FusedEnv env{t.smem_bytes};
    run_body(t.func_id, env, t.a.b);
}

extern "C" int pagoda_fused_run(int device, int n, const int32_t* shapes, const void* args_base, size_t args_stride,
                                size_t args_bytes, int threads_per_task, int64_t* elapsed_ns, float* kernel_ms)
{
    if (n < 0 || (n > 0 && !shapes) || args_bytes > PAGODA_ARGS_MAX || threads_per_task < 32 ||
        threads_per_task > 1024 || threads_per_task % 32)
        return -EINVAL;
    if (cudaSetDevice(device) != cudaSuccess) return -ENODEV;
    std::vector<FusedTask> h(n);
    uint32_t max_smem = 0;
    const char* a = static_cast<const char*>(args_base);
    for (int i = 0; i < n; i++) {
        const int32_t* s = shapes + 5 * (size_t)i;
        if (s[1] != 1 || s[0] < 1 || s[2] < 0) return -EINVAL;   /* one thread block per task */
        h[i].func_id = s[4];
        h[i].smem_bytes = ((uint32_t)s[2] + PAGODA_GRANULE - 1) / PAGODA_GRANULE * PAGODA_GRANULE;
        max_smem = std::max(max_smem, h[i].smem_bytes);
        memset(&h[i].a, 0, sizeof h[i].a);
        if (a && args_bytes) memcpy(h[i].a.b, a + (size_t)i * args_stride, args_bytes);
    }
    if (cudaFuncSetAttribute(fused_tasks_kernel, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)max_smem) !=
        cudaSuccess)
        return -EINVAL;
    FusedTask* d = nullptr;
    if (n && cudaMalloc(&d, sizeof(FusedTask) * (size_t)n) != cudaSuccess) return -ENOMEM;
    cudaEvent_t e0, e1;
    cudaEventCreate(&e0);
    cudaEventCreate(&e1);
    cudaStream_t st;
    cudaStreamCreateWithFlags(&st, cudaStreamNonBlocking);
    cudaError_t err = cudaDeviceSynchronize();
    const uint64_t t0 = mono_ns();
    if (n) {   /* the task table is part of the timed region, as Pagoda's spawns are */
        cudaMemcpyAsync(d, h.data(), sizeof(FusedTask) * (size_t)n, cudaMemcpyHostToDevice, st);
        cudaEventRecord(e0, st);
        fused_tasks_kernel<<<n, threads_per_task, max_smem, st>>>(d);
        cudaEventRecord(e1, st);
    }
    if (err == cudaSuccess) err = cudaStreamSynchronize(st);
    const uint64_t t1 = mono_ns();
    if (kernel_ms) {
        *kernel_ms = 0.f;
        if (n && err == cudaSuccess) cudaEventElapsedTime(kernel_ms, e0, e1);
    }
    if (elapsed_ns) *elapsed_ns = (int64_t)(t1 - t0);
    cudaEventDestroy(e0);
    cudaEventDestroy(e1);
    cudaStreamDestroy(st);
    if (d) cudaFree(d);
    return err == cudaSuccess ? 0 : -EIO;
}

/* ------------------------------------------------------------------ pool */
extern "C" int64_t pagoda_inflight_warps(pagoda_ctx* c);

/* pure picker: index of the smallest load, ties to the lowest index */
extern "C" int pagoda_pick_least_loaded(const int64_t* loads, int n)
{
    if (!loads || n < 1) return -EINVAL;
    int best = 0;
    for (int i = 1; i < n; i++)
        if (loads[i] < loads[best]) best = i;
    return best;
}

struct pagoda_pool {
    std::vector<pagoda_ctx*> ctx;
    std::vector<int64_t> pending;   /* warps picked but not yet counted by the context */
    std::mutex m;
};

extern "C" int pagoda_pool_init(int n_dev, const int* devices, const pagoda_config* cfg, pagoda_pool** out)
{
    if (!out || n_dev < 1 || !devices) return -EINVAL;
    pagoda_pool* p = new pagoda_pool;
    pagoda_config c;
    if (cfg) c = *cfg;
    else pagoda_config_default(&c);
    for (int i = 0; i < n_dev; i++) {
        c.device = devices[i];
        pagoda_ctx* x = nullptr;
        int rc = pagoda_init(&c, &x);
        if (rc) {
            for (auto* y : p->ctx) pagoda_shutdown(y);
            delete p;
            return rc;
        }
        p->ctx.push_back(x);
    }
    p->pending.assign(n_dev, 0);
    *out = p;
    return 0;
}

extern "C" int pagoda_pool_size(pagoda_pool* p) { return p ? (int)p->ctx.size() : -EINVAL; }

extern "C" pagoda_ctx* pagoda_pool_ctx(pagoda_pool* p, int i)
{
    return (p && i >= 0 && i < (int)p->ctx.size()) ? p->ctx[i] : nullptr;
}

extern "C" int pagoda_pool_pick(pagoda_pool* p, int warps_hint)
{
    if (!p) return -EINVAL;
    std::lock_guard<std::mutex> lk(p->m);
    std::vector<int64_t> load(p->ctx.size());
    for (size_t i = 0; i < p->ctx.size(); i++) load[i] = pagoda_inflight_warps(p->ctx[i]) + p->pending[i];
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
    pagoda_task_t id = pagoda_taskSpawn(p->ctx[i], threads, n_tb, shmem_bytes, sync_flag, func_id,
                                        args_per_dev ? args_per_dev[i] : nullptr, args_bytes);
    {
        std::lock_guard<std::mutex> lk(p->m);
        p->pending[i] -= w;   /* now counted by the context itself (or failed) */
    }
    if (index_out) *index_out = i;
    return id;
}

/* Batched least-loaded spawning: runs of up to `chunk` tasks go
 * to the context with the fewest in-flight warps at the time of the pick (each
 * run one pagoda_taskSpawnShapes on that context, with that device's args). */
extern "C" int64_t pagoda_pool_spawn_shapes(pagoda_pool* p, int n, const int32_t* shapes,
                                            const void* const* args_base_per_dev, size_t args_stride,
                                            size_t args_bytes, int chunk, pagoda_task_t* ids_out, int32_t* dev_out)
{
    if (!p || n < 0 || (n > 0 && !shapes) || chunk < 1) return -EINVAL;
    for (int base = 0; base < n; base += chunk) {
        const int m = std::min(chunk, n - base);
        int64_t w = 0;
        for (int i = 0; i < m; i++) {
            const int32_t* s = shapes + 5 * (size_t)(base + i);
            w += (int64_t)((s[0] + 31) / 32) * s[1];
        }
        const int d = pagoda_pool_pick(p, (int)std::min<int64_t>(w, INT32_MAX));
        if (d < 0) return d;
        const char* a = args_base_per_dev ? static_cast<const char*>(args_base_per_dev[d]) : nullptr;
        const int64_t rc = pagoda_taskSpawnShapes(p->ctx[d], m, shapes + 5 * (size_t)base,
                                                  a ? a + (size_t)base * args_stride : nullptr, args_stride, args_bytes,
                                                  ids_out ? ids_out + base : nullptr);
        {
            std::lock_guard<std::mutex> lk(p->m);
            p->pending[d] -= (int64_t)std::min<int64_t>(w, INT32_MAX);
        }
        if (rc < 0) return rc;
        if (dev_out)
            for (int i = 0; i < m; i++) dev_out[base + i] = d;
    }
    return n;
}

extern "C" int pagoda_pool_waitAll(pagoda_pool* p)
{
    if (!p) return -EINVAL;
    int rc = 0;
    for (auto* c : p->ctx) {
        int r = pagoda_waitAll(c);
        if (r && !rc) rc = r;
    }
    return rc;
}

extern "C" int pagoda_pool_shutdown(pagoda_pool* p)
{
    if (!p) return -EINVAL;
    int rc = 0;
    for (auto* c : p->ctx) {
        int r = pagoda_shutdown(c);
        if (r && !rc) rc = r;
    }
    delete p;
    return rc;
}
