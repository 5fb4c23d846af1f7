/*
 * naive.cu — the two baselines that sit beside the MasterKernel:
 *
 * 1. The naive baseline: every task is its own kernel launch
 *    <<<n_tb, warps*32, shmem>>> of the SAME body (NativeEnv), issued
 *    round-robin on up to 32 streams — the paper's CUDA-HyperQ comparison
 *    (set CUDA_DEVICE_MAX_CONNECTIONS=32 before the CUDA
 *    context is created).
 * 2. The static-fusion baseline (NEXT-2): every task fused into
 *    ONE kernel launch, one thread block of a fixed thread count per task
 *    (the paper uses 256), the task's shape and args read from a device table.
 * (The multi-GPU pool lives in pool.cu.)
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
