// What does a gpu-scope fence wait for?  Warp 1 of block 0 times fence.acq_rel.gpu
// (MEMBAR.ALL.GPU + ERRBAR) while an "agitator" warp (warp 0 of block 0 = same SM,
// or warp 0 of block 1 = another SM) keeps PCIe traffic in flight:
//   mode 0: agitator idle; 1: bulk TMA reads of pinned host memory into smem;
//   2: posted stores to pinned host memory; 3: plain loads of pinned host memory.
// Build: nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o membar_probe membar_probe.cu
#include <cuda_runtime.h>
#include <stdio.h>
#include <stdint.h>
#include <thread>
#include <atomic>

__device__ __forceinline__ uint64_t gtime() { uint64_t t; asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t)); return t; }

__global__ void probe(int mode, int same_sm, const char* host, volatile uint64_t* hostw, uint64_t* out, volatile int* stop)
{
    extern __shared__ __align__(128) unsigned char sm[];
    __shared__ uint64_t bar;
    const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
    if (threadIdx.x == 0) {
        asm volatile("mbarrier.init.shared::cta.b64 [%0], 1;" :: "r"((uint32_t)__cvta_generic_to_shared(&bar)));
        asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    }
    __syncthreads();
    const bool agitator = same_sm ? (blockIdx.x == 0 && warp == 0) : (blockIdx.x == 1 && warp == 0);
    const bool timer = blockIdx.x == 0 && warp == 1;
    if (agitator && mode != 0) {
        uint32_t phase = 0;
        uint64_t i = 0;
        while (*stop == 0) {
            if (mode == 1) {
                if (lane == 0) {
                    uint32_t b = (uint32_t)__cvta_generic_to_shared(&bar);
                    asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" :: "r"(b), "r"(65536u) : "memory");
                    asm volatile("cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
                                 :: "r"((uint32_t)__cvta_generic_to_shared(sm)), "l"(host + ((i * 65536) & ((64u << 20) - 1))), "r"(65536u), "r"(b) : "memory");
                    uint32_t done = 0;
                    while (!done) asm volatile("{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0,1,0,p; }" : "=r"(done) : "r"(b), "r"(phase) : "memory");
                    phase ^= 1;
                }
                __syncwarp();
            } else if (mode == 2) {
                hostw[(i * 32 + lane) & 4095] = i;
            } else if (mode == 3) {
                uint64_t v = *(volatile const uint64_t*)(host + ((i * 4096 + lane * 128) & ((64u << 20) - 1)));
                if (v == 0x1234567) out[8] = v;
            }
            i++;
        }
    }
    if (timer && lane == 0) {
        uint64_t tot = 0, mx = 0;
        const int n = 2000;
        for (int k = 0; k < n; k++) {
            uint64_t t0 = gtime();
            asm volatile("fence.acq_rel.gpu;" ::: "memory");
            uint64_t d = gtime() - t0;
            tot += d;
            mx = d > mx ? d : mx;
            for (int j = 0; j < 100; j++) __nanosleep(100);
        }
        out[0] = tot / n;
        out[1] = mx;
        *(volatile int*)stop = 1;
    }
}

int main()
{
    char* host; cudaHostAlloc(&host, 64u << 20, cudaHostAllocMapped);
    uint64_t* hostw; cudaHostAlloc(&hostw, 4096 * 8, cudaHostAllocMapped);
    uint64_t* out; cudaMalloc(&out, 64 * 8);
    int* stop; cudaMalloc(&stop, 4);
    // contention source: a big H2D copy loop on another stream + thread
    char* hbig; cudaHostAlloc(&hbig, 256u << 20, 0);
    char* dbig; cudaMalloc(&dbig, 256u << 20);
    cudaStream_t s1, s2; cudaStreamCreateWithFlags(&s1, cudaStreamNonBlocking); cudaStreamCreateWithFlags(&s2, cudaStreamNonBlocking);
    cudaFuncSetAttribute(probe, cudaFuncAttributeMaxDynamicSharedMemorySize, 65536 + 1024);
    for (int cont = 0; cont < 3; cont++) {
        std::atomic<int> go{1};
        std::thread th;
        if (cont) th = std::thread([&] { cudaSetDevice(0); while (go) { if (cont == 1) cudaMemcpyAsync(dbig, hbig, 256u << 20, cudaMemcpyHostToDevice, s2); else cudaMemcpyAsync(hbig, dbig, 256u << 20, cudaMemcpyDeviceToHost, s2); cudaStreamSynchronize(s2); } });
        for (int mode = 0; mode < 4; mode++)
            for (int same = 1; same >= 0; same--) {
                if (mode == 0 && same == 0) continue;
                cudaMemsetAsync(stop, 0, 4, s1);
                probe<<<2, 64, 65536 + 1024, s1>>>(mode, same, host, hostw, out, stop);
                uint64_t h[2];
                cudaMemcpyAsync(h, out, 16, cudaMemcpyDeviceToHost, s1);
                cudaStreamSynchronize(s1);
                printf("{\"contention\": \"%s\", \"agitator\": \"%s\", \"where\": \"%s\", \"fence_avg_ns\": %llu, \"fence_max_ns\": %llu}\n",
                       cont == 0 ? "none" : cont == 1 ? "h2d_copy" : "d2h_copy",
                       mode == 0 ? "idle" : mode == 1 ? "tma_host_reads" : mode == 2 ? "host_posted_writes" : "host_loads",
                       same ? "same_sm" : "other_sm", (unsigned long long)h[0], (unsigned long long)h[1]);
                fflush(stdout);
            }
        go = 0;
        if (cont) th.join();
    }
    printf("{\"status\": \"%s\"}\n", cudaGetErrorString(cudaGetLastError()));
    return 0;
}
