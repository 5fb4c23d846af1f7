// The paper's host API under its own names (include/pagoda.hpp), called from C++
// the way Fig. 1a calls it.  Built and run by tests/test_cpp_api.py.
//   no GPU:   every paper call fails loudly with the C ABI's codes; prints "nodev"
//   a B200:   spawn MARK / GATE tasks, check / wait / waitAll, verify; prints "ok"
#include <cuda_runtime.h>

#include <cstdio>
#include <vector>

#include "pagoda.hpp"

#define REQUIRE(c)                                                   \
    do {                                                             \
        if (!(c)) {                                                  \
            std::fprintf(stderr, "FAILED %s (line %d)\n", #c, __LINE__); \
            return 1;                                                \
        }                                                            \
    } while (0)

int main()
{
    const int n = 64, threads = 100;   // 4 warps per task, 28 idle padding lanes
    uint32_t *out = nullptr, *cnt = nullptr;
    volatile uint32_t* flag = nullptr;
    // device buffers are prepared BEFORE the MasterKernel starts (it holds every SM)
    const bool gpu = cudaMalloc(&out, 4 * 128 * n) == cudaSuccess;
    if (gpu) {
        REQUIRE(cudaMalloc(&cnt, 4 * n) == cudaSuccess);
        REQUIRE(cudaMemset(out, 0, 4 * 128 * n) == cudaSuccess && cudaMemset(cnt, 0, 4 * n) == cudaSuccess);
        REQUIRE(cudaHostAlloc((void**)&flag, 64, cudaHostAllocMapped) == cudaSuccess);
        REQUIRE(cudaDeviceSynchronize() == cudaSuccess);
        *flag = 0;
    }
    const int rc = pagoda::init();
    if (rc == -ENODEV) {
        REQUIRE(pagoda::taskSpawn(128, 1, 0, 0, PAGODA_NOP, nullptr, 0) == -EINVAL);
        REQUIRE(pagoda::wait(0) == -EINVAL && pagoda::check(0) == -EINVAL && pagoda::waitAll() == -EINVAL);
        REQUIRE(pagoda::shutdown() == -EINVAL);
        std::printf("nodev\n");
        return 0;
    }
    REQUIRE(rc == 0 && gpu);
    REQUIRE(pagoda::init() == -EALREADY);
    std::vector<pagoda_task_t> ids;
    for (int k = 0; k < n; k++) {
        pagoda_mark_args a{out, cnt + k, (uint32_t)(128 * k), (uint32_t)(k + 1)};
        ids.push_back(pagoda::taskSpawn(threads, 1, 0, 0, PAGODA_MARK, a));
        REQUIRE(ids.back() == k);   // ids strictly increasing from 0
    }
    pagoda_gate_args g{flag};
    const pagoda_task_t gated = pagoda::taskSpawn(32, 1, 0, 0, PAGODA_GATE, g);
    REQUIRE(gated == n);
    // tasks complete in any order: wait for the last, then the first, and check it
    REQUIRE(pagoda::wait(ids[n - 1]) == 0 && pagoda::wait(ids[0]) == 0 && pagoda::check(ids[0]) == 1);
    REQUIRE(pagoda::check(gated) == 0);   // still gated
    *flag = 1;
    REQUIRE(pagoda::wait(gated) == 0 && pagoda::check(gated) == 1);
    REQUIRE(pagoda::waitAll() == 0);
    REQUIRE(pagoda::check(gated + 1) == -EINVAL);
    REQUIRE(pagoda::shutdown() == 0);
    std::vector<uint32_t> o(128 * n), c(n);
    REQUIRE(cudaMemcpy(o.data(), out, 4 * 128 * n, cudaMemcpyDeviceToHost) == cudaSuccess);
    REQUIRE(cudaMemcpy(c.data(), cnt, 4 * n, cudaMemcpyDeviceToHost) == cudaSuccess);
    for (int k = 0; k < n; k++) {
        REQUIRE(c[k] == (uint32_t)threads);
        for (int t = 0; t < 128; t++) REQUIRE(o[128 * k + t] == (t < threads ? (uint32_t)(k + 1) : 0u));
    }
    std::printf("ok\n");
    return 0;
}
