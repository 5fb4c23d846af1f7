/*
 * pagoda.hpp — the paper's host API under its own names (Table 1 P:120-131,
 * §3): taskSpawn / wait / check / waitAll, for C++ callers.
 *
 * The C ABI (pagoda.h) prefixes every symbol with `pagoda_` because the bare
 * names wait/check would collide with POSIX wait(2).  Here they
 * live in namespace pagoda instead, over one process-wide DEFAULT context, so a
 * program reads like the paper's Fig. 1a:
 *
 *     pagoda::init();                                   // MasterKernel starts
 *     pagoda_task_t t = pagoda::taskSpawn(128, 1, 0, 0, PAGODA_MB, &args, sizeof args);
 *     pagoda::wait(t);                                  // or pagoda::check(t) / pagoda::waitAll()
 *     pagoda::shutdown();
 *
 * Header-only: every function forwards to the C ABI with the same argument
 * meaning, layout, ownership and error codes (negative errno; see pagoda.h).
 * No exceptions.  Thread-safe like the C calls; init / shutdown must not race
 * other calls.
 */
#ifndef PAGODA_HPP
#define PAGODA_HPP
#include <errno.h>

#include "pagoda.h"
#include "pagoda_tasks.h"

namespace pagoda {

/* The default context used by the paper-named calls (nullptr before init / after shutdown). */
inline pagoda_ctx*& default_context()
{
    static pagoda_ctx* ctx = nullptr;
    return ctx;
}

/* Start the default context (cfg nullptr = pagoda_config_default).  Returns 0,
 * -EALREADY if it exists, or pagoda_init's error (-ENODEV without an sm_100 GPU). */
inline int init(const pagoda_config* cfg = nullptr)
{
    if (default_context()) return -EALREADY;
    pagoda_ctx* c = nullptr;
    const int rc = pagoda_init(cfg, &c);
    if (rc == 0) default_context() = c;
    return rc;
}

/* taskSpawn (Table 1): see pagoda_taskSpawn.  -EINVAL before init. */
inline pagoda_task_t taskSpawn(int threads, int n_threadblocks, int shmem_bytes, int sync_flag, int func_id,
                               const void* args, size_t args_bytes)
{
    pagoda_ctx* c = default_context();
    return c ? pagoda_taskSpawn(c, threads, n_threadblocks, shmem_bytes, sync_flag, func_id, args, args_bytes)
             : (pagoda_task_t)-EINVAL;
}

/* Typed convenience: args is one of the pagoda_*_args blocks of pagoda_tasks.h. */
template <class Args>
inline pagoda_task_t taskSpawn(int threads, int n_threadblocks, int shmem_bytes, int sync_flag, int func_id,
                               const Args& args)
{
    static_assert(sizeof(Args) <= PAGODA_ARGS_MAX, "task arguments are at most 40 bytes (P:502-508)");
    return taskSpawn(threads, n_threadblocks, shmem_bytes, sync_flag, func_id, &args, sizeof(Args));
}

/* wait (Table 1): block until task id is done; 0 or -errno. */
inline int wait(pagoda_task_t id)
{
    pagoda_ctx* c = default_context();
    return c ? pagoda_wait(c, id) : -EINVAL;
}

/* check (Table 1): non-blocking; 1 done, 0 pending, -errno. */
inline int check(pagoda_task_t id)
{
    pagoda_ctx* c = default_context();
    return c ? pagoda_check(c, id) : -EINVAL;
}

/* waitAll (Table 1): every task spawned before the call is done; 0 or -errno. */
inline int waitAll()
{
    pagoda_ctx* c = default_context();
    return c ? pagoda_waitAll(c) : -EINVAL;
}

/* waitAll, stop the MasterKernel and free the default context. */
inline int shutdown()
{
    pagoda_ctx* c = default_context();
    if (!c) return -EINVAL;
    default_context() = nullptr;
    return pagoda_shutdown(c);
}

}  // namespace pagoda
#endif
