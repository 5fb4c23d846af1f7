/*
 * pagoda_device.cuh — device API seen by task bodies (Table 1, §3
 * P:410-418): getTid, syncBlock, getSMPtr, plus small extensions.
 *
 * A task body is a __device__ subroutine templated on an "Env"
 * that supplies these calls.  Inside the MasterKernel the Env is
 * pagoda::TaskEnv, whose values come from the executor warp's WarpTable slot
 * (Table 2); the naive one-kernel-per-task baseline instantiates
 * the same bodies with pagoda::NativeEnv (threadIdx / __syncthreads / dynamic
 * shared memory), so both run identical arithmetic.
 *
 * The paper-named free functions getTid() / syncBlock() / getSMPtr() are also
 * provided for bodies written without an Env: they read the calling warp's
 * WarpTable slot from the MTB's shared memory ("warpId ... is used
 * to generate the threadID in the getTid() function").
 *
 * Contract (same as CUDA's for __syncthreads): every thread of a thread block
 * -- including the idle lanes that pad the block to whole warps -- must call
 * syncBlock() the same number of times, convergently.
 */
#ifndef PAGODA_DEVICE_CUH
#define PAGODA_DEVICE_CUH
#include <stdint.h>

namespace pagoda {

/* One WarpTable slot (Table 2), 32 bytes, written by the scheduler
 * warp before it releases the executor warp (Alg. 2 L9-14 P:846-851). */
struct WarpSlot {
    uint32_t smem_off;    /* byte offset of this TB's shared memory from the MTB's shared-memory base (SMindex) */
    uint32_t smem_bytes;  /* granted bytes (request rounded up to 512) */
    uint16_t tb;          /* thread-block index j within the task */
    uint16_t threads_tb;  /* requested threads per TB */
    uint8_t  task;        /* task slot in the MTB (eNum); 0xFF = terminate */
    uint8_t  warp_in_tb;  /* warp index within the TB */
    uint8_t  warps_tb;    /* warps per TB */
    uint8_t  n_tb;        /* TBs in the task */
    uint8_t  bar_id;      /* named barrier (barId), 0 = none */
    uint8_t  tbslot;      /* per-MTB TB record */
    uint16_t n_tb_all;    /* TBs of the whole task (> n_tb when it is spread over several MTBs) */
    uint64_t task_id;     /* host-visible id (for tracing) */
};
static_assert(sizeof(WarpSlot) == 32, "WarpSlot is 32 bytes");

enum : uint8_t { SLOT_TERMINATE = 0xFF, SLOT_SCHED = 0xFE /* take over the scheduler token */ };

/* Byte offsets inside the MTB's dynamic shared memory (the control block is
 * laid out in csrc/mk_layout.cuh, which static_asserts them).  The task arena
 * follows the control block, or the resident tables when a context has them. */
constexpr uint32_t kWarpTableOffset = 512;
constexpr uint32_t kControlBytes = 6656;            /* arena offset without resident tables (13 granules) */
constexpr uint32_t kResidentOffset = 8192;          /* room reserved for the control block + resident tables */
constexpr uint32_t kResidentTdesBytes = 8 * 64 * 32 * 4;   /* 3DES SP tables, one copy per lane */
constexpr uint32_t kResidentTdesAddr = 8192;        /* shared-WINDOW address of the resident tables: a
                                                       constant, so lookups carry it as an immediate */
constexpr uint32_t kDevErrorPtrOffset = 4736;       /* MtbShared.dev_error: the device error word's address, for
                                                       the paper-named free syncBlock() (which has no TaskEnv) */
constexpr uint32_t kDevErrSyncWithoutFlag = 1u;     /* == PAGODA_DEVERR_SYNC_WITHOUT_FLAG (pagoda.h) */

__device__ __forceinline__ uint32_t lane_id() { return threadIdx.x & 31u; }

__device__ __forceinline__ void named_bar_sync(uint32_t id, uint32_t nthreads)
{
    asm volatile("bar.sync %0, %1;" ::"r"(id), "r"(nthreads) : "memory");
}

__device__ __forceinline__ uint64_t globaltimer_ns()
{
    uint64_t t;
    asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
    return t;
}

__device__ __forceinline__ uint32_t smem_u32(const void* p)
{
    return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

/* ---------------------------------------------------------------- TaskEnv
 * Everything a body asks for is read from the executor warp's WarpTable slot in
 * shared memory when asked (no register holds it across the body). */
constexpr uint32_t kStageBarOffset = 256;     /* per-warp TMA staging mbarriers (MtbShared.stage_bar) */
constexpr uint32_t kStagePhaseOffset = 4608;  /* their parities, one u32 per warp (MtbShared.stage_ph) */

struct TaskEnv {
    uint32_t* dev_error;    /* device error word */
    uint32_t  resident;     /* shared-window address of the MTB-resident 3DES tables, 0 if none */

    static __device__ __forceinline__ unsigned char* mk_smem()
    {   /* the __shared__ symbol itself, so nvcc emits LDS/STS, not generic LD/ST */
        extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
        return pagoda_mk_smem;
    }
    __device__ __forceinline__ const WarpSlot& s() const
    {
        return *reinterpret_cast<const WarpSlot*>(mk_smem() + kWarpTableOffset + (threadIdx.x >> 5) * sizeof(WarpSlot));
    }
    __device__ __forceinline__ int getTid() const
    {
        const WarpSlot& w = s();
        return ((int)w.tb * (int)w.warps_tb + (int)w.warp_in_tb) * 32 + (int)lane_id();
    }
    __device__ __forceinline__ int getBlockIdx() const { return s().tb; }
    __device__ __forceinline__ int getBlockTid() const { return (int)s().warp_in_tb * 32 + (int)lane_id(); }
    __device__ __forceinline__ int getBlockDim() const { return s().threads_tb; }
    __device__ __forceinline__ int getBlockWarps() const { return s().warps_tb; }
    __device__ __forceinline__ int getNumBlocks() const { return s().n_tb_all; }
    __device__ __forceinline__ char* getSMPtr() const { return reinterpret_cast<char*>(mk_smem()) + s().smem_off; }
    __device__ __forceinline__ uint32_t getSMBytes() const { return s().smem_bytes; }
    /* MTB-resident, lane-replicated 3DES SP tables (context flag PAGODA_RESIDENT_TDES) */
    __device__ __forceinline__ uint32_t getResidentTdes() const { return resident; }
    /* true if syncBlock() is legal: a 1-warp TB, or a TB spawned with sync=1 */
    __device__ __forceinline__ bool canSync() const { return s().warps_tb == 1 || s().bar_id != 0; }
    __device__ __forceinline__ void syncBlock() const
    {
        const uint32_t wtb = s().warps_tb, bar = s().bar_id;
        if (wtb == 1) {
            __syncwarp();
        } else if (bar != 0) {
            named_bar_sync(bar, 32u * wtb);
        } else {
            /* spawned with sync=0: contract violation */
            atomicOr(dev_error, kDevErrSyncWithoutFlag);
            __syncwarp();
        }
    }
    /* Warp-collective: bulk-copy `bytes` (multiple of 16, both addresses
     * 16-byte aligned) from global memory into shared memory with the TMA
     * engine (cp.async.bulk ... mbarrier::complete_tx), then wait for it.
     * Other warps of the TB must syncBlock() before reading what this warp staged. */
    __device__ __forceinline__ void stage(void* smem_dst, const void* gsrc, uint32_t bytes) const
    {
        if (bytes == 0) return;
        const uint32_t warp = threadIdx.x >> 5;
        const uint32_t bar = smem_u32(mk_smem() + kStageBarOffset + warp * 8u);
        uint32_t* stage_phase = reinterpret_cast<uint32_t*>(mk_smem() + kStagePhaseOffset + warp * 4u);
        if (lane_id() == 0) {
            asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(bar), "r"(bytes) : "memory");
            asm volatile(
                "cp.async.bulk.shared::cta.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
                    smem_u32(smem_dst)),
                "l"(gsrc), "r"(bytes), "r"(bar)
                : "memory");
        }
        uint32_t ph = *stage_phase, done = 0;
        while (!done) {
            asm volatile(
                "{ .reg .pred p; mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2; selp.u32 %0, 1, 0, p; }"
                : "=r"(done)
                : "r"(bar), "r"(ph)
                : "memory");
        }
        *stage_phase = ph ^ 1u;
        __syncwarp();
    }
};

/* ---------------------------------------------------------------- NativeEnv
 * For the naive baseline: one task = one ordinary kernel launch. */
struct NativeEnv {
    __device__ __forceinline__ int getTid() const { return (int)(blockIdx.x * blockDim.x + threadIdx.x); }
    __device__ __forceinline__ int getBlockIdx() const { return (int)blockIdx.x; }
    __device__ __forceinline__ int getBlockTid() const { return (int)threadIdx.x; }
    __device__ __forceinline__ int getBlockDim() const { return threads_tb; }
    __device__ __forceinline__ int getBlockWarps() const { return (int)(blockDim.x >> 5); }
    __device__ __forceinline__ int getNumBlocks() const { return (int)gridDim.x; }
    __device__ __forceinline__ char* getSMPtr() const
    {
        extern __shared__ __align__(1024) char native_smem[];
        return native_smem;
    }
    __device__ __forceinline__ uint32_t getSMBytes() const { return smem_bytes; }
    __device__ __forceinline__ uint32_t getResidentTdes() const { return 0; }
    __device__ __forceinline__ bool canSync() const { return true; }
    __device__ __forceinline__ void syncBlock() const { __syncthreads(); }
    __device__ __forceinline__ void stage(void* smem_dst, const void* gsrc, uint32_t bytes) const
    {
        /* plain cooperative copy inside the warp */
        const int4* s = reinterpret_cast<const int4*>(gsrc);
        int4* d = reinterpret_cast<int4*>(smem_dst);
        for (uint32_t i = lane_id(); i < bytes / 16u; i += 32u) d[i] = s[i];
        __syncwarp();
    }
    int threads_tb;
    uint32_t smem_bytes;
};

/* ---------------------------------------------------------------- FusedEnv
 * For the static-fusion baseline: all tasks fused into one
 * monolithic kernel, one thread block of a fixed size per (single-TB) task. */
struct FusedEnv {
    __device__ __forceinline__ int getTid() const { return (int)threadIdx.x; }
    __device__ __forceinline__ int getBlockIdx() const { return 0; }
    __device__ __forceinline__ int getBlockTid() const { return (int)threadIdx.x; }
    __device__ __forceinline__ int getBlockDim() const { return (int)blockDim.x; }
    __device__ __forceinline__ int getBlockWarps() const { return (int)(blockDim.x >> 5); }
    __device__ __forceinline__ int getNumBlocks() const { return 1; }
    __device__ __forceinline__ char* getSMPtr() const
    {
        extern __shared__ __align__(1024) char native_smem[];
        return native_smem;
    }
    __device__ __forceinline__ uint32_t getSMBytes() const { return smem_bytes; }
    __device__ __forceinline__ uint32_t getResidentTdes() const { return 0; }
    __device__ __forceinline__ bool canSync() const { return true; }
    __device__ __forceinline__ void syncBlock() const { __syncthreads(); }
    __device__ __forceinline__ void stage(void* smem_dst, const void* gsrc, uint32_t bytes) const
    {
        const int4* s = reinterpret_cast<const int4*>(gsrc);
        int4* d = reinterpret_cast<int4*>(smem_dst);
        for (uint32_t i = lane_id(); i < bytes / 16u; i += 32u) d[i] = s[i];
        __syncwarp();
    }
    uint32_t smem_bytes;
};

} // namespace pagoda

/* ---------------------------------------------------------------- paper API
 * Free functions with the paper's names (Table 1) for bodies that
 * do not take an Env.  Valid only inside a task running on the MasterKernel. */
__device__ __forceinline__ const pagoda::WarpSlot& pagoda_my_slot()
{
    extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
    return reinterpret_cast<const pagoda::WarpSlot*>(pagoda_mk_smem + pagoda::kWarpTableOffset)[threadIdx.x >> 5];
}
__device__ __forceinline__ int getTid()
{
    const pagoda::WarpSlot& s = pagoda_my_slot();
    return ((int)s.tb * (int)s.warps_tb + (int)s.warp_in_tb) * 32 + (int)pagoda::lane_id();
}
__device__ __forceinline__ void syncBlock()
{   /* same semantics as TaskEnv::syncBlock: a multi-warp TB spawned with sync=0 has no barrier ID,
     * which is a contract violation: flag it, later host calls return -EIO */
    extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
    const pagoda::WarpSlot& s = pagoda_my_slot();
    if (s.warps_tb == 1) {
        __syncwarp();
    } else if (s.bar_id != 0) {
        pagoda::named_bar_sync(s.bar_id, 32u * s.warps_tb);
    } else {
        uint32_t* err = *reinterpret_cast<uint32_t* const*>(pagoda_mk_smem + pagoda::kDevErrorPtrOffset);
        atomicOr(err, pagoda::kDevErrSyncWithoutFlag);
        __syncwarp();
    }
}
__device__ __forceinline__ char* getSMPtr()
{
    extern __shared__ __align__(1024) unsigned char pagoda_mk_smem[];
    return reinterpret_cast<char*>(pagoda_mk_smem) + pagoda_my_slot().smem_off;
}

#endif
