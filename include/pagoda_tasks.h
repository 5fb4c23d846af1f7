/*
 * pagoda_tasks.h — the task bodies compiled into the MasterKernel and their
 * argument blocks (device pointers; each block <= PAGODA_ARGS_MAX = 40 bytes,
 * the TaskTable entry's "task inputs" field).
 *
 * Bodies are __device__ subroutines, not __global__ kernels (Fig. 1b
 * "Task Kernels as subroutines" P:343-344).  Definitions of what each computes
 * are DESIGN.md "Task bodies" (the paper names them, Tables 3-4).
 * Every body is correct for any thread count and block count; threads beyond
 * the requested count of a block (warp rounding) are idle but still call
 * syncBlock() convergently.
 */
#ifndef PAGODA_TASKS_H
#define PAGODA_TASKS_H
#include <stdint.h>

enum pagoda_func_id {
    /* runtime test bodies */
    PAGODA_NOP  = 0,   /* no work */
    PAGODA_MARK = 1,   /* out[base+getTid()] = tag for live threads; cnt += live threads */
    PAGODA_TID  = 2,   /* out[base+getTid()] = (getBlockIdx()<<16) | getBlockTid() */
    PAGODA_BAR  = 3,   /* phases of write / syncBlock / read neighbour warp; errors -> err[0] */
    PAGODA_SMEM = 4,   /* fill getSMPtr()[0:bytes], spin, syncBlock, verify; errors -> err[0] */
    PAGODA_SPIN = 5,   /* busy-wait ns (%globaltimer) */
    PAGODA_GATE = 6,   /* spin until *flag != 0 (flag in pinned host memory) */
    PAGODA_HOLD = 7,   /* brute-force schedules: count the warp in *started, fill getSMPtr()[0:grant] with a
                          pattern, hold until *flag != 0, verify the pattern after syncBlock; errors -> err[0] */
    PAGODA_PAPER = 8,  /* written against the paper's free functions only (Table 1: getTid,
                          syncBlock, getSMPtr; no Env): out[base + getTid()] = getTid() + 1 for live threads,
                          syncBlock(), then each thread checks its warp-mate 32 lanes on; errors -> err[0] */
    /* paper benchmarks (Table 3) */
    PAGODA_MB   = 16,  /* Mandelbrot 64x64 tile */
    PAGODA_TDES = 17,  /* 3DES EDE3 ECB over a packet */
    PAGODA_MM   = 18,  /* 32x32x32 fp32 matrix multiply */
    PAGODA_FB   = 19,  /* FilterBank, one channel of 2048 */
    PAGODA_BF   = 20,  /* BeamFormer, 4 ch x 512 complex */
    PAGODA_CONV = 21,  /* separable 17-tap convolution, 128x128 (row pass through args.scratch, 64 KiB per TB) */
    PAGODA_DCT  = 22,  /* 8x8 DCT-II over 128x128 */
    /* variants */
    PAGODA_MM_TC = 23, /* the MM task on the tensor cores: 3xTF32 mma.sync (args: pagoda_mm_args) */
    PAGODA_MM64 = 24   /* Table 4's MatrixMul size: row-major 64x64x64 fp32 (args: pagoda_mm_args);
                          stages A and B (32 KiB) when granted >= 32768 bytes and sync */
};

typedef struct { uint32_t* out; uint32_t* cnt; uint32_t base; uint32_t tag; } pagoda_mark_args;
typedef struct { uint32_t* out; uint32_t base; uint32_t pad; } pagoda_tid_args;
typedef struct { uint32_t* err; uint32_t* scratch; uint32_t phases; uint32_t pad; } pagoda_bar_args;
typedef struct { uint32_t* err; uint32_t bytes; uint32_t spin_ns; uint32_t seed; uint32_t pad; } pagoda_smem_args;
typedef struct { uint64_t ns; } pagoda_spin_args;
typedef struct { const volatile uint32_t* flag; } pagoda_gate_args;
/* flag / started may be pinned host memory (mapped): the host releases and watches the task */
typedef struct { const volatile uint32_t* flag; uint32_t* err; uint32_t* started; uint32_t seed; uint32_t pad; }
    pagoda_hold_args;
typedef struct { uint32_t* out; uint32_t* err; uint32_t base; uint32_t pad; } pagoda_paper_args;

/* MB: pixel (px,py) of tile (tx,ty): c = (x0 + (64tx+px)*dx, y0 + (64ty+py)*dx) */
typedef struct { uint16_t* out; float x0, y0, dx; int32_t tx, ty, maxit; } pagoda_mb_args;
/* TDES: nblk 8-byte blocks in -> out; tables from pagoda_tdes_tables() in device memory */
typedef struct { const uint64_t* in; uint64_t* out; const uint32_t* tables; uint32_t nblk; uint32_t pad; } pagoda_tdes_args;
/* MM: row-major 32x32 fp32 */
typedef struct { const float* A; const float* B; float* C; } pagoda_mm_args;
/* FB: r[2048], H[32], F[32] -> y[2048]; scratch: 1 KiB device scratch used when the shmem grant is < 1 KiB */
typedef struct { const float* r; const float* H; const float* F; float* y; float* scratch; } pagoda_fb_args;
/* BF: x[4][512] complex, h[4][16] complex, w[4 beams][4 ch] complex -> out[4][512] power */
typedef struct { const float* x; const float* h; const float* w; float* out; } pagoda_bf_args;
/* CONV: img[128][128], krow[17], kcol[17] -> out[128][128]; scratch: 64 KiB row-pass buffer */
typedef struct { const float* img; const float* krow; const float* kcol; float* out; float* scratch; } pagoda_conv_args;
/* DCT: img[128][128], coef[8][8] (C[u][x]) -> out[128][128] */
typedef struct { const float* img; const float* coef; float* out; } pagoda_dct_args;

#endif
