/*
 * oracle.h — TEST INFRASTRUCTURE ONLY.  The plain, slow, sequential CPU
 * definition of what the Pagoda hot path computes (Yeh et al., PPoPP'17,
 * /root/reference/PAPER.md, cited as P:<line>).  Only tests/, __graft_entry__.smoke()
 * and bench.py's cpu_baseline / --impl reference legs may load it.  It shares no
 * code, header, table or constant with the CUDA product (paper_conf_ppopp_yehsser17_b200/,
 * include/); the product never calls it.
 *
 * What the method computes: running every spawned task's body
 * exactly once, independently.  So the oracle API runs each body EAGERLY at
 * spawn time, in spawn order; wait/check/waitAll are then trivial.
 *
 * Precision: the paper states none; BASELINE.json's north
 * star fixes "fp32 tasks", and the body definitions (restated in
 * DESIGN.md "Readings") fix the fp32 operation order (fmaf where the definition
 * says fma, no contraction elsewhere: build with -ffp-contract=off).  Every
 * fp32 body is pinned in tests/ against fp64 library routines / closed forms
 * within the textbook error bound; error bounds alone cannot tell fmaf from
 * mul+add or one summation order from another, so each fp32 body also has a
 * hand-derived closed-form pin whose exact value exists only under the defined
 * order (tests/test_oracle_bodies.py "fma / order pins": one cancelling step
 * gives 2^-24 fused and in order, 0 unfused or reordered).  MB, defined
 * without fma, is pinned by the whole-config checksum of an independent numpy
 * emulation (scripts/gen_mandelbrot_pins.py), which a contracted build misses.
 */
#ifndef PAGODA_ORACLE_H
#define PAGODA_ORACLE_H
#include <stddef.h>
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

/* ---- task function ids (the oracle's own numbering; the harness maps by name) */
enum {
    ORC_NOP = 0, ORC_MARK = 1, ORC_TID = 2,
    ORC_MB = 16, ORC_TDES = 17, ORC_MM = 18, ORC_FB = 19, ORC_BF = 20,
    ORC_CONV = 21, ORC_DCT = 22, ORC_MM_TC = 23
};

/* ---- per-body argument blocks (host pointers; each <= 40 bytes) */
typedef struct { uint16_t* out; float x0, y0, dx; int32_t tx, ty, maxit; } orc_mb_args;
typedef struct { const uint8_t* in; uint8_t* out; const uint8_t* key24; uint32_t nbytes; } orc_tdes_args;
typedef struct { const float* A; const float* B; float* C; } orc_mm_args;
typedef struct { const float* r; const float* H; const float* F; float* y; } orc_fb_args;
typedef struct { const float* x; const float* h; const float* w; float* out; } orc_bf_args;
typedef struct { const float* img; const float* krow; const float* kcol; float* out; } orc_conv_args;
typedef struct { const float* img; const float* coef; float* out; } orc_dct_args;
typedef struct { uint32_t* out; uint32_t* cnt; uint32_t base; uint32_t tag; } orc_mark_args;
typedef struct { uint32_t* out; uint32_t base; } orc_tid_args;

/* ---- bodies (one task each) */
void orc_mandelbrot_tile(uint16_t* out, float x0, float y0, float dx, int tx, int ty, int maxit);
void orc_des_key_schedule(const uint8_t key8[8], uint64_t subkeys[16]);
uint64_t orc_des_block(uint64_t block, const uint64_t subkeys[16], int decrypt);
void orc_tdes_ecb(const uint8_t* in, uint8_t* out, size_t nbytes, const uint8_t key24[24], int decrypt);
void orc_mm32(const float* A, const float* B, float* C);
void orc_mm64(const float* A, const float* B, float* C);       /* Table 4's 64x64 size (NEXT-4) */
void orc_mm32_f64(const float* A, const float* B, float* C);   /* exact product, one rounding (NEXT-4) */
void orc_filterbank(const float* r, const float* H, const float* F, float* y);
void orc_beamformer(const float* x, const float* h, const float* w, float* out);
void orc_conv(const float* img, const float* krow, const float* kcol, float* out);
void orc_dct(const float* img, const float* coef, float* out);

/* ---- the Table 1 host API, sequential */
typedef struct orc_ctx orc_ctx;
int     orc_init(int exec_warps_per_mtb, int arena_bytes, orc_ctx** out);
int64_t orc_taskSpawn(orc_ctx* c, int threads, int n_tb, int shmem_bytes, int sync_flag,
                      int func_id, const void* args, size_t args_bytes);
int     orc_wait(orc_ctx* c, int64_t id);
int     orc_check(orc_ctx* c, int64_t id);
int     orc_waitAll(orc_ctx* c);
int     orc_shutdown(orc_ctx* c);
void    orc_destroy(orc_ctx* c);

/* ---- occupancy metric: resident warps / (64 * n_sm), in percent */
double  orc_occupancy_pct(int resident_warps, int n_sm);

/* ---- trace-ledger checker (SURVEY §8(c) "Trace-ledger format and checker").
 * Replays per-MTB scheduler events in seq order and checks the allocator
 * invariants.  Returns 0 if every invariant holds, else a negative code and
 * writes a message into err (err_len bytes). */
typedef struct {
    uint32_t seq;        /* per-MTB logical clock */
    uint16_t mtb;
    uint8_t  kind;       /* 1 = ALLOC, 2 = FREE_WARPS, 3 = FREE_TB */
    uint8_t  bar_id;     /* 0 = none */
    uint64_t task_id;
    uint32_t warp_mask;  /* executor warps of this TB */
    uint16_t tb;
    uint16_t gran_off;
    uint16_t gran_len;
    uint16_t pad;
    uint32_t pad2;
} orc_ledger_event;      /* 32 bytes */

typedef struct { uint64_t task_id; uint32_t warps_total; uint32_t n_tb; } orc_ledger_task;

int orc_ledger_check(const orc_ledger_event* ev, size_t n_ev, int n_mtb, int exec_warps,
                     int arena_granules, int n_bar_ids, const orc_ledger_task* tasks,
                     size_t n_tasks, char* err, size_t err_len);

/* ---- executor-interval and completion checker (SURVEY §8(c) invariants 2-4:
 * "a warp never runs two tasks at once", "exactly one completion record, and it
 * comes after the last t_end of its warps").  One record per (task, TB, warp)
 * that ran, with %globaltimer start/end; one completion record per task with
 * the time it was posted to the host.  Cross-checked against the ledger: every
 * executed warp must lie in its TB's ALLOC mask on the same MTB (Alg. 2 L9-12,
 * P:846-851), every allocated warp must have run once (Alg. 1 L29-33,
 * P:781-785), and a task completes only after all its warps ended (Alg. 1
 * L41-43).  Returns 0 or a negative code with a message in err. */
typedef struct {
    uint64_t task_id;
    uint16_t tb;
    uint16_t smid;       /* informational */
    uint16_t mtb;
    uint16_t warp;
    uint64_t t_start, t_end;
} orc_exec_record;       /* 32 bytes */

typedef struct { uint64_t task_id; uint64_t t_done; } orc_completion;   /* 16 bytes */

int orc_exec_check(const orc_ledger_event* ev, size_t n_ev, const orc_exec_record* ex, size_t n_ex,
                   const orc_completion* comp, size_t n_comp, const orc_ledger_task* tasks,
                   size_t n_tasks, char* err, size_t err_len);

#ifdef __cplusplus
}
#endif
#endif
