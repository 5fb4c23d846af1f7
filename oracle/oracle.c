/*
 * oracle.c — TEST INFRASTRUCTURE ONLY (see oracle.h).  Plain C11, built with
 * -O2 -ffp-contract=off: every fp32 operation is rounded on its own, fmaf()
 * appears exactly where the body definition says "fma".  No blocking, no
 * reordering, no SIMD tricks: each function is its definition written out.
 *
 * Citations: P:<line> = /root/reference/PAPER.md; §8(c) = SURVEY.md §8(c),
 * whose body definitions DESIGN.md "Readings" restates (the paper gives names,
 * sources and sizes only, Tables 3-4).
 */
#include "oracle.h"

#include <errno.h>
#include <math.h>
#include <stdio.h>
#include <stdlib.h>
#include <string.h>

/* ======================================================================
 * MB — Mandelbrot tile (Table 3, Table 4; the
 * iteration rule, region and escape test are §8(c)'s reading: strict '>',
 * count includes the escaping step, no contraction).
 * ==================================================================== */
void orc_mandelbrot_tile(uint16_t* out, float x0, float y0, float dx, int tx, int ty, int maxit)
{
    for (int py = 0; py < 64; py++) {
        for (int px = 0; px < 64; px++) {
            int gx = 64 * tx + px, gy = 64 * ty + py;
            float cr = x0 + (float)gx * dx;
            float ci = y0 + (float)gy * dx;
            float zr = 0.0f, zi = 0.0f;
            int n = 0;
            while (n < maxit) {
                float zr2 = zr * zr;
                float zi2 = zi * zi;
                if (zr2 + zi2 > 4.0f) break;
                float t = zr + zr;
                zi = t * zi + ci;        /* a multiply, then an add: never fused */
                zr = (zr2 - zi2) + cr;
                n++;
            }
            out[py * 64 + px] = (uint16_t)n;
        }
    }
}

/* ======================================================================
 * 3DES — TDEA EDE3 in ECB over the packet (Table 3 P:1046-1047 cites NIST
 * FIPS 46-3 [5]).  Textbook DES: every permutation is applied
 * bit by bit from the FIPS 46-3 tables (bit 1 = most significant bit).
 * ==================================================================== */
static const uint8_t IP[64] = {
    58, 50, 42, 34, 26, 18, 10, 2, 60, 52, 44, 36, 28, 20, 12, 4,
    62, 54, 46, 38, 30, 22, 14, 6, 64, 56, 48, 40, 32, 24, 16, 8,
    57, 49, 41, 33, 25, 17, 9,  1, 59, 51, 43, 35, 27, 19, 11, 3,
    61, 53, 45, 37, 29, 21, 13, 5, 63, 55, 47, 39, 31, 23, 15, 7};
static const uint8_t FP[64] = {
    40, 8, 48, 16, 56, 24, 64, 32, 39, 7, 47, 15, 55, 23, 63, 31,
    38, 6, 46, 14, 54, 22, 62, 30, 37, 5, 45, 13, 53, 21, 61, 29,
    36, 4, 44, 12, 52, 20, 60, 28, 35, 3, 43, 11, 51, 19, 59, 27,
    34, 2, 42, 10, 50, 18, 58, 26, 33, 1, 41, 9,  49, 17, 57, 25};
static const uint8_t E[48] = {
    32, 1,  2,  3,  4,  5,  4,  5,  6,  7,  8,  9,  8,  9,  10, 11,
    12, 13, 12, 13, 14, 15, 16, 17, 16, 17, 18, 19, 20, 21, 20, 21,
    22, 23, 24, 25, 24, 25, 26, 27, 28, 29, 28, 29, 30, 31, 32, 1};
static const uint8_t P[32] = {
    16, 7, 20, 21, 29, 12, 28, 17, 1,  15, 23, 26, 5,  18, 31, 10,
    2,  8, 24, 14, 32, 27, 3,  9,  19, 13, 30, 6,  22, 11, 4,  25};
static const uint8_t PC1[56] = {
    57, 49, 41, 33, 25, 17, 9,  1,  58, 50, 42, 34, 26, 18,
    10, 2,  59, 51, 43, 35, 27, 19, 11, 3,  60, 52, 44, 36,
    63, 55, 47, 39, 31, 23, 15, 7,  62, 54, 46, 38, 30, 22,
    14, 6,  61, 53, 45, 37, 29, 21, 13, 5,  28, 20, 12, 4};
static const uint8_t PC2[48] = {
    14, 17, 11, 24, 1,  5,  3,  28, 15, 6,  21, 10,
    23, 19, 12, 4,  26, 8,  16, 7,  27, 20, 13, 2,
    41, 52, 31, 37, 47, 55, 30, 40, 51, 45, 33, 48,
    44, 49, 39, 56, 34, 53, 46, 42, 50, 36, 29, 32};
static const uint8_t SHIFTS[16] = {1, 1, 2, 2, 2, 2, 2, 2, 1, 2, 2, 2, 2, 2, 2, 1};
static const uint8_t S[8][4][16] = {
    {{14, 4, 13, 1, 2, 15, 11, 8, 3, 10, 6, 12, 5, 9, 0, 7},
     {0, 15, 7, 4, 14, 2, 13, 1, 10, 6, 12, 11, 9, 5, 3, 8},
     {4, 1, 14, 8, 13, 6, 2, 11, 15, 12, 9, 7, 3, 10, 5, 0},
     {15, 12, 8, 2, 4, 9, 1, 7, 5, 11, 3, 14, 10, 0, 6, 13}},
    {{15, 1, 8, 14, 6, 11, 3, 4, 9, 7, 2, 13, 12, 0, 5, 10},
     {3, 13, 4, 7, 15, 2, 8, 14, 12, 0, 1, 10, 6, 9, 11, 5},
     {0, 14, 7, 11, 10, 4, 13, 1, 5, 8, 12, 6, 9, 3, 2, 15},
     {13, 8, 10, 1, 3, 15, 4, 2, 11, 6, 7, 12, 0, 5, 14, 9}},
    {{10, 0, 9, 14, 6, 3, 15, 5, 1, 13, 12, 7, 11, 4, 2, 8},
     {13, 7, 0, 9, 3, 4, 6, 10, 2, 8, 5, 14, 12, 11, 15, 1},
     {13, 6, 4, 9, 8, 15, 3, 0, 11, 1, 2, 12, 5, 10, 14, 7},
     {1, 10, 13, 0, 6, 9, 8, 7, 4, 15, 14, 3, 11, 5, 2, 12}},
    {{7, 13, 14, 3, 0, 6, 9, 10, 1, 2, 8, 5, 11, 12, 4, 15},
     {13, 8, 11, 5, 6, 15, 0, 3, 4, 7, 2, 12, 1, 10, 14, 9},
     {10, 6, 9, 0, 12, 11, 7, 13, 15, 1, 3, 14, 5, 2, 8, 4},
     {3, 15, 0, 6, 10, 1, 13, 8, 9, 4, 5, 11, 12, 7, 2, 14}},
    {{2, 12, 4, 1, 7, 10, 11, 6, 8, 5, 3, 15, 13, 0, 14, 9},
     {14, 11, 2, 12, 4, 7, 13, 1, 5, 0, 15, 10, 3, 9, 8, 6},
     {4, 2, 1, 11, 10, 13, 7, 8, 15, 9, 12, 5, 6, 3, 0, 14},
     {11, 8, 12, 7, 1, 14, 2, 13, 6, 15, 0, 9, 10, 4, 5, 3}},
    {{12, 1, 10, 15, 9, 2, 6, 8, 0, 13, 3, 4, 14, 7, 5, 11},
     {10, 15, 4, 2, 7, 12, 9, 5, 6, 1, 13, 14, 0, 11, 3, 8},
     {9, 14, 15, 5, 2, 8, 12, 3, 7, 0, 4, 10, 1, 13, 11, 6},
     {4, 3, 2, 12, 9, 5, 15, 10, 11, 14, 1, 7, 6, 0, 8, 13}},
    {{4, 11, 2, 14, 15, 0, 8, 13, 3, 12, 9, 7, 5, 10, 6, 1},
     {13, 0, 11, 7, 4, 9, 1, 10, 14, 3, 5, 12, 2, 15, 8, 6},
     {1, 4, 11, 13, 12, 3, 7, 14, 10, 15, 6, 8, 0, 5, 9, 2},
     {6, 11, 13, 8, 1, 4, 10, 7, 9, 5, 0, 15, 14, 2, 3, 12}},
    {{13, 2, 8, 4, 6, 15, 11, 1, 10, 9, 3, 14, 5, 0, 12, 7},
     {1, 15, 13, 8, 10, 3, 7, 4, 12, 5, 6, 11, 0, 14, 9, 2},
     {7, 11, 4, 1, 9, 12, 14, 2, 0, 6, 10, 13, 15, 3, 5, 8},
     {2, 1, 14, 7, 4, 10, 8, 13, 15, 12, 9, 0, 3, 5, 6, 11}}};

/* out bit i (1-based, MSB first) = in bit tab[i-1] of an in_bits-wide word */
static uint64_t permute(uint64_t in, int in_bits, const uint8_t* tab, int out_bits)
{
    uint64_t out = 0;
    for (int i = 0; i < out_bits; i++)
        out = (out << 1) | ((in >> (in_bits - tab[i])) & 1u);
    return out;
}

void orc_des_key_schedule(const uint8_t key8[8], uint64_t subkeys[16])
{
    uint64_t k = 0;
    for (int i = 0; i < 8; i++) k = (k << 8) | key8[i];
    uint64_t cd = permute(k, 64, PC1, 56);
    uint32_t c = (uint32_t)(cd >> 28) & 0x0FFFFFFFu, d = (uint32_t)cd & 0x0FFFFFFFu;
    for (int r = 0; r < 16; r++) {
        for (int s = 0; s < SHIFTS[r]; s++) {
            c = ((c << 1) | (c >> 27)) & 0x0FFFFFFFu;
            d = ((d << 1) | (d >> 27)) & 0x0FFFFFFFu;
        }
        subkeys[r] = permute(((uint64_t)c << 28) | d, 56, PC2, 48);
    }
}

static uint32_t des_f(uint32_t r, uint64_t k48)
{
    uint64_t e = permute(r, 32, E, 48) ^ k48;
    uint32_t s = 0;
    for (int j = 0; j < 8; j++) {
        unsigned six = (unsigned)(e >> (42 - 6 * j)) & 63u;
        unsigned row = ((six >> 5) << 1) | (six & 1u);
        unsigned col = (six >> 1) & 15u;
        s = (s << 4) | S[j][row][col];
    }
    return (uint32_t)permute(s, 32, P, 32);
}

uint64_t orc_des_block(uint64_t block, const uint64_t subkeys[16], int decrypt)
{
    uint64_t ip = permute(block, 64, IP, 64);
    uint32_t l = (uint32_t)(ip >> 32), r = (uint32_t)ip;
    for (int i = 0; i < 16; i++) {
        uint32_t nl = r;
        r = l ^ des_f(r, subkeys[decrypt ? 15 - i : i]);
        l = nl;
    }
    return permute(((uint64_t)r << 32) | l, 64, FP, 64);
}

void orc_tdes_ecb(const uint8_t* in, uint8_t* out, size_t nbytes, const uint8_t key24[24], int decrypt)
{
    uint64_t k1[16], k2[16], k3[16];
    orc_des_key_schedule(key24, k1);
    orc_des_key_schedule(key24 + 8, k2);
    orc_des_key_schedule(key24 + 16, k3);
    for (size_t b = 0; b + 8 <= nbytes; b += 8) {
        uint64_t x = 0;
        for (int i = 0; i < 8; i++) x = (x << 8) | in[b + i];     /* big-endian block */
        if (!decrypt)   /* EDE3: C = E_K3(D_K2(E_K1(P))) */
            x = orc_des_block(orc_des_block(orc_des_block(x, k1, 0), k2, 1), k3, 0);
        else            /* P = D_K1(E_K2(D_K3(C))) */
            x = orc_des_block(orc_des_block(orc_des_block(x, k3, 1), k2, 0), k1, 1);
        for (int i = 7; i >= 0; i--) { out[b + i] = (uint8_t)x; x >>= 8; }
    }
}

/* ======================================================================
 * MM — 32x32x32 fp32 (Table 3 P:1041-1042 "MatrixMul", CUDA SDK [22];
 * BASELINE.json config 3 fixes 32^3): C[i][j] = fma-chain over k ascending.
 * ==================================================================== */
void orc_mm32(const float* A, const float* B, float* C)
{
    for (int i = 0; i < 32; i++)
        for (int j = 0; j < 32; j++) {
            float acc = 0.0f;
            for (int k = 0; k < 32; k++) acc = fmaf(A[i * 32 + k], B[k * 32 + j], acc);
            C[i * 32 + j] = acc;
        }
}

/* MM 64x64x64 fp32: Table 4's "MatrixMul ... 64 x 64 matrix" (SURVEY §8(f)
 * NEXT-4): the same definition at n = 64, C[i][j] = fma-chain over k ascending. */
void orc_mm64(const float* A, const float* B, float* C)
{
    for (int i = 0; i < 64; i++)
        for (int j = 0; j < 64; j++) {
            float acc = 0.0f;
            for (int k = 0; k < 64; k++) acc = fmaf(A[i * 64 + k], B[k * 64 + j], acc);
            C[i * 64 + j] = acc;
        }
}

/* MM on the tensor cores: the same product C = A B,
 * whose summation order the hardware picks; the definition is the exact
 * product, here accumulated in fp64 (each fp32 x fp32 product is exact in
 * fp64) and rounded once to fp32.  Parity: |g - o| <= 1e-5 sum_k |a_ik b_kj|. */
void orc_mm32_f64(const float* A, const float* B, float* C)
{
    for (int i = 0; i < 32; i++)
        for (int j = 0; j < 32; j++) {
            double acc = 0.0;
            for (int k = 0; k < 32; k++) acc += (double)A[i * 32 + k] * (double)B[k * 32 + j];
            C[i * 32 + j] = (float)acc;
        }
}

/* ======================================================================
 * FB — FilterBank, Fig. 1c made precise (§8(c) FB): one channel,
 * N_sim=2048, N_col=32, N_samp=8.  Causal convolution (guard read as >= 0),
 * buffers initialised to 0, down-sample VD[m]=VH[8m], up-sample VU[8m]=VD[m].
 * ==================================================================== */
void orc_filterbank(const float* r, const float* H, const float* F, float* y)
{
    enum { NSIM = 2048, NCOL = 32, NSAMP = 8 };
    float VH[NSIM], VD[NSIM / NSAMP], VU[NSIM];
    for (int j = 0; j < NSIM; j++) {                 /* convolve H */
        float acc = 0.0f;
        for (int k = 0; k < NCOL && k <= j; k++) acc = fmaf(H[k], r[j - k], acc);
        VH[j] = acc;
    }
    for (int m = 0; m < NSIM / NSAMP; m++) VD[m] = VH[m * NSAMP];          /* down-sample */
    for (int j = 0; j < NSIM; j++) VU[j] = (j % NSAMP == 0) ? VD[j / NSAMP] : 0.0f;  /* up-sample */
    for (int j = 0; j < NSIM; j++) {                 /* convolve F */
        float acc = 0.0f;
        for (int k = 0; k < NCOL && k <= j; k++) acc = fmaf(F[k], VU[j - k], acc);
        y[j] = acc;
    }
}

/* ======================================================================
 * BF — BeamFormer (Table 3; §8(c) BF): 4 channels x 512 complex
 * samples, 16-tap complex FIR per channel, 4 beams of complex weights,
 * output power.  Complex MAC order: re=fma(a.re,b.re,re); re=fma(-a.im,b.im,re);
 * im=fma(a.re,b.im,im); im=fma(a.im,b.re,im).  Complex values are (re, im) pairs.
 * ==================================================================== */
static void cmac(float* re, float* im, const float* a, const float* b)
{
    *re = fmaf(a[0], b[0], *re);
    *re = fmaf(-a[1], b[1], *re);
    *im = fmaf(a[0], b[1], *im);
    *im = fmaf(a[1], b[0], *im);
}

void orc_beamformer(const float* x, const float* h, const float* w, float* out)
{
    enum { NCH = 4, NT = 512, L = 16, NB = 4 };
    float v[NCH][NT][2];
    for (int c = 0; c < NCH; c++)
        for (int t = 0; t < NT; t++) {
            float re = 0.0f, im = 0.0f;
            for (int k = 0; k < L && k <= t; k++)
                cmac(&re, &im, &h[(c * L + k) * 2], &x[(c * NT + (t - k)) * 2]);
            v[c][t][0] = re;
            v[c][t][1] = im;
        }
    for (int b = 0; b < NB; b++)
        for (int t = 0; t < NT; t++) {
            float re = 0.0f, im = 0.0f;
            for (int c = 0; c < NCH; c++) cmac(&re, &im, &w[(b * NCH + c) * 2], v[c][t]);
            out[b * NT + t] = fmaf(re, re, im * im);
        }
}

/* ======================================================================
 * CONV — separable convolution, CUDA SDK [19] (Table 3 P:1037-1038,
 * P:1734-1737), 128x128, radius 8 (17 taps), zero outside the image, the SDK
 * CPU form tmp[y][x] = sum_d img[y][x+d]*krow[8-d], then the column pass.
 * ==================================================================== */
void orc_conv(const float* img, const float* krow, const float* kcol, float* out)
{
    enum { N = 128, R = 8 };
    float tmp[N * N];
    for (int y = 0; y < N; y++)
        for (int x = 0; x < N; x++) {
            float acc = 0.0f;
            for (int d = -R; d <= R; d++)
                if (x + d >= 0 && x + d < N) acc = fmaf(img[y * N + x + d], krow[R - d], acc);
            tmp[y * N + x] = acc;
        }
    for (int y = 0; y < N; y++)
        for (int x = 0; x < N; x++) {
            float acc = 0.0f;
            for (int d = -R; d <= R; d++)
                if (y + d >= 0 && y + d < N) acc = fmaf(tmp[(y + d) * N + x], kcol[R - d], acc);
            out[y * N + x] = acc;
        }
}

/* ======================================================================
 * DCT — 8x8 DCT-II over a 128x128 image, CUDA SDK [21] (Table 3):
 * per block Y = C X C^T with T[u][y] = sum_x C[u][x] X[x][y] (x ascending),
 * Y[u][v] = sum_y T[u][y] C[v][y] (y ascending).  C is an input (fp32).
 * ==================================================================== */
void orc_dct(const float* img, const float* coef, float* out)
{
    enum { N = 128 };
    for (int by = 0; by < N / 8; by++)
        for (int bx = 0; bx < N / 8; bx++) {
            float T[8][8];
            for (int u = 0; u < 8; u++)
                for (int y = 0; y < 8; y++) {
                    float acc = 0.0f;
                    for (int x = 0; x < 8; x++)
                        acc = fmaf(coef[u * 8 + x], img[(by * 8 + x) * N + bx * 8 + y], acc);
                    T[u][y] = acc;
                }
            for (int u = 0; u < 8; u++)
                for (int v = 0; v < 8; v++) {
                    float acc = 0.0f;
                    for (int y = 0; y < 8; y++) acc = fmaf(T[u][y], coef[v * 8 + y], acc);
                    out[(by * 8 + u) * N + bx * 8 + v] = acc;
                }
        }
}

/* ======================================================================
 * Host API (Table 1; §3), sequential.
 * Validation table = SURVEY §8(b) "Validation": all warps of a task live in
 * one MTB, shared memory <= the MTB arena (§5.1), and
 * barrier IDs are a pool of 16 per MTB with ID 0 reserved.
 * ==================================================================== */
struct orc_ctx {
    int exec_warps, arena_bytes, shut;
    int64_t next_id;
};

#define ORC_ARGS_MAX 40
#define ORC_GRANULE 512   /* §5.1: the smallest allocation is 512 B */
#define ORC_BAR_IDS 15    /* 16 named barriers, ID 0 kept for the MTB itself */
#define ORC_MAX_SPREAD 16384   /* MTB entries of one task: a quarter of the default 65536-entry ring */

int orc_init(int exec_warps_per_mtb, int arena_bytes, orc_ctx** out)
{
    if (!out || exec_warps_per_mtb < 1 || exec_warps_per_mtb > 32 || arena_bytes < 0) return -EINVAL;
    orc_ctx* c = (orc_ctx*)calloc(1, sizeof *c);
    if (!c) return -ENOMEM;
    c->exec_warps = exec_warps_per_mtb;
    c->arena_bytes = arena_bytes;
    *out = c;
    return 0;
}

static int known_func(int f)
{
    switch (f) {
    case ORC_NOP: case ORC_MARK: case ORC_TID: case ORC_MB: case ORC_TDES: case ORC_MM:
    case ORC_FB: case ORC_BF: case ORC_CONV: case ORC_DCT: case ORC_MM_TC: return 1;
    default: return 0;
    }
}

static size_t args_size(int f)
{
    switch (f) {
    case ORC_NOP: return 0;
    case ORC_MARK: return sizeof(orc_mark_args);
    case ORC_TID: return sizeof(orc_tid_args);
    case ORC_MB: return sizeof(orc_mb_args);
    case ORC_TDES: return sizeof(orc_tdes_args);
    case ORC_MM: case ORC_MM_TC: return sizeof(orc_mm_args);
    case ORC_FB: return sizeof(orc_fb_args);
    case ORC_BF: return sizeof(orc_bf_args);
    case ORC_CONV: return sizeof(orc_conv_args);
    case ORC_DCT: return sizeof(orc_dct_args);
    default: return 0;
    }
}

int64_t orc_taskSpawn(orc_ctx* c, int threads, int n_tb, int shmem_bytes, int sync_flag,
                      int func_id, const void* args, size_t args_bytes)
{
    if (!c) return -EINVAL;
    if (c->shut) return -ESHUTDOWN;
    if (threads < 1 || threads > 1024 || n_tb < 1 || shmem_bytes < 0) return -EINVAL;
    /* Every thread block must fit one MTB.  The paper keeps all warps of a task in one MTB
     * yet runs "64K threads" per task (Fig. 8); read: a task whose
     * TBs do not fit one MTB is spread, TB by TB, over k = ceil(n_tb / cap) MTB entries, cap =
     * the TBs one MTB hosts (warps, shared memory, 15 barrier IDs when it syncs), and it
     * consumes k task ids, the first being its id (DESIGN.md "Readings" 6). */
    int warps_tb = (threads + 31) / 32;
    if (warps_tb > c->exec_warps) return -EINVAL;
    long gran_tb = (shmem_bytes + ORC_GRANULE - 1) / ORC_GRANULE;
    if (gran_tb * ORC_GRANULE > c->arena_bytes) return -EINVAL;
    long cap = c->exec_warps / warps_tb;
    if (gran_tb && c->arena_bytes / (gran_tb * ORC_GRANULE) < cap) cap = c->arena_bytes / (gran_tb * ORC_GRANULE);
    if (sync_flag && warps_tb > 1 && cap > ORC_BAR_IDS) cap = ORC_BAR_IDS;
    const long k = (n_tb + cap - 1) / cap;
    if (k > 1 && (n_tb > 65535 || k > ORC_MAX_SPREAD)) return -EINVAL;
    if (!known_func(func_id)) return -EINVAL;
    if (args_bytes > ORC_ARGS_MAX || (args_bytes > 0 && !args)) return -EINVAL;
    if (args_bytes < args_size(func_id)) return -EINVAL;

    int64_t id = c->next_id;
    c->next_id += k;
    long total_threads_rounded = (long)warps_tb * 32 * n_tb;
    switch (func_id) {
    case ORC_NOP: break;
    case ORC_MARK: {   /* every live thread t: out[base+t] = tag, cnt += 1 */
        const orc_mark_args* a = (const orc_mark_args*)args;
        for (int b = 0; b < n_tb; b++)
            for (int t = 0; t < threads; t++) {
                a->out[a->base + (uint32_t)(b * warps_tb * 32 + t)] = a->tag;
                a->cnt[0] += 1;
            }
        (void)total_threads_rounded;
        break;
    }
    case ORC_TID: {    /* out[base + getTid()] = (blockIdx << 16) | blockTid */
        const orc_tid_args* a = (const orc_tid_args*)args;
        for (int b = 0; b < n_tb; b++)
            for (int t = 0; t < threads; t++)
                a->out[a->base + (uint32_t)(b * warps_tb * 32 + t)] = ((uint32_t)b << 16) | (uint32_t)t;
        break;
    }
    case ORC_MB: {
        const orc_mb_args* a = (const orc_mb_args*)args;
        orc_mandelbrot_tile(a->out, a->x0, a->y0, a->dx, a->tx, a->ty, a->maxit);
        break;
    }
    case ORC_TDES: {
        const orc_tdes_args* a = (const orc_tdes_args*)args;
        orc_tdes_ecb(a->in, a->out, a->nbytes, a->key24, 0);
        break;
    }
    case ORC_MM: {
        const orc_mm_args* a = (const orc_mm_args*)args;
        orc_mm32(a->A, a->B, a->C);
        break;
    }
    case ORC_MM_TC: {
        const orc_mm_args* a = (const orc_mm_args*)args;
        orc_mm32_f64(a->A, a->B, a->C);
        break;
    }
    case ORC_FB: {
        const orc_fb_args* a = (const orc_fb_args*)args;
        orc_filterbank(a->r, a->H, a->F, a->y);
        break;
    }
    case ORC_BF: {
        const orc_bf_args* a = (const orc_bf_args*)args;
        orc_beamformer(a->x, a->h, a->w, a->out);
        break;
    }
    case ORC_CONV: {
        const orc_conv_args* a = (const orc_conv_args*)args;
        orc_conv(a->img, a->krow, a->kcol, a->out);
        break;
    }
    case ORC_DCT: {
        const orc_dct_args* a = (const orc_dct_args*)args;
        orc_dct(a->img, a->coef, a->out);
        break;
    }
    }
    return id;
}

int orc_wait(orc_ctx* c, int64_t id)
{
    if (!c) return -EINVAL;
    if (id < 0 || id >= c->next_id) return -EINVAL;
    return 0;
}

int orc_check(orc_ctx* c, int64_t id)
{
    if (!c) return -EINVAL;
    if (id < 0 || id >= c->next_id) return -EINVAL;
    return 1;
}

int orc_waitAll(orc_ctx* c) { return c ? 0 : -EINVAL; }

int orc_shutdown(orc_ctx* c)
{
    if (!c) return -EINVAL;
    if (c->shut) return -ESHUTDOWN;
    c->shut = 1;
    return 0;
}

void orc_destroy(orc_ctx* c) { free(c); }

double orc_occupancy_pct(int resident_warps, int n_sm)
{
    return 100.0 * (double)resident_warps / (64.0 * (double)n_sm);
}

/* ======================================================================
 * Trace-ledger checker.  Per MTB the scheduler warp is the single owner of
 * the allocator, so its events are a total order.
 * Kinds: 1 ALLOC (one TB: warps, granules, barrier), 2 FREE_WARPS (warps of
 * one TB returned — warps free one by one), 3 FREE_TB (the TB's
 * granules and barrier ID, returned by its last warp).
 * ==================================================================== */
typedef struct {
    uint64_t task_id; uint16_t tb; uint16_t mtb;
    uint32_t warps_live; uint32_t warps_alloc;
    uint16_t gran_off, gran_len; uint8_t bar_id; uint8_t tb_res_live;
} tb_rec;

static int ev_cmp(const void* a, const void* b)
{
    const orc_ledger_event* x = (const orc_ledger_event*)a;
    const orc_ledger_event* y = (const orc_ledger_event*)b;
    if (x->mtb != y->mtb) return x->mtb < y->mtb ? -1 : 1;
    if (x->seq != y->seq) return x->seq < y->seq ? -1 : 1;
    return 0;
}

#define FAIL(...) do { if (err && err_len) snprintf(err, err_len, __VA_ARGS__); rc = -1; goto done; } while (0)

int orc_ledger_check(const orc_ledger_event* ev_in, size_t n_ev, int n_mtb, int exec_warps,
                     int arena_granules, int n_bar_ids, const orc_ledger_task* tasks,
                     size_t n_tasks, char* err, size_t err_len)
{
    int rc = 0;
    orc_ledger_event* ev = (orc_ledger_event*)malloc((n_ev ? n_ev : 1) * sizeof *ev);
    tb_rec* recs = (tb_rec*)calloc(n_ev ? n_ev : 1, sizeof *recs);
    size_t n_recs = 0;
    uint32_t* live_w = (uint32_t*)calloc((size_t)n_mtb, sizeof(uint32_t));
    uint32_t* live_b = (uint32_t*)calloc((size_t)n_mtb, sizeof(uint32_t));
    int gwords = (arena_granules + 63) / 64;
    uint64_t* live_g = (uint64_t*)calloc((size_t)n_mtb * (size_t)(gwords ? gwords : 1), sizeof(uint64_t));
    if (!ev || !recs || !live_w || !live_b || !live_g) FAIL("out of memory");
    memcpy(ev, ev_in, n_ev * sizeof *ev);
    qsort(ev, n_ev, sizeof *ev, ev_cmp);

    uint32_t valid_w = 0;   /* worker warps 0..exec_warps-1 (every warp executes) */
    for (int w = 0; w < exec_warps && w < 32; w++) valid_w |= 1u << w;

    for (size_t i = 0; i < n_ev; i++) {
        const orc_ledger_event* e = &ev[i];
        if (e->mtb >= n_mtb) FAIL("event %zu: mtb %u out of range", i, e->mtb);
        if (i > 0 && ev[i - 1].mtb == e->mtb && ev[i - 1].seq == e->seq)
            FAIL("mtb %u: duplicate seq %u", e->mtb, e->seq);
        uint64_t* g = live_g + (size_t)e->mtb * (size_t)gwords;
        /* find this TB's record */
        tb_rec* r = NULL;
        for (size_t k = n_recs; k-- > 0;)
            if (recs[k].task_id == e->task_id && recs[k].tb == e->tb) { r = &recs[k]; break; }
        if (e->kind == 1) {
            if (r) FAIL("task %llu tb %u allocated twice", (unsigned long long)e->task_id, e->tb);
            if (e->warp_mask == 0 || (e->warp_mask & ~valid_w))
                FAIL("task %llu tb %u: bad warp mask %08x", (unsigned long long)e->task_id, e->tb, e->warp_mask);
            if (e->warp_mask & live_w[e->mtb])
                FAIL("mtb %u seq %u: warp double-assigned (mask %08x live %08x)", e->mtb, e->seq, e->warp_mask, live_w[e->mtb]);
            if ((int)e->gran_off + (int)e->gran_len > arena_granules)
                FAIL("mtb %u seq %u: granules [%u,+%u) exceed arena %d", e->mtb, e->seq, e->gran_off, e->gran_len, arena_granules);
            for (int q = e->gran_off; q < e->gran_off + e->gran_len; q++)
                if (g[q / 64] >> (q % 64) & 1u)
                    FAIL("mtb %u seq %u: granule %d double-allocated", e->mtb, e->seq, q);
            if (e->bar_id) {
                if (e->bar_id > n_bar_ids) FAIL("mtb %u seq %u: barrier id %u out of range", e->mtb, e->seq, e->bar_id);
                if (live_b[e->mtb] >> e->bar_id & 1u) FAIL("mtb %u seq %u: barrier id %u double-assigned", e->mtb, e->seq, e->bar_id);
                live_b[e->mtb] |= 1u << e->bar_id;
            }
            live_w[e->mtb] |= e->warp_mask;
            for (int q = e->gran_off; q < e->gran_off + e->gran_len; q++) g[q / 64] |= 1ull << (q % 64);
            r = &recs[n_recs++];
            r->task_id = e->task_id; r->tb = e->tb; r->mtb = e->mtb;
            r->warps_live = r->warps_alloc = e->warp_mask;
            r->gran_off = e->gran_off; r->gran_len = e->gran_len; r->bar_id = e->bar_id;
            r->tb_res_live = 1;
        } else if (e->kind == 2) {
            if (!r) FAIL("mtb %u seq %u: FREE_WARPS of unknown task %llu tb %u", e->mtb, e->seq, (unsigned long long)e->task_id, e->tb);
            if (r->mtb != e->mtb) FAIL("task %llu: freed on another MTB", (unsigned long long)e->task_id);
            if (e->warp_mask & ~r->warps_live)
                FAIL("mtb %u seq %u: FREE_WARPS %08x not live for task %llu tb %u (live %08x)", e->mtb, e->seq, e->warp_mask, (unsigned long long)e->task_id, e->tb, r->warps_live);
            r->warps_live &= ~e->warp_mask;
            live_w[e->mtb] &= ~e->warp_mask;
        } else if (e->kind == 3) {
            if (!r) FAIL("mtb %u seq %u: FREE_TB of unknown task %llu tb %u", e->mtb, e->seq, (unsigned long long)e->task_id, e->tb);
            if (!r->tb_res_live) FAIL("task %llu tb %u: TB resources freed twice", (unsigned long long)e->task_id, e->tb);
            if (e->gran_off != r->gran_off || e->gran_len != r->gran_len || e->bar_id != r->bar_id)
                FAIL("task %llu tb %u: FREE_TB resources differ from ALLOC", (unsigned long long)e->task_id, e->tb);
            for (int q = r->gran_off; q < r->gran_off + r->gran_len; q++) g[q / 64] &= ~(1ull << (q % 64));
            if (r->bar_id) live_b[e->mtb] &= ~(1u << r->bar_id);
            r->tb_res_live = 0;
        } else {
            FAIL("event %zu: unknown kind %u", i, e->kind);
        }
    }
    /* per task: every TB allocated once, all on one MTB, warps add up; drained at the end */
    for (size_t t = 0; t < n_tasks; t++) {
        uint32_t seen_tb = 0, warps = 0; int mtb = -1;
        for (size_t k = 0; k < n_recs; k++) {
            if (recs[k].task_id != tasks[t].task_id) continue;
            if (recs[k].tb >= tasks[t].n_tb) FAIL("task %llu: tb %u >= n_tb", (unsigned long long)tasks[t].task_id, recs[k].tb);
            seen_tb++;
            warps += (uint32_t)__builtin_popcount(recs[k].warps_alloc);
            if (mtb >= 0 && mtb != recs[k].mtb) FAIL("task %llu: TBs on MTBs %d and %u", (unsigned long long)tasks[t].task_id, mtb, recs[k].mtb);
            mtb = recs[k].mtb;
            if (recs[k].warps_live || recs[k].tb_res_live)
                FAIL("task %llu tb %u: resources never freed", (unsigned long long)tasks[t].task_id, recs[k].tb);
        }
        if (seen_tb != tasks[t].n_tb) FAIL("task %llu: %u TBs allocated, expected %u", (unsigned long long)tasks[t].task_id, seen_tb, tasks[t].n_tb);
        if (warps != tasks[t].warps_total) FAIL("task %llu: %u warps allocated, expected %u", (unsigned long long)tasks[t].task_id, warps, tasks[t].warps_total);
    }
    if (n_recs != 0) {
        /* every allocated TB must belong to a listed task */
        for (size_t k = 0; k < n_recs; k++) {
            int found = 0;
            for (size_t t = 0; t < n_tasks && !found; t++) found = tasks[t].task_id == recs[k].task_id;
            if (!found) FAIL("ALLOC for unlisted task %llu", (unsigned long long)recs[k].task_id);
        }
    }
done:
    free(ev); free(recs); free(live_w); free(live_b); free(live_g);
    return rc;
}

/* ======================================================================
 * Executor intervals + completion records (oracle.h orc_exec_check).
 * Sorted copies and binary searches: the brute-force schedules replay
 * ~10^5 records per session.
 * ==================================================================== */
typedef struct { uint64_t task_id; uint16_t tb, mtb; uint32_t mask, seen; } alloc_key;

static int ak_cmp(const void* a, const void* b)
{
    const alloc_key* x = (const alloc_key*)a;
    const alloc_key* y = (const alloc_key*)b;
    if (x->task_id != y->task_id) return x->task_id < y->task_id ? -1 : 1;
    return (int)x->tb - (int)y->tb;
}
static int ex_task_cmp(const void* a, const void* b)   /* (task, tb, warp) */
{
    const orc_exec_record* x = (const orc_exec_record*)a;
    const orc_exec_record* y = (const orc_exec_record*)b;
    if (x->task_id != y->task_id) return x->task_id < y->task_id ? -1 : 1;
    if (x->tb != y->tb) return (int)x->tb - (int)y->tb;
    return (int)x->warp - (int)y->warp;
}
static int ex_warp_cmp(const void* a, const void* b)   /* (mtb, warp, t_start) */
{
    const orc_exec_record* x = (const orc_exec_record*)a;
    const orc_exec_record* y = (const orc_exec_record*)b;
    if (x->mtb != y->mtb) return (int)x->mtb - (int)y->mtb;
    if (x->warp != y->warp) return (int)x->warp - (int)y->warp;
    if (x->t_start != y->t_start) return x->t_start < y->t_start ? -1 : 1;
    return 0;
}
static int comp_cmp(const void* a, const void* b)
{
    const orc_completion* x = (const orc_completion*)a;
    const orc_completion* y = (const orc_completion*)b;
    return x->task_id < y->task_id ? -1 : x->task_id > y->task_id ? 1 : 0;
}

int orc_exec_check(const orc_ledger_event* ev, size_t n_ev, const orc_exec_record* ex_in, size_t n_ex,
                   const orc_completion* comp_in, size_t n_comp, const orc_ledger_task* tasks,
                   size_t n_tasks, char* err, size_t err_len)
{
    int rc = 0;
    size_t n_al = 0;
    alloc_key* al = (alloc_key*)malloc((n_ev ? n_ev : 1) * sizeof *al);
    orc_exec_record* ex = (orc_exec_record*)malloc((n_ex ? n_ex : 1) * sizeof *ex);
    orc_exec_record* exw = (orc_exec_record*)malloc((n_ex ? n_ex : 1) * sizeof *exw);
    orc_completion* cp = (orc_completion*)malloc((n_comp ? n_comp : 1) * sizeof *cp);
    orc_completion* tid = NULL;   /* sorted task ids */
    if (!al || !ex || !exw || !cp) FAIL("out of memory");
    for (size_t i = 0; i < n_ev; i++)
        if (ev[i].kind == 1) {
            alloc_key k = {ev[i].task_id, ev[i].tb, ev[i].mtb, ev[i].warp_mask, 0};
            al[n_al++] = k;
        }
    qsort(al, n_al, sizeof *al, ak_cmp);
    for (size_t i = 1; i < n_al; i++)
        if (ak_cmp(&al[i - 1], &al[i]) == 0)
            FAIL("task %llu tb %u allocated twice", (unsigned long long)al[i].task_id, al[i].tb);
    memcpy(ex, ex_in, n_ex * sizeof *ex);
    memcpy(exw, ex_in, n_ex * sizeof *exw);
    qsort(ex, n_ex, sizeof *ex, ex_task_cmp);
    qsort(exw, n_ex, sizeof *exw, ex_warp_cmp);
    memcpy(cp, comp_in, n_comp * sizeof *cp);
    qsort(cp, n_comp, sizeof *cp, comp_cmp);

    /* 1. every execution interval is well formed and lies in its TB's allocation */
    for (size_t i = 0; i < n_ex; i++) {
        const orc_exec_record* r = &ex[i];
        if (r->t_end < r->t_start)
            FAIL("task %llu tb %u warp %u: interval ends before it starts", (unsigned long long)r->task_id, r->tb, r->warp);
        if (i > 0 && ex_task_cmp(&ex[i - 1], r) == 0)
            FAIL("task %llu tb %u warp %u ran twice", (unsigned long long)r->task_id, r->tb, r->warp);
        alloc_key k = {r->task_id, r->tb, 0, 0, 0};
        alloc_key* a = (alloc_key*)bsearch(&k, al, n_al, sizeof *al, ak_cmp);
        if (!a) FAIL("task %llu tb %u ran without an ALLOC", (unsigned long long)r->task_id, r->tb);
        if (a->mtb != r->mtb)
            FAIL("task %llu tb %u ran on MTB %u, allocated on MTB %u", (unsigned long long)r->task_id, r->tb, r->mtb, a->mtb);
        if (r->warp >= 32 || !((a->mask >> r->warp) & 1u))
            FAIL("task %llu tb %u ran on warp %u outside its ALLOC mask %08x", (unsigned long long)r->task_id, r->tb, r->warp, a->mask);
        a->seen |= 1u << r->warp;
    }
    for (size_t i = 0; i < n_al; i++)
        if (al[i].seen != al[i].mask)
            FAIL("task %llu tb %u: warps %08x allocated, %08x ran", (unsigned long long)al[i].task_id, al[i].tb, al[i].mask, al[i].seen);
    /* 2. a warp never runs two tasks at once */
    for (size_t i = 1; i < n_ex; i++) {
        const orc_exec_record *p = &exw[i - 1], *q = &exw[i];
        if (p->mtb == q->mtb && p->warp == q->warp && q->t_start < p->t_end)
            FAIL("mtb %u warp %u: task %llu starts at %llu before task %llu ends at %llu", q->mtb, q->warp,
                 (unsigned long long)q->task_id, (unsigned long long)q->t_start, (unsigned long long)p->task_id,
                 (unsigned long long)p->t_end);
    }
    /* 3. exactly one completion per task, after the last warp of the task ended */
    for (size_t i = 1; i < n_comp; i++)
        if (cp[i - 1].task_id == cp[i].task_id) FAIL("task %llu completed twice", (unsigned long long)cp[i].task_id);
    for (size_t t = 0; t < n_tasks; t++) {
        orc_completion k = {tasks[t].task_id, 0};
        const orc_completion* c = (const orc_completion*)bsearch(&k, cp, n_comp, sizeof *cp, comp_cmp);
        if (!c) FAIL("task %llu has no completion record", (unsigned long long)tasks[t].task_id);
        /* the task's execution records are contiguous in ex (sorted by task first) */
        size_t lo = 0, hi = n_ex;
        while (lo < hi) {
            const size_t mid = (lo + hi) / 2;
            if (ex[mid].task_id < tasks[t].task_id) lo = mid + 1;
            else hi = mid;
        }
        uint64_t last_end = 0;
        uint32_t warps = 0;
        for (size_t i = lo; i < n_ex && ex[i].task_id == tasks[t].task_id; i++) {
            if (ex[i].t_end > last_end) last_end = ex[i].t_end;
            warps++;
        }
        if (warps != tasks[t].warps_total)
            FAIL("task %llu: %u warps ran, expected %u", (unsigned long long)tasks[t].task_id, warps, tasks[t].warps_total);
        if (c->t_done < last_end)
            FAIL("task %llu completed at %llu before its last warp ended at %llu", (unsigned long long)tasks[t].task_id,
                 (unsigned long long)c->t_done, (unsigned long long)last_end);
    }
    tid = (orc_completion*)malloc((n_tasks ? n_tasks : 1) * sizeof *tid);
    if (!tid) FAIL("out of memory");
    for (size_t t = 0; t < n_tasks; t++) tid[t].task_id = tasks[t].task_id, tid[t].t_done = 0;
    qsort(tid, n_tasks, sizeof *tid, comp_cmp);
    for (size_t i = 0; i < n_comp; i++)
        if (!bsearch(&cp[i], tid, n_tasks, sizeof *tid, comp_cmp))
            FAIL("completion record of unlisted task %llu", (unsigned long long)cp[i].task_id);
done:
    free(al); free(ex); free(exw); free(cp); free(tid);
    return rc;
}
