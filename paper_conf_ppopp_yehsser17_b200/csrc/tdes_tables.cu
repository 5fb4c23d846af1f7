/*
 * tdes_tables.cu — host-side preparation of the 3DES task's device tables
 * (pagoda_tdes_tables in include/pagoda.h).  The permutation tables below are
 * the product's own transcription of NIST FIPS 46-3 (the standard the paper
 * cites for 3DES, [5] P:1627-1629); the CPU oracle keeps an independent copy,
 * and the known-answer tests pin both.
 *
 * Output layout (bytes):
 *   [0, 2048)        SP[8][64] u32: P(S_j(six) placed in nibble j) for the 6-bit
 *                    input six = b1..b6 of box j (b1 = most significant)
 *   [2048, 2432)     48 round keys as (kx, ky) u32 pairs, execution order
 *                    K1 rounds 1..16, K2 rounds 16..1 (decrypt), K3 rounds 1..16;
 *                    kx bytes 0..3 = the key chunks of S-boxes 0,6,4,2, ky of 7,5,3,1
 *   [2432, 18816)    IPT[8][256] u64: IP of byte b (b = 0 most significant) alone
 *   [18816, 35200)   FPT[8][256] u64: IP^-1 likewise
 */
#include <stdint.h>
#include <string.h>

#include "pagoda.h"

namespace {

/* FIPS 46-3 tables, 1-based bit numbers, bit 1 = most significant */
const int kIP[64] = {58, 50, 42, 34, 26, 18, 10, 2, 60, 52, 44, 36, 28, 20, 12, 4, 62, 54, 46, 38, 30, 22,
                     14, 6,  64, 56, 48, 40, 32, 24, 16, 8, 57, 49, 41, 33, 25, 17, 9,  1,  59, 51, 43, 35,
                     27, 19, 11, 3,  61, 53, 45, 37, 29, 21, 13, 5, 63, 55, 47, 39, 31, 23, 15, 7};
const int kPerm[32] = {16, 7, 20, 21, 29, 12, 28, 17, 1, 15, 23, 26, 5,  18, 31, 10,
                       2,  8, 24, 14, 32, 27, 3,  9,  19, 13, 30, 6, 22, 11, 4,  25};
const int kPC1[56] = {57, 49, 41, 33, 25, 17, 9,  1,  58, 50, 42, 34, 26, 18, 10, 2,  59, 51, 43,
                      35, 27, 19, 11, 3,  60, 52, 44, 36, 63, 55, 47, 39, 31, 23, 15, 7,  62, 54,
                      46, 38, 30, 22, 14, 6,  61, 53, 45, 37, 29, 21, 13, 5,  28, 20, 12, 4};
const int kPC2[48] = {14, 17, 11, 24, 1,  5,  3,  28, 15, 6,  21, 10, 23, 19, 12, 4,
                      26, 8,  16, 7,  27, 20, 13, 2,  41, 52, 31, 37, 47, 55, 30, 40,
                      51, 45, 33, 48, 44, 49, 39, 56, 34, 53, 46, 42, 50, 36, 29, 32};
const int kRot[16] = {1, 1, 2, 2, 2, 2, 2, 2, 1, 2, 2, 2, 2, 2, 2, 1};
/* S-boxes, each 4 rows x 16 columns flattened */
const uint8_t kS[8][64] = {
    {14, 4,  13, 1, 2,  15, 11, 8,  3,  10, 6,  12, 5,  9,  0, 7,  0, 15, 7,  4,  14, 2,
     13, 1,  10, 6, 12, 11, 9,  5,  3,  8,  4,  1,  14, 8,  13, 6, 2, 11, 15, 12, 9,  7,
     3,  10, 5,  0, 15, 12, 8,  2,  4,  9,  1,  7,  5,  11, 3,  14, 10, 0, 6,  13},
    {15, 1,  8,  14, 6,  11, 3, 4,  9,  7, 2,  13, 12, 0, 5,  10, 3,  13, 4,  7,  15, 2,
     8,  14, 12, 0,  1,  10, 6, 9,  11, 5, 0,  14, 7,  11, 10, 4, 13, 1,  5,  8,  12, 6,
     9,  3,  2,  15, 13, 8,  10, 1, 3,  15, 4,  2,  11, 6,  7,  12, 0,  5,  14, 9},
    {10, 0,  9,  14, 6,  3,  15, 5,  1, 13, 12, 7, 11, 4,  2,  8,  13, 7,  0, 9,  3,  4,
     6,  10, 2,  8,  5,  14, 12, 11, 15, 1, 13, 6, 4,  9,  8,  15, 3,  0, 11, 1,  2,  12,
     5,  10, 14, 7,  1,  10, 13, 0,  6, 9,  8,  7, 4,  15, 14, 3,  11, 5, 2,  12},
    {7,  13, 14, 3,  0,  6,  9,  10, 1, 2,  8,  5,  11, 12, 4,  15, 13, 8,  11, 5, 6, 15,
     0,  3,  4,  7,  2,  12, 1,  10, 14, 9, 10, 6,  9,  0,  12, 11, 7,  13, 15, 1, 3, 14,
     5,  2,  8,  4,  3,  15, 0,  6,  10, 1, 13, 8,  9,  4,  5,  11, 12, 7,  2,  14},
    {2,  12, 4,  1,  7,  10, 11, 6,  8,  5,  3,  15, 13, 0, 14, 9,  14, 11, 2, 12, 4, 7,
     13, 1,  5,  0,  15, 10, 3,  9,  8,  6,  4,  2,  1,  11, 10, 13, 7,  8,  15, 9, 12, 5,
     6,  3,  0,  14, 11, 8,  12, 7,  1,  14, 2,  13, 6,  15, 0,  9,  10, 4,  5, 3},
    {12, 1,  10, 15, 9,  2,  6,  8,  0,  13, 3,  4,  14, 7,  5,  11, 10, 15, 4,  2,  7, 12,
     9,  5,  6,  1,  13, 14, 0,  11, 3,  8,  9,  14, 15, 5,  2,  8,  12, 3,  7,  0,  4, 10,
     1,  13, 11, 6,  4,  3,  2,  12, 9,  5,  15, 10, 11, 14, 1,  7,  6,  0,  8,  13},
    {4,  11, 2,  14, 15, 0,  8,  13, 3,  12, 9,  7,  5,  10, 6,  1,  13, 0,  11, 7,  4, 9,
     1,  10, 14, 3,  5,  12, 2,  15, 8,  6,  1,  4,  11, 13, 12, 3,  7,  14, 10, 15, 6, 8,
     0,  5,  9,  2,  6,  11, 13, 8,  1,  4,  10, 7,  9,  5,  0,  15, 14, 2,  3,  12},
    {13, 2,  8,  4,  6,  15, 11, 1,  10, 9,  3,  14, 5,  0,  12, 7,  1,  15, 13, 8,  10, 3,
     7,  4,  12, 5,  6,  11, 0,  14, 9,  2,  7,  11, 4,  1,  9,  12, 14, 2,  0,  6,  10, 13,
     15, 3,  5,  8,  2,  1,  14, 7,  4,  10, 8,  13, 15, 12, 9,  0,  3,  5,  6,  11}};

/* generic bit permutation: output bit k (1-based from the MSB of an n_out-bit
 * word) takes input bit tab[k-1] (1-based from the MSB of an n_in-bit word) */
uint64_t bits_permute(uint64_t x, const int* tab, int n_in, int n_out)
{
    uint64_t y = 0;
    for (int k = 0; k < n_out; k++)
        if ((x >> (n_in - tab[k])) & 1u) y |= 1ull << (n_out - 1 - k);
    return y;
}

void subkeys(const uint8_t* key8, uint64_t out[16])
{
    uint64_t k = 0;
    for (int i = 0; i < 8; i++) k = (k << 8) | key8[i];
    const uint64_t cd = bits_permute(k, kPC1, 64, 56);
    uint64_t c = cd >> 28, d = cd & 0xFFFFFFFull;
    for (int r = 0; r < 16; r++) {
        for (int s = 0; s < kRot[r]; s++) {
            c = ((c << 1) | (c >> 27)) & 0xFFFFFFFull;
            d = ((d << 1) | (d >> 27)) & 0xFFFFFFFull;
        }
        out[r] = bits_permute((c << 28) | d, kPC2, 56, 48);
    }
}

} // namespace

extern "C" int pagoda_tdes_tables(const uint8_t key24[24], void* dst)
{
    if (!key24 || !dst) return -22;
    uint8_t* out = static_cast<uint8_t*>(dst);
    uint32_t* sp = reinterpret_cast<uint32_t*>(out);
    for (int j = 0; j < 8; j++)
        for (int six = 0; six < 64; six++) {
            const int row = ((six >> 4) & 2) | (six & 1), col = (six >> 1) & 15;
            const uint64_t nib = (uint64_t)kS[j][row * 16 + col] << (28 - 4 * j);
            sp[j * 64 + six] = (uint32_t)bits_permute(nib, kPerm, 32, 32);
        }
    uint32_t* rk = reinterpret_cast<uint32_t*>(out + 2048);
    uint64_t k1[16], k2[16], k3[16];
    subkeys(key24, k1);
    subkeys(key24 + 8, k2);
    subkeys(key24 + 16, k3);
    for (int r = 0; r < 48; r++) {
        const uint64_t k = r < 16 ? k1[r] : (r < 32 ? k2[31 - r] : k3[r - 32]);
        uint32_t c[8];   /* c[j] = the 6 key bits that meet S-box j's input */
        for (int j = 0; j < 8; j++) c[j] = (uint32_t)((k >> (42 - 6 * j)) & 63u);
        rk[2 * r + 0] = c[0] | (c[6] << 8) | (c[4] << 16) | (c[2] << 24);   /* kx: boxes 0,6,4,2 */
        rk[2 * r + 1] = c[7] | (c[5] << 8) | (c[3] << 16) | (c[1] << 24);   /* ky: boxes 7,5,3,1 */
    }
    int fp[64];   /* IP^-1: IP maps input bit kIP[k] to output bit k+1 */
    for (int k = 0; k < 64; k++) fp[kIP[k] - 1] = k + 1;
    uint64_t* ipt = reinterpret_cast<uint64_t*>(out + 2432);
    uint64_t* fpt = reinterpret_cast<uint64_t*>(out + 2432 + 16384);
    for (int b = 0; b < 8; b++)
        for (int v = 0; v < 256; v++) {
            const uint64_t x = (uint64_t)v << (56 - 8 * b);
            ipt[b * 256 + v] = bits_permute(x, kIP, 64, 64);
            fpt[b * 256 + v] = bits_permute(x, fp, 64, 64);
        }
    return 0;
}
