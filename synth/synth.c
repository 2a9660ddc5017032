/*
 * synth.c — seeded synthetic INPUT generators.
 *
 * This module is shared by the CUDA path's drivers (bench.py, smoke) and by
 * the tests that feed the oracle.  It holds NONE of the method's arithmetic:
 * no translation, no paging, no histogram-of-a-block, no LSH key, no SSD.
 * It only draws random bytes with a counter-based generator (splitmix64) and
 * lays them out as the paper's workloads are laid out:
 *
 *   - the "file" of the apointer microbenchmarks (§VI-C):
 *     word j (uint64, little endian) = sm64(file_seed + j), so every page is
 *     distinct and a wrong-frame bug shows up as a mismatch;
 *   - the collage dataset (§VI-E): N records, each the
 *     colour counts of 1024 drawn RGB samples ("tiny image" pixels,
 *     PAPER.md:411 / [22]) stored as 768 uint32 at record i * rec_stride,
 *     zero padding to the stride (4 KiB);
 *   - the collage target image: W x H RGB uint8, each
 *     32x32 block drawn from a pool of source tiles (+-2 noise) or planted as
 *     an exact copy of a dataset tile's samples;
 *   - the LSH random projections / offsets ([21]): int16
 *     approximately-Gaussian entries (sum of 4 random bytes - 510) and int32
 *     offsets in [0, w).  These are the random numbers the method draws; they
 *     are passed to both sides as inputs.
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC synth.c -o libsynth.so
 */
#include <stdint.h>
#include <string.h>

/* splitmix64 output for counter x (Steele et al.; sm64(0)=0xe220a8397b1dcdaf). */
static inline uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}

uint64_t synth_sm64(uint64_t x) { return sm64(x); }

/* File contents: word j = sm64(seed + j); a ragged tail takes the low bytes
 * of the next word. */
void synth_file(uint8_t* buf, uint64_t bytes, uint64_t seed) {
    uint64_t nwords = bytes / 8;
    uint64_t* w = (uint64_t*)buf; /* buffers come from mmap/malloc: 8-B aligned */
    #pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < (int64_t)nwords; ++j) w[j] = sm64(seed + (uint64_t)j);
    uint64_t tail = bytes - nwords * 8;
    if (tail) {
        uint64_t last = sm64(seed + nwords);
        memcpy(buf + nwords * 8, &last, tail);
    }
}

/* Tile i's RGB samples (1024 pixels x 3 channels, interleaved).  Channel c
 * of tile i is a "blob": mean m_c ~ U[0,255], spread s_c ~ U[4,64]; a sample
 * is m_c + d*s_c/510 with d = (sum of 4 random bytes) - 510, clamped. */
static void tile_px(uint64_t seed, uint64_t i, uint8_t* px) {
    int mean[3], spread[3];
    for (int c = 0; c < 3; ++c) {
        uint64_t u = sm64(seed ^ ((i << 12) | (uint64_t)(4000 + c)));
        mean[c] = (int)(u & 255);
        spread[c] = 4 + (int)((u >> 8) % 61);
    }
    for (int p = 0; p < 1024; ++p)
        for (int c = 0; c < 3; ++c) {
            uint64_t u = sm64(seed ^ ((i << 12) | (uint64_t)(p * 3 + c)));
            int d = (int)(u & 255) + (int)((u >> 8) & 255) + (int)((u >> 16) & 255) +
                    (int)((u >> 24) & 255) - 510;
            int v = mean[c] + d * spread[c] / 510;
            px[p * 3 + c] = (uint8_t)(v < 0 ? 0 : v > 255 ? 255 : v);
        }
}

void synth_tile_pixels(uint64_t seed, uint64_t i, uint8_t* px) { tile_px(seed, i, px); }

/* Dataset records: record i at byte i*rec_stride holds 768 uint32 sample
 * counts (channel-major, [c*256 + value]); the rest of the stride is zero.
 * Records [first, first+count) are written (lets callers generate slices). */
void synth_records(uint8_t* buf, uint64_t first, uint64_t count, uint32_t rec_stride,
                   uint64_t seed) {
    #pragma omp parallel for schedule(dynamic, 256)
    for (int64_t k = 0; k < (int64_t)count; ++k) {
        uint64_t i = first + (uint64_t)k;
        uint8_t px[3072];
        uint32_t cnt[768];
        tile_px(seed, i, px);
        memset(cnt, 0, sizeof cnt);
        for (int p = 0; p < 1024; ++p)
            for (int c = 0; c < 3; ++c) cnt[c * 256 + px[p * 3 + c]]++;
        uint8_t* rec = buf + (uint64_t)k * rec_stride;
        if (rec_stride >= 3072) {
            memcpy(rec, cnt, 3072);
            memset(rec + 3072, 0, rec_stride - 3072);
        }
    }
}

/* Target image W x H (multiples of 32), RGB interleaved, row-major.
 * Block b = by*(W/32)+bx.  With probability copy_permille/1000 the block is
 * an exact copy of a uniformly drawn dataset tile (planted self-query);
 * otherwise it is a tile from a pool of `pool` source tiles with +-2 noise
 * per sample.  src[b] = tile id used, is_copy[b] = 1 for exact copies. */
void synth_target(uint8_t* img, uint32_t W, uint32_t H, uint64_t N, uint64_t ds_seed,
                  uint64_t seed, uint32_t pool, uint32_t copy_permille, int64_t* src,
                  uint8_t* is_copy) {
    uint32_t bw = W / 32, bh = H / 32;
    #pragma omp parallel for schedule(dynamic, 16)
    for (int64_t b = 0; b < (int64_t)bw * bh; ++b) {
        uint64_t u = sm64(seed ^ (0xB10CULL << 40) ^ (uint64_t)b);
        int copy = (u % 1000) < copy_permille;
        uint64_t j;
        if (copy) {
            j = sm64(u) % N;
        } else {
            uint64_t r = (u >> 20) % (pool ? pool : 1);
            j = sm64(seed ^ (0x9001ULL << 40) ^ r) % N;
        }
        uint8_t px[3072];
        tile_px(ds_seed, j, px);
        uint32_t bx = (uint32_t)(b % bw), by = (uint32_t)(b / bw);
        for (int y = 0; y < 32; ++y)
            for (int x = 0; x < 32; ++x)
                for (int c = 0; c < 3; ++c) {
                    int p = y * 32 + x;
                    int v = px[p * 3 + c];
                    if (!copy) {
                        uint64_t n = sm64(seed ^ (((uint64_t)b << 12) | (uint64_t)(p * 3 + c)));
                        v += (int)(n % 5) - 2;
                        v = v < 0 ? 0 : v > 255 ? 255 : v;
                    }
                    img[((uint64_t)(by * 32 + y) * W + (bx * 32 + x)) * 3 + c] = (uint8_t)v;
                }
        if (src) src[b] = (int64_t)j;
        if (is_copy) is_copy[b] = (uint8_t)copy;
    }
}

/* LSH random draws ([21] p-stable, integerised; reading A5):
 * proj[(t*K+k)*768 + d] = (sum of 4 random bytes) - 510   (int16)
 * bias[t*K+k]           = U[0, w)                         (int32)        */
void synth_lsh_params(int16_t* proj, int32_t* bias, uint32_t L, uint32_t K, int32_t w,
                      uint64_t seed) {
    for (uint64_t tk = 0; tk < (uint64_t)L * K; ++tk) {
        for (uint64_t d = 0; d < 768; ++d) {
            uint64_t u = sm64(seed ^ (0x1D5ULL << 48) ^ (tk << 12) ^ d);
            int s = (int)(u & 255) + (int)((u >> 8) & 255) + (int)((u >> 16) & 255) +
                    (int)((u >> 24) & 255) - 510;
            proj[tk * 768 + d] = (int16_t)s;
        }
        uint64_t u = sm64(seed ^ (0xB1A5ULL << 48) ^ tk);
        bias[tk] = (int32_t)(u % (uint64_t)(w > 0 ? w : 1));
    }
}
