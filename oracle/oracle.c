/*
 * oracle.c — the CPU ORACLE for the apointer dereference path and its photo
 * collage consumer.  TEST INFRASTRUCTURE ONLY: only tests/,
 * __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs
 * may load this library.  It shares no code, header, table or constant
 * generator with the CUDA path (paper_conf_isca_shaharbs16_b200/csrc) and
 * never includes or links it.
 *
 * Plain, slow, obviously correct.  Every function cites the passage it
 * follows (PAPER.md line numbers, section in parentheses; DESIGN.md readings
 * as R-Ax, numbered like SURVEY.md §8(c)).
 *
 * O1  reads: an apointer "behave[s] just like regular memory pointers"
 *     (§III-C); a read through it returns the file's bytes at
 *     the offset, page faults are invisible to values.  So
 *     the oracle is plain file indexing: no cache, no pages, no frames.
 *     The access sequences (SEQ/UNIFORM/DIVERGENT, R-A23/A24) and the
 *     per-thread FNV-1a-64 checksum are workload definitions.
 *
 * O3  collage (§VI-E), step by step in the paper's order:
 *     histogram of each 32x32 block -> LSH keys -> candidates from the
 *     buckets indexed by the keys -> Euclidean (squared, R-A2) distance ->
 *     closest candidate (lexicographic (dist, idx), R-A3).
 *
 * Build: gcc -O2 -fopenmp -shared -fPIC oracle.c -o liboracle.so
 */
#include <stdint.h>
#include <stdlib.h>
#include <string.h>

/* ------------------------------------------------------------------ */
/* Counter-based generator used by the workload definitions (R-A23).   */
/* splitmix64 output for counter x; sm64(0) = 0xe220a8397b1dcdaf.      */
/* ------------------------------------------------------------------ */
static uint64_t or_sm64_(uint64_t x) {
    uint64_t z = x + 0x9e3779b97f4a7c15ULL;
    z = (z ^ (z >> 30)) * 0xbf58476d1ce4e5b9ULL;
    z = (z ^ (z >> 27)) * 0x94d049bb133111ebULL;
    return z ^ (z >> 31);
}
uint64_t or_sm64(uint64_t x) { return or_sm64_(x); }

/* Per-thread checksum of the values a thread read, in access order:
 * FNV-1a-64 over the value's 64-bit little-endian words (a 4-B value is one
 * zero-extended word; a 16-B value is its low word then its high word). */
#define OR_FNV_OFFSET 0xcbf29ce484222325ULL
#define OR_FNV_PRIME 0x100000001b3ULL

static uint64_t or_fnv_value(uint64_t h, const uint8_t* v, uint32_t elem) {
    if (elem == 4) {
        uint32_t x;
        memcpy(&x, v, 4);
        h = (h ^ (uint64_t)x) * OR_FNV_PRIME;
    } else {
        for (uint32_t k = 0; k < elem; k += 8) {
            uint64_t x;
            memcpy(&x, v + k, 8);
            h = (h ^ x) * OR_FNV_PRIME;
        }
    }
    return h;
}
uint64_t or_fnv_words(uint64_t h, const uint8_t* v, uint32_t elem) {
    return or_fnv_value(h, v, elem);
}

/* O1: value(region, off) = the sizeof(T) bytes of the file at off
 * (PAPER.md:121, 141-143). */
static const uint8_t* or_value_at(const uint8_t* file, uint64_t off) { return file + off; }

/* SEQ pattern (R-A24, hit-mode of SURVEY §8(d) M2h): warp w of W reads
 * units w, w+W, ... of `unit` bytes of [0, span); inside a unit lane l reads
 * element j*32+l for j = 0 .. unit/(32*elem)-1; elements past `span` are not
 * read; the whole sweep repeats `passes` times.
 * If out_copy != NULL it receives the bytes read at their offsets (C1);
 * otherwise ck[t] is thread t's checksum. */
void or_read_seq(const uint8_t* file, uint64_t span, uint32_t unit, uint32_t elem,
                 uint64_t nthreads, uint32_t passes, uint8_t* out_copy, uint64_t* ck,
                 int threads) {
    uint64_t W = nthreads / 32;
    uint64_t nunits = (span + unit - 1) / unit;
    uint32_t per_unit = unit / (32 * elem);
    #pragma omp parallel for schedule(dynamic, 64) num_threads(threads)
    for (int64_t t = 0; t < (int64_t)nthreads; ++t) {
        uint64_t w = (uint64_t)t / 32, lane = (uint64_t)t % 32;
        uint64_t h = OR_FNV_OFFSET;
        for (uint32_t pass = 0; pass < passes; ++pass)
            for (uint64_t u = w; u < nunits; u += W)
                for (uint32_t j = 0; j < per_unit; ++j) {
                    uint64_t off = u * unit + ((uint64_t)j * 32 + lane) * elem;
                    if (off + elem > span) continue;
                    const uint8_t* v = or_value_at(file, off);
                    if (out_copy) memcpy(out_copy + off, v, elem);
                    else h = or_fnv_value(h, v, elem);
                }
        if (ck) ck[t] = h;
    }
}

/* UNIFORM pattern (R-A23): read i of thread t is at element
 * sm64(seed ^ (t<<24) ^ i) mod (bytes/elem). */
uint64_t or_uniform_off(uint64_t bytes, uint32_t elem, uint64_t seed, uint64_t t, uint64_t i) {
    return (or_sm64_(seed ^ (t << 24) ^ i) % (bytes / elem)) * elem;
}

void or_read_uniform(const uint8_t* file, uint64_t bytes, uint32_t elem, uint64_t nthreads,
                     uint32_t reads, uint64_t seed, uint64_t* ck, int threads) {
    #pragma omp parallel for schedule(static) num_threads(threads)
    for (int64_t t = 0; t < (int64_t)nthreads; ++t) {
        uint64_t h = OR_FNV_OFFSET;
        for (uint32_t i = 0; i < reads; ++i)
            h = or_fnv_value(h, or_value_at(file, or_uniform_off(bytes, elem, seed, t, i)), elem);
        ck[t] = h;
    }
}

/* DIVERGENT pattern (R-A23): the 32 lanes of warp w are on
 * 32 distinct pages: page = (sm64(seed ^ (w<<24) ^ i) + lane*(npg/32)) mod npg
 * with npg = bytes/page (whole pages); element inside the page =
 * sm64(seed ^ (t<<24) ^ i ^ 0xD1B54A32D192ED03) mod (page/elem). */
uint64_t or_divergent_off(uint64_t bytes, uint32_t page, uint32_t elem, uint64_t seed,
                          uint64_t t, uint64_t i) {
    uint64_t npg = bytes / page;
    uint64_t w = t / 32, lane = t % 32;
    uint64_t pg = (or_sm64_(seed ^ (w << 24) ^ i) + lane * (npg / 32)) % npg;
    uint64_t el = or_sm64_(seed ^ (t << 24) ^ i ^ 0xD1B54A32D192ED03ULL) % (page / elem);
    return pg * page + el * elem;
}

void or_read_divergent(const uint8_t* file, uint64_t bytes, uint32_t page, uint32_t elem,
                       uint64_t nthreads, uint32_t reads, uint64_t seed, uint64_t* ck,
                       int threads) {
    #pragma omp parallel for schedule(static) num_threads(threads)
    for (int64_t t = 0; t < (int64_t)nthreads; ++t) {
        uint64_t h = OR_FNV_OFFSET;
        for (uint32_t i = 0; i < reads; ++i)
            h = or_fnv_value(
                h, or_value_at(file, or_divergent_off(bytes, page, elem, seed, t, i)), elem);
        ck[t] = h;
    }
}

/* The offsets a random-pattern run reads, in access order: out[t*reads+i]
 * = the offset of read i of thread t (pattern 1 = UNIFORM over `bytes`,
 * 2 = DIVERGENT with pattern page size `page`).  Used by the O2 link-count
 * invariant (oracle/invariants.py link_events). */
void or_offsets(int pattern, uint64_t bytes, uint32_t page, uint32_t elem, uint64_t seed,
                uint64_t nthreads, uint32_t reads, uint64_t* out) {
    for (uint64_t t = 0; t < nthreads; ++t)
        for (uint32_t i = 0; i < reads; ++i)
            out[t * reads + i] = pattern == 1 ? or_uniform_off(bytes, elem, seed, t, i)
                                              : or_divergent_off(bytes, page, elem, seed, t, i);
}

/* ------------------------------------------------------------------ */
/* O3 — photo collage                               */
/* ------------------------------------------------------------------ */

/* Step 1-2 ("calculates the histogram of each 32x32 block";
 * R-A7): img is W x H RGB, interleaved, row-major; block b = by*(W/32)+bx;
 * hist[c*256 + v] = number of pixels of the block whose channel c equals v. */
void or_block_hist(const uint8_t* img, uint32_t W, uint32_t H, uint64_t b, uint32_t* hist) {
    (void)H;
    uint32_t bw = W / 32;
    uint32_t bx = (uint32_t)(b % bw), by = (uint32_t)(b / bw);
    memset(hist, 0, 768 * sizeof(uint32_t));
    for (uint32_t y = 0; y < 32; ++y)
        for (uint32_t x = 0; x < 32; ++x)
            for (uint32_t c = 0; c < 3; ++c) {
                uint8_t v = img[((uint64_t)(by * 32 + y) * W + (bx * 32 + x)) * 3 + c];
                hist[c * 256 + v] += 1;
            }
}

/* floor(a / b) for b > 0, also for negative a (R-A5). */
static int64_t or_floor_div(int64_t a, int64_t b) {
    int64_t q = a / b;
    if ((a % b != 0) && (a < 0)) q -= 1;
    return q;
}
int64_t or_floordiv(int64_t a, int64_t b) { return or_floor_div(a, b); }

/* Step 3 ("LSH keys derived from their histograms"; [21]
 * p-stable scheme; integer form R-A5):
 *   h_k = floor((sum_d proj[t][k][d] * hist[d] + bias[t][k]) / w)
 *   x = sm64(t); for k: x = sm64(x ^ (uint32)h_k);  key = x >> (64 - bucket_bits).  */
uint32_t or_lsh_key(const uint32_t* hist, uint32_t t, uint32_t K, const int16_t* proj,
                    const int32_t* bias, int32_t w, uint32_t bucket_bits) {
    uint64_t x = or_sm64_((uint64_t)t);
    for (uint32_t k = 0; k < K; ++k) {
        const int16_t* pr = proj + ((uint64_t)t * K + k) * 768;
        int64_t dot = 0;
        for (uint32_t d = 0; d < 768; ++d) dot += (int64_t)pr[d] * (int64_t)hist[d];
        int64_t h = or_floor_div(dot + bias[(uint64_t)t * K + k], w);
        x = or_sm64_(x ^ (uint64_t)(uint32_t)h);
    }
    return (uint32_t)(x >> (64 - bucket_bits));
}

/* The dataset index ("The dataset images are placed in buckets
 * indexed by the LSH keys derived from their histograms"): per table t a CSR
 * offsets[t*(B+1) + key] .. ids[t*N + ...], ids ascending inside a bucket.
 * Record i's histogram is the 768 uint32 at file + i*rec_stride (R-A1). */
void or_build_index(const uint8_t* file, uint32_t rec_stride, uint64_t N, uint32_t L,
                    uint32_t K, const int16_t* proj, const int32_t* bias, int32_t w,
                    uint32_t bucket_bits, uint32_t* offsets, uint32_t* ids, int threads) {
    uint64_t B = 1ULL << bucket_bits;
    uint32_t* keys = (uint32_t*)malloc(N * sizeof(uint32_t));
    for (uint32_t t = 0; t < L; ++t) {
        #pragma omp parallel for schedule(static) num_threads(threads)
        for (int64_t i = 0; i < (int64_t)N; ++i) {
            uint32_t hist[768];
            memcpy(hist, file + (uint64_t)i * rec_stride, sizeof hist);
            keys[i] = or_lsh_key(hist, t, K, proj, bias, w, bucket_bits);
        }
        uint32_t* off = offsets + (uint64_t)t * (B + 1);
        memset(off, 0, (B + 1) * sizeof(uint32_t));
        for (uint64_t i = 0; i < N; ++i) off[keys[i] + 1] += 1;
        for (uint64_t k = 0; k < B; ++k) off[k + 1] += off[k];
        uint32_t* fill = (uint32_t*)malloc(B * sizeof(uint32_t));
        memcpy(fill, off, B * sizeof(uint32_t));
        for (uint64_t i = 0; i < N; ++i) ids[(uint64_t)t * N + fill[keys[i]]++] = (uint32_t)i;
        free(fill);
    }
    free(keys);
}

/* Step 5 ("Euclidean distance between image color
 * histograms"; squared, integer, R-A2): sum_d (a[d] - b[d])^2. */
uint32_t or_ssd(const uint32_t* a, const uint32_t* b) {
    uint64_t s = 0;
    for (int d = 0; d < 768; ++d) {
        int64_t e = (int64_t)a[d] - (int64_t)b[d];
        s += (uint64_t)(e * e);
    }
    return (uint32_t)s;
}

/* Steps 1-6 for blocks [b0, b0+nb): winners[2*k] = image index,
 * winners[2*k+1] = its distance; (0xFFFFFFFF, 0xFFFFFFFF) if no candidate
 * (R-A4).  Candidates are read at file + id*rec_stride ("reads
 * the candidate histograms from the respective buckets stored in a file"). */
void or_collage(const uint8_t* img, uint32_t W, uint32_t H, uint32_t L, uint32_t K,
                uint32_t bucket_bits, const int16_t* proj, const int32_t* bias, int32_t w,
                const uint8_t* file, uint32_t rec_stride, uint64_t N, const uint32_t* offsets,
                const uint32_t* ids, uint64_t b0, uint64_t nb, uint32_t* winners, int threads) {
    uint64_t B = 1ULL << bucket_bits;
    #pragma omp parallel for schedule(dynamic, 1) num_threads(threads)
    for (int64_t k = 0; k < (int64_t)nb; ++k) {
        uint64_t b = b0 + (uint64_t)k;
        uint32_t hist[768], rec[768];
        or_block_hist(img, W, H, b, hist);
        uint32_t best_idx = 0xFFFFFFFFu, best_dist = 0xFFFFFFFFu;
        for (uint32_t t = 0; t < L; ++t) {
            uint32_t key = or_lsh_key(hist, t, K, proj, bias, w, bucket_bits);
            const uint32_t* off = offsets + (uint64_t)t * (B + 1);
            for (uint32_t j = off[key]; j < off[key + 1]; ++j) {
                uint32_t id = ids[(uint64_t)t * N + j];
                memcpy(rec, file + (uint64_t)id * rec_stride, sizeof rec);
                uint32_t d = or_ssd(hist, rec);
                if (d < best_dist || (d == best_dist && id < best_idx)) {
                    best_dist = d;
                    best_idx = id;
                }
            }
        }
        winners[2 * k] = best_idx;
        winners[2 * k + 1] = best_dist;
    }
}

/* ------------------------------------------------------------------ */
/* Writes (NEXT N3; Fig. 3 `*ptr = 25`): the file after the */
/* benchmark's stores is the file with each stored element replaced --    */
/* plain indexing again (a store through an apointer is a store to the    */
/* file).  Workload definitions as DESIGN.md / include/ap.h.              */
/* ------------------------------------------------------------------ */
static void or_wval(uint64_t seed, uint64_t e, uint32_t elem, uint8_t* out) {
    if (elem == 4) {
        uint32_t v = (uint32_t)or_sm64_(seed ^ e);
        memcpy(out, &v, 4);
    } else if (elem == 8) {
        uint64_t v = or_sm64_(seed ^ e);
        memcpy(out, &v, 8);
    } else {
        uint64_t a = or_sm64_(seed ^ (2 * e)), b = or_sm64_(seed ^ (2 * e + 1));
        memcpy(out, &a, 8);
        memcpy(out + 8, &b, 8);
    }
}

static uint64_t or_gcd(uint64_t a, uint64_t b) {
    while (b) {
        uint64_t t = a % b;
        a = b;
        b = t;
    }
    return a;
}

/* the permutation's multiplier: largest odd a <= floor(M * 0.618...) (the
 * golden-ratio fraction 0x9E3779B97F4A7C15 / 2^64), stepped up by 2 until
 * gcd(a, M) = 1; element k of the write sequence goes to k*a mod M. */
uint64_t or_perm_mult(uint64_t M) {
    uint64_t a = (uint64_t)(((unsigned __int128)M * 0x9E3779B97F4A7C15ull) >> 64) | 1;
    if (a >= M) a = 1;
    while (or_gcd(a, M) != 1) a += 2;
    return a % M;
}

uint64_t or_perm_idx(uint64_t k, uint64_t M) {
    unsigned __int128 A = or_perm_mult(M);
    return (uint64_t)(((unsigned __int128)(k % M) * A) % M);
}

/* pattern 0 (SEQ): every whole element of [0, span); pattern 1 (UNIFORM):
 * element or_perm_idx(t*reads + i, bytes/elem) for t < nthreads, i < reads. */
void or_apply_writes(uint8_t* buf, uint64_t bytes, uint32_t elem, int pattern, uint64_t nthreads,
                     uint32_t reads, uint64_t span, uint64_t seed) {
    if (pattern == 0) {
        for (uint64_t e = 0; (e + 1) * elem <= span; ++e) or_wval(seed, e, elem, buf + e * elem);
    } else {
        uint64_t M = bytes / elem;
        for (uint64_t k = 0; k < nthreads * (uint64_t)reads; ++k) {
            uint64_t e = or_perm_idx(k, M);
            or_wval(seed, e, elem, buf + e * elem);
        }
    }
}

/* ------------------------------------------------------------------ */
/* Compute-intensity workloads (Fig. 6; NEXT N4): the */
/* per-thread accumulators of ap_bench_compute, from their definitions:  */
/* warp w reads pages w, w+W, ...; lane l's j-th element is word         */
/* (page*P/E + 32j + l); a 16-B element is four independent words.       */
/* FFT is the plain O(n^2) DFT in double (tolerance in the test).        */
/* ------------------------------------------------------------------ */
#include <math.h>
#ifndef M_PI
#define M_PI 3.14159265358979323846
#endif

static uint32_t or_lcg_n(uint32_t x, uint32_t n) {
    for (uint32_t i = 0; i < n; ++i) x = x * 1664525u + 1013904223u;
    return x;
}

static int or_cmp_u32(const void* a, const void* b) {
    uint32_t x = *(const uint32_t*)a, y = *(const uint32_t*)b;
    return x < y ? -1 : x > y;
}

/* contribution of one 32-word vector x (one word per lane) to each lane */
static void or_work_vec(int work, const uint32_t* x, const uint32_t* x2, uint32_t iters,
                        double* add_lane) {
    if (work == 0) {
        for (int l = 0; l < 32; ++l) add_lane[l] += (double)x[l] + (double)x2[l];
    } else if (work == 1) {
        for (int l = 0; l < 32; ++l) add_lane[l] += (double)x[l];
    } else if (work == 2) {
        for (int l = 0; l < 32; ++l) add_lane[l] += (double)or_lcg_n(x[l], iters);
    } else if (work == 3) {
        uint32_t s = 0;
        for (int l = 0; l < 32; ++l) s += x[l];
        for (int l = 0; l < 32; ++l) add_lane[l] += (double)s;
    } else if (work == 4) {
        for (int k = 0; k < 32; ++k) {
            double re = 0, im = 0;
            for (int n = 0; n < 32; ++n) {
                double xr = (double)(x[n] & 0xffffu), xi = (double)(x[n] >> 16);
                double ang = -2.0 * M_PI * (double)(n * k % 32) / 32.0;
                re += xr * cos(ang) - xi * sin(ang);
                im += xr * sin(ang) + xi * cos(ang);
            }
            add_lane[k] += floor((re * re + im * im) / 65536.0);
        }
    } else {
        uint32_t s[32];
        memcpy(s, x, sizeof s);
        qsort(s, 32, sizeof(uint32_t), or_cmp_u32);
        for (int l = 0; l < 32; ++l) add_lane[l] += (double)s[l] * (double)(l + 1);
    }
}

/* acc[t] (as double; integer workloads are exact below 2^53) */
void or_compute(const uint8_t* file, uint64_t span, uint32_t unit, uint32_t elem,
                uint64_t nthreads, int work, uint32_t iters, double* acc, int threads) {
    uint64_t W = nthreads / 32;
    uint64_t nunits = span / unit;
    uint32_t per_unit = unit / (32 * elem);
    uint64_t second = span / 4; /* in words */
    const uint32_t* words = (const uint32_t*)file;
    #pragma omp parallel for schedule(dynamic, 1) num_threads(threads)
    for (int64_t w = 0; w < (int64_t)W; ++w) {
        double lanes[32] = {0};
        for (uint64_t u = (uint64_t)w; u < nunits; u += W)
            for (uint32_t j = 0; j < per_unit; ++j)
                for (uint32_t q = 0; q < elem / 4; ++q) {
                    uint32_t x[32], x2[32];
                    for (int l = 0; l < 32; ++l) {
                        uint64_t e = u * (unit / elem) + 32ull * j + l; /* element index */
                        uint64_t wi = e * (elem / 4) + q;               /* word index */
                        x[l] = words[wi];
                        x2[l] = work == 0 ? words[wi + second] : 0;
                    }
                    or_work_vec(work, x, x2, iters, lanes);
                }
        for (int l = 0; l < 32; ++l) acc[w * 32 + l] = lanes[l];
    }
}
