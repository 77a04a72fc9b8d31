/*
 * synth.c — seeded, counter-based synthetic input generator.
 *
 * This module is shared test/bench infrastructure. It holds NONE of the
 * method's arithmetic (no TCA-BME encoding, no SpMM): it only draws the dense
 * fp16 weight matrix W (with an unstructured keep-mask) and the dense fp16
 * activation matrix X that both the CUDA path and the CPU oracle consume.
 *
 * Recipe:
 *   splitmix64(x)      : the standard SplitMix64 finaliser.
 *   key(seed, tag)     = splitmix64(seed) ^ splitmix64(tag)
 *   h(seed, tag, idx)  = splitmix64(key(seed, tag) + idx),  idx = i*cols + j
 *   keep (tag 1)       : keep W[i][j] iff (h >> 11) < floor((1 - s) * 2^53)
 *   W value (tag 2)    : fp16_rne(2 * ((h >> 11) * 2^-53) - 1); a value whose
 *                        bits are +-0 is replaced by 0x3C00 (1.0) so that kept
 *                        entries are always non-zero (reading A7)
 *   X value (tag 3)    : fp16_rne(2 * ((h >> 11) * 2^-53) - 1), dense
 *   "int" mode         : W in {-2,-1,1,2} (tag 2: (h>>11) % 4), X in {-1,0,1}
 *                        (tag 3: (h>>11) % 3 - 1) — integer-exact SpMM cases.
 * Sparsity s = fraction of zeros (NNZ = M*K*(1-s)); i.i.d.
 * uniform positions like the paper's unstructured pruned weights.
 */
#include <stdint.h>
#include <stddef.h>
#include <math.h>
#include <pthread.h>

static inline uint64_t sm64(uint64_t x) {
    uint64_t z = x + 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}

uint64_t synth_splitmix64(uint64_t x) { return sm64(x); }

uint64_t synth_hash(uint64_t seed, uint64_t tag, uint64_t idx) {
    return sm64((sm64(seed) ^ sm64(tag)) + idx);
}

/* IEEE binary64 -> binary16, round-to-nearest-even, for finite |d| < 65520. */
static uint16_t f64_to_f16_rne(double d) {
    union { double d; uint64_t u; } v = { d };
    uint16_t sign = (uint16_t)((v.u >> 48) & 0x8000u);
    uint64_t mag = v.u & 0x7FFFFFFFFFFFFFFFull;
    if (mag == 0) return sign;
    int e = (int)(mag >> 52) - 1023;            /* unbiased exponent */
    uint64_t m = (mag & 0xFFFFFFFFFFFFFull) | (1ull << 52); /* 53-bit significand */
    /* half: normal if e >= -14, value = 1.m10 * 2^e; subnormal: m * 2^-24 */
    int shift;                                   /* bits of m to drop */
    uint16_t he;
    if (e >= -14) { shift = 52 - 10; he = (uint16_t)(e + 15); }
    else          { shift = 52 - 10 + (-14 - e); he = 0; }
    if (shift > 63) return sign;                 /* underflows to zero */
    uint64_t q = m >> shift;
    uint64_t rem = m & ((1ull << shift) - 1);
    uint64_t half = 1ull << (shift - 1);
    if (rem > half || (rem == half && (q & 1))) q++;
    /* q includes the hidden bit for normals (bit 10). */
    uint32_t bits;
    if (he == 0) {
        bits = (uint32_t)q;                      /* may round up into the smallest normal: ok */
    } else {
        if (q >> 11) { q >>= 1; he++; }          /* mantissa overflow */
        bits = ((uint32_t)he << 10) | (uint32_t)(q & 0x3FF);
    }
    return (uint16_t)(sign | bits);
}

uint16_t synth_f64_to_f16(double d) { return f64_to_f16_rne(d); }

static inline double unit_m11(uint64_t h) {       /* uniform in [-1, 1) */
    return 2.0 * ((double)(h >> 11) * 0x1.0p-53) - 1.0;
}

typedef struct {
    uint16_t *out; int64_t rows, cols, r0, r1, row_off;
    uint64_t seed; double s; int mode; int which; /* which: 0 = W, 1 = X */
} job_t;

static void *worker(void *arg) {
    job_t *j = (job_t *)arg;
    const uint64_t thr = (uint64_t)floor((1.0 - j->s) * 9007199254740992.0); /* (1-s)*2^53 */
    const uint64_t k1 = sm64(j->seed) ^ sm64(1), k2 = sm64(j->seed) ^ sm64(2), k3 = sm64(j->seed) ^ sm64(3);
    for (int64_t i = j->r0; i < j->r1; ++i) {
        for (int64_t c = 0; c < j->cols; ++c) {
            uint64_t idx = (uint64_t)((i + j->row_off) * j->cols + c);   /* index in the full matrix */
            uint16_t bits;
            if (j->which == 0) {
                uint64_t hk = sm64(k1 + idx);
                if ((hk >> 11) >= thr) { bits = 0; }
                else {
                    uint64_t hv = sm64(k2 + idx);
                    if (j->mode == 1) {
                        static const uint16_t iv[4] = { 0xC000, 0xBC00, 0x3C00, 0x4000 }; /* -2,-1,1,2 */
                        bits = iv[(hv >> 11) % 4];
                    } else {
                        bits = f64_to_f16_rne(unit_m11(hv));
                        if ((bits & 0x7FFF) == 0) bits = 0x3C00;
                    }
                }
            } else {
                uint64_t hv = sm64(k3 + idx);
                if (j->mode == 1) {
                    static const uint16_t xv[3] = { 0xBC00, 0x0000, 0x3C00 }; /* -1,0,1 */
                    bits = xv[(hv >> 11) % 3];
                } else {
                    bits = f64_to_f16_rne(unit_m11(hv));
                }
            }
            j->out[i * j->cols + c] = bits;
        }
    }
    return NULL;
}

static int run(uint16_t *out, int64_t row_off, int64_t rows, int64_t cols, uint64_t seed, double s,
               int mode, int which, int nthreads) {
    if (!out || rows < 0 || cols < 0 || row_off < 0) return -1;
    if (nthreads < 1) nthreads = 1;
    if (nthreads > 256) nthreads = 256;
    if ((int64_t)nthreads > rows) nthreads = rows > 0 ? (int)rows : 1;
    pthread_t th[256]; job_t jb[256];
    for (int t = 0; t < nthreads; ++t) {
        jb[t] = (job_t){ out, rows, cols, rows * t / nthreads, rows * (t + 1) / nthreads, row_off, seed, s, mode, which };
        if (nthreads == 1) { worker(&jb[t]); return 0; }
        pthread_create(&th[t], NULL, worker, &jb[t]);
    }
    for (int t = 0; t < nthreads; ++t) pthread_join(th[t], NULL);
    return 0;
}

/* W: [rows][cols] row-major fp16 bits. mode 0 = uniform values, 1 = integer values. */
int synth_weight(uint16_t *W, int64_t rows, int64_t cols, uint64_t seed, double sparsity,
                 int mode, int nthreads) {
    if (!(sparsity >= 0.0 && sparsity <= 1.0)) return -1;
    return run(W, 0, rows, cols, seed, sparsity, mode, 0, nthreads);
}

/* Rows [row0, row0 + rows) of the W above (a row shard without generating the whole matrix). */
int synth_weight_rows(uint16_t *W, int64_t row0, int64_t rows, int64_t cols, uint64_t seed, double sparsity,
                      int mode, int nthreads) {
    if (!(sparsity >= 0.0 && sparsity <= 1.0)) return -1;
    return run(W, row0, rows, cols, seed, sparsity, mode, 0, nthreads);
}

/* X: [rows][cols] row-major fp16 bits, dense. */
int synth_activation(uint16_t *X, int64_t rows, int64_t cols, uint64_t seed, int mode, int nthreads) {
    return run(X, 0, rows, cols, seed, 0.0, mode, 1, nthreads);
}
