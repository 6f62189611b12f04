/* Config-5 synthetic banded Markov generator ("Config 5
 * generator"): the same counter-based splitmix64 emission as
 * workloads.banded_markov (the numpy definition, which stays the spec), in C
 * with OpenMP over source states so 100M-row inputs take seconds.  INPUT
 * generation only: it emits off-diagonal rates, never a diagonal, a solve or
 * any other step of the method.  tests/test_workloads.py checks that both
 * produce identical arrays.
 *
 * Per source state j, stream s = seed ^ (j * 0x9E3779B97F4A7C15):
 *   irregular: m = next(s) % (2(mu-3)+1), else m = mu-3;
 *   for off in (-1, +1), if j+off in [0, n): emit j+off with rate(next(s));
 *   then until m more targets or 64*max(m,1) attempts: r = next(s);
 *   k = r % (2w-2); delta = k < w-1 ? k-w : k-w+3; accept j+delta if in range
 *   and not already emitted, with rate(next(s)).
 * rate(r) = 1 + (r >> 11) 2^-53.  Output sorted by column j, then emission. */
#include <stddef.h>
#include <stdint.h>

#define GOLDEN 0x9E3779B97F4A7C15ULL

static inline uint64_t next(uint64_t* s) {
    uint64_t z = (*s += GOLDEN);
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ULL;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBULL;
    return z ^ (z >> 31);
}

static inline double rate_from(uint64_t r) { return 1.0 + (double)(r >> 11) * 0x1.0p-53; }

/* Emits the targets of source j into tgt/rate (capacity cap); returns the count. */
static int emit(int64_t j, int64_t n, int mu, int64_t w, int irregular, uint64_t seed, int cap, int64_t* tgt,
                double* rate) {
    uint64_t s = seed ^ ((uint64_t)j * GOLDEN);
    const int extra = mu - 3;
    const int64_t m = irregular ? (int64_t)(next(&s) % (uint64_t)(2 * extra + 1)) : extra;
    int cnt = 0;
    for (int off = -1; off <= 1; off += 2) {
        if (j + off < 0 || j + off >= n) continue;
        const uint64_t r = next(&s);
        if (tgt) { tgt[cnt] = j + off; rate[cnt] = rate_from(r); }
        ++cnt;
    }
    const int64_t want = cnt + m, max_att = 64 * (m > 1 ? m : 1);
    const uint64_t span = (uint64_t)(2 * w - 2);
    int64_t local[64];
    int64_t* seen = tgt ? tgt : local;
    if (!tgt) {   /* counting pass: keep the targets locally for the duplicate test */
        int c = 0;
        if (j - 1 >= 0) local[c++] = j - 1;
        if (j + 1 < n) local[c++] = j + 1;
    }
    for (int64_t att = 0; cnt < want && att < max_att; ++att) {
        const uint64_t r = next(&s);
        const int64_t k = (int64_t)(r % span);
        const int64_t delta = k < w - 1 ? k - w : 2 + (k - (w - 1));
        const int64_t cand = j + delta;
        if (cand < 0 || cand >= n) continue;
        int dup = 0;
        for (int t = 0; t < cnt; ++t) dup |= seen[t] == cand;
        if (dup) continue;
        const uint64_t rr = next(&s);
        seen[cnt] = cand;
        if (tgt) rate[cnt] = rate_from(rr);
        ++cnt;
    }
    (void)cap;
    return cnt;
}

/* Pass 1: off[j+1] = number of targets of source j, then the prefix sum
 * (off[0] = 0; off has n+1 entries, caller-allocated).  Returns nnz, or -1 on
 * bad arguments. */
int64_t wl_banded_markov_count(int64_t n, int mu, int64_t width, int irregular, uint64_t seed, int64_t* off) {
    if (n < 2 || mu < 3 || width < 2 || 2 * (mu - 3) + 2 > 64) return -1;
    const int64_t w = width < n ? width : n;
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < n; ++j) off[j + 1] = emit(j, n, mu, w, irregular, seed, 0, NULL, NULL);
    off[0] = 0;
    for (int64_t j = 0; j < n; ++j) off[j + 1] += off[j];
    return off[n];
}

/* Pass 2: emission into caller-allocated row/col/rate (off from pass 1). */
void wl_banded_markov_fill(int64_t n, int mu, int64_t width, int irregular, uint64_t seed, const int64_t* off,
                           int32_t* row, int32_t* col, double* rate) {
    const int64_t w = width < n ? width : n;
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < n; ++j) {
        int64_t t[64];
        double r[64];
        const int c = emit(j, n, mu, w, irregular, seed, 64, t, r);
        for (int i = 0; i < c; ++i) {
            row[off[j] + i] = (int32_t)t[i];
            col[off[j] + i] = (int32_t)j;
            rate[off[j] + i] = r[i];
        }
    }
}
