// Ingest of off-diagonal transition rates into CSR + diagonal.
//
// Paper: the rate of x_j -> x_i is A(x_i, x_j) = sum_k A_k (eq. 2),
// the diagonal is A(x,x) = -sum_{x' != x} A(x', x) (eq. 4), so the
// columns of A sum to zero.  Readings (R14): duplicates are summed
// in input order, exact-zero sums are dropped, a_jj is the negated sum of
// column j taken in ascending row order.
#include <cmath>
#include <cfloat>
#include <algorithm>

#include "cme_internal.h"

namespace cme {

cme_status ingest_coo(int64_t n, int64_t nnz, const int32_t* row, const int32_t* col,
                      const double* rate, int32_t B, uint32_t flags, Csr& out) {
    const bool given = (flags & CME_DIAG_GIVEN) != 0;
    if (n <= 0 || n > INT32_MAX || nnz < 0 || (nnz > 0 && (!row || !col || !rate)) ||
        (flags & ~CME_DIAG_GIVEN) || B < 1) {
        set_error("ingest: bad sizes, pointers, batch or flags");
        return CME_ERR_INVALID_ARG;
    }
    // validation: the first offending entry decides the status (input order,
    // members in order within an entry)
    for (int64_t e = 0; e < nnz; ++e) {
        const int32_t i = row[e], j = col[e];
        if (i < 0 || i >= n || j < 0 || j >= n) {
            set_error("ingest: index out of range at entry " + std::to_string(e));
            return CME_ERR_INVALID_ARG;
        }
        for (int32_t b = 0; b < B; ++b) {
            const double a = rate[(size_t)b * nnz + e];
            if (!std::isfinite(a)) {
                set_error("ingest: non-finite rate at entry " + std::to_string(e));
                return CME_ERR_INVALID_ARG;
            }
            if (i == j) {
                if (!given) {
                    set_error("ingest: diagonal entry without CME_DIAG_GIVEN at entry " + std::to_string(e));
                    return CME_ERR_INVALID_ARG;
                }
            } else if (a < 0.0) {
                set_error("ingest: negative rate at entry " + std::to_string(e));
                return CME_ERR_NEGATIVE_RATE;
            }
        }
    }
    // bucket entries by row, keeping input order inside a row
    std::vector<int64_t> start(n + 1, 0);
    for (int64_t e = 0; e < nnz; ++e) ++start[row[e] + 1];
    for (int64_t i = 0; i < n; ++i) start[i + 1] += start[i];
    std::vector<int64_t> byrow(nnz);
    {
        std::vector<int64_t> fill(start.begin(), start.end() - 1);
        for (int64_t e = 0; e < nnz; ++e) byrow[fill[row[e]]++] = e;
    }
    // per row: stable order by column; equal columns merge left to right,
    // per member; an entry is stored if any member's sum is non-zero
    auto rate_of = [&](int64_t e, int32_t b) { return rate[(size_t)b * nnz + e]; };
    std::vector<int64_t> cnt(n + 1, 0);
    std::vector<double> gdiag(given ? (size_t)n * B : 0, 0.0);
#pragma omp parallel
    {
        std::vector<double> s(B);
#pragma omp for schedule(dynamic, 4096)
        for (int64_t i = 0; i < n; ++i) {
            int64_t* b0 = byrow.data() + start[i];
            int64_t* e0 = byrow.data() + start[i + 1];
            std::stable_sort(b0, e0, [&](int64_t p, int64_t q) { return col[p] < col[q]; });
            int64_t kept = 0;
            for (int64_t* p = b0; p < e0;) {
                const int32_t j = col[*p];
                std::fill(s.begin(), s.end(), 0.0);
                for (; p < e0 && col[*p] == j; ++p)
                    for (int32_t b = 0; b < B; ++b) s[b] += rate_of(*p, b);
                bool nz = false;
                for (int32_t b = 0; b < B; ++b) nz |= s[b] != 0.0;
                if (j == i) {  // only reachable with CME_DIAG_GIVEN
                    for (int32_t b = 0; b < B; ++b) gdiag[(size_t)i * B + b] = s[b];
                } else if (nz) {
                    ++kept;
                }
            }
            cnt[i + 1] = kept;
        }
    }
    out.n = n;
    out.B = B;
    out.rp.assign(n + 1, 0);
    for (int64_t i = 0; i < n; ++i) out.rp[i + 1] = out.rp[i] + cnt[i + 1];
    out.ci.resize(out.rp[n]);
    out.v.resize((size_t)out.rp[n] * B);
#pragma omp parallel
    {
        std::vector<double> s(B);
#pragma omp for schedule(dynamic, 4096)
        for (int64_t i = 0; i < n; ++i) {
            const int64_t* b0 = byrow.data() + start[i];
            const int64_t* e0 = byrow.data() + start[i + 1];
            int64_t o = out.rp[i];
            for (const int64_t* p = b0; p < e0;) {
                const int32_t j = col[*p];
                std::fill(s.begin(), s.end(), 0.0);
                for (; p < e0 && col[*p] == j; ++p)
                    for (int32_t b = 0; b < B; ++b) s[b] += rate_of(*p, b);
                bool nz = false;
                for (int32_t b = 0; b < B; ++b) nz |= s[b] != 0.0;
                if (j != i && nz) {
                    out.ci[o] = j;
                    for (int32_t b = 0; b < B; ++b) out.v[(size_t)o * B + b] = s[b];
                    ++o;
                }
            }
        }
    }
    // column sums in ascending row order: transpose (stable by row) then sum
    std::vector<int64_t> cstart(n + 1, 0);
    for (int64_t p = 0; p < out.rp[n]; ++p) ++cstart[out.ci[p] + 1];
    for (int64_t j = 0; j < n; ++j) cstart[j + 1] += cstart[j];
    std::vector<int64_t> tp(out.rp[n]);
    {
        std::vector<int64_t> fill(cstart.begin(), cstart.end() - 1);
        for (int64_t i = 0; i < n; ++i)
            for (int64_t p = out.rp[i]; p < out.rp[i + 1]; ++p) tp[fill[out.ci[p]]++] = p;
    }
    out.d.assign((size_t)n * B, 0.0);
    int64_t bad_zero = -1, bad_diag = -1;
#pragma omp parallel for schedule(static) reduction(max : bad_zero, bad_diag)
    for (int64_t j = 0; j < n; ++j) {
        for (int32_t b = 0; b < B; ++b) {
            double s = 0.0;
            for (int64_t q = cstart[j]; q < cstart[j + 1]; ++q) s += out.v[(size_t)tp[q] * B + b];
            if (s == 0.0) { bad_zero = std::max(bad_zero, n - j); break; }
            if (!given) {
                out.d[(size_t)j * B + b] = -s;
            } else {
                const double dj = gdiag[(size_t)j * B + b];
                out.d[(size_t)j * B + b] = dj;
                if (!(dj < 0.0) || std::fabs(s + dj) > 64.0 * DBL_EPSILON * std::fabs(dj))
                    bad_diag = std::max(bad_diag, n - j);
            }
        }
    }
    // report the smallest offending state, zero outflow first (like a serial scan)
    if (bad_zero > 0 || bad_diag > 0) {
        const int64_t jz = bad_zero > 0 ? n - bad_zero : n, jd = bad_diag > 0 ? n - bad_diag : n;
        if (jz <= jd) {
            set_error("ingest: state " + std::to_string(jz) + " has zero outflow");
            return CME_ERR_ZERO_OUTFLOW;
        }
        set_error("ingest: given diagonal of state " + std::to_string(jd) + " is not -colsum");
        return CME_ERR_INVALID_ARG;
    }
    return CME_OK;
}

}  // namespace cme
