// Host packer: DIAG band + warp-grained sliced ELL with local rearrangement.
//
// Paper: ELL column-major arrays padded to a warp multiple, DIA for
// the dense {-1,0,+1} band when its density beats 8 B / 12 B = 2/3,
// sliced ELL with slice = warp decoupled from the block, rows
// rearranged inside a block to even out slice widths.  The exact
// layout ("v0") is frozen in DESIGN.md section 5 so that the oracle packer and
// this one agree byte for byte.
#include <algorithm>
#include <cstring>
#include <unordered_map>
#include <unordered_set>

#include "cme_internal.h"

namespace cme {

namespace {
// Position of column c in row r of A (columns ascending), or -1.  Stored
// entries are non-zero (in at least one batch member), so presence = A_rc != 0.
inline int64_t entry(const Csr& A, int64_t r, int64_t c) {
    const int32_t* b = A.ci.data() + A.rp[r];
    const int32_t* e = A.ci.data() + A.rp[r + 1];
    const int32_t* p = std::lower_bound(b, e, (int32_t)c);
    return (p != e && *p == c) ? A.rp[r] + (p - b) : -1;
}
}  // namespace

bool band_rule(const Csr& A, int band_mode) {
    if (band_mode == CME_BAND_ALWAYS) return true;
    if (band_mode == CME_BAND_NEVER) return false;
    const int64_t n = A.n;
    int64_t cnt = 0;
#pragma omp parallel for reduction(+ : cnt) schedule(static)
    for (int64_t i = 0; i < n; ++i)
        cnt += (i > 0 && entry(A, i, i - 1) >= 0) + (i + 1 < n && entry(A, i, i + 1) >= 0);
    const int64_t den = 2 * n - 2;
    return den > 0 && 3 * cnt >= 2 * den;
}

void pack_rows(const Csr& A, int64_t r0, int64_t r1, int64_t col_shift, int32_t window,
               bool band_on, int32_t group, int32_t global_kmax, Packed& P) {
    const int64_t n = r1 - r0;  // local rows
    P = Packed();
    P.n = n;
    P.band_on = band_on;
    P.window = window > 1 ? window : 1;
    P.group = group;
    const int32_t nb = A.B;
    P.B = nb;
    P.n_slots = (n + 31) / 32 * 32;
    P.n_slices = P.n_slots / 32;
    std::vector<int32_t> c(n);
#pragma omp parallel for schedule(static)
    for (int64_t l = 0; l < n; ++l) {
        const int64_t r = r0 + l;
        int64_t k = A.rp[r + 1] - A.rp[r];
        if (band_on) k -= (r > 0 && entry(A, r, r - 1) >= 0) + (r + 1 < A.n && entry(A, r, r + 1) >= 0);
        c[l] = (int32_t)k;
    }
    // local rearrangement: each window's slots take its rows by (-c, row)
    P.row_of.resize(P.n_slots);
    for (int64_t s = 0; s < P.n_slots; ++s) P.row_of[s] = (int32_t)s;
    if (P.window > 1) {
        const int64_t W = P.window;
#pragma omp parallel for schedule(static)
        for (int64_t w0 = 0; w0 < n; w0 += W) {
            int32_t* b = P.row_of.data() + w0;
            int32_t* e = P.row_of.data() + std::min(w0 + W, n);
            std::stable_sort(b, e, [&](int32_t a, int32_t bb) { return c[a] > c[bb]; });
        }
    }
    // slice width = exact max ELL count of its rows; `group` slices
    // share their max (8 = the 256-row block-sliced ELL of [5]); 0 = global width
    P.slice_w.assign(P.n_slices, 0);
    P.slice_off.assign(P.n_slices + 1, 0);
    for (int64_t q = 0; q < P.n_slices; ++q) {
        int32_t w = 0;
        for (int64_t s = q * 32; s < std::min(q * 32 + 32, n); ++s) w = std::max(w, c[P.row_of[s]]);
        P.slice_w[q] = group == 0 ? global_kmax : w;
    }
    if (group > 1)
        for (int64_t g0 = 0; g0 < P.n_slices; g0 += group) {
            const int64_t g1 = std::min<int64_t>(g0 + group, P.n_slices);
            const int32_t wg = *std::max_element(P.slice_w.begin() + g0, P.slice_w.begin() + g1);
            std::fill(P.slice_w.begin() + g0, P.slice_w.begin() + g1, wg);
        }
    for (int64_t q = 0; q < P.n_slices; ++q) P.slice_off[q + 1] = P.slice_off[q] + 32 * (int64_t)P.slice_w[q];
    P.n_ell = P.slice_off[P.n_slices];
    // values are member-minor: val[e*B + b], lo/up/inv_d[s*B + b]
    P.val.assign((size_t)P.n_ell * nb, 0.0);
    P.col.assign(P.n_ell, 0);
    P.lo.assign((size_t)P.n_slots * nb, 0.0);
    P.up.assign((size_t)P.n_slots * nb, 0.0);
    P.inv_d.assign((size_t)P.n_slots * nb, 0.0);
    P.dneg.assign((size_t)P.n_slots * nb, 0.0);
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t s = 0; s < P.n_slots; ++s) {
        const int64_t q = s >> 5, lane = s & 31;
        const int64_t e0 = P.slice_off[q] + lane;   // entry t of this slot: e0 + 32 t
        int32_t* cq = P.col.data() + e0;
        const int32_t w = P.slice_w[q];
        if (s >= n) {  // pad slot beyond the last row
            for (int32_t t = 0; t < w; ++t) cq[32 * t] = (int32_t)(r1 - 1 - col_shift);
            continue;
        }
        const int64_t l = P.row_of[s], r = r0 + l;
        for (int32_t b = 0; b < nb; ++b) {
            P.inv_d[(size_t)s * nb + b] = 1.0 / (-A.d[(size_t)r * nb + b]);
            P.dneg[(size_t)s * nb + b] = -A.d[(size_t)r * nb + b];
        }
        if (band_on) {
            const int64_t pl = r > 0 ? entry(A, r, r - 1) : -1, pu = r + 1 < A.n ? entry(A, r, r + 1) : -1;
            for (int32_t b = 0; b < nb; ++b) {
                P.lo[(size_t)s * nb + b] = pl >= 0 ? A.v[(size_t)pl * nb + b] : 0.0;
                P.up[(size_t)s * nb + b] = pu >= 0 ? A.v[(size_t)pu * nb + b] : 0.0;
            }
        }
        int32_t t = 0;
        for (int64_t p = A.rp[r]; p < A.rp[r + 1]; ++p) {
            const int64_t j = A.ci[p];
            if (band_on && (j == r - 1 || j == r + 1)) continue;
            for (int32_t b = 0; b < nb; ++b) P.val[(size_t)(e0 + 32 * t) * nb + b] = A.v[(size_t)p * nb + b];
            cq[32 * t] = (int32_t)(j - col_shift);
            ++t;
        }
        for (; t < w; ++t) cq[32 * t] = (int32_t)(r - col_shift);
    }
}

bool encode_compact(const Packed& P, int64_t own_off, Compact& C) {
    C = Compact();
    if (P.n_slices == 0 || P.dneg.size() != (size_t)P.n_slots * P.B) return false;
    int32_t ws = 0;
    if (P.window > 1) {
        if (P.window > 256 || (P.window & (P.window - 1))) return false;
        while ((1 << ws) < P.window) ++ws;
    }
    const int64_t n = P.n;
    // every stored offset j - r must fit int16 (pad entries hold their own row: 0)
    bool ok = true;
#pragma omp parallel for schedule(dynamic, 256) reduction(&& : ok)
    for (int64_t s = 0; s < n; ++s) {
        const int64_t q = s >> 5, e0 = P.slice_off[q] + (s & 31), r = own_off + P.row_of[s];
        for (int32_t t = 0; t < P.slice_w[q]; ++t) {
            const int64_t dlt = (int64_t)P.col[e0 + 32 * t] - r;
            ok = ok && dlt >= INT16_MIN && dlt <= INT16_MAX;
        }
    }
    if (!ok) return false;
    C.valid = true;
    C.win_shift = ws;
    C.col16.assign(P.n_ell, 0);
    if (ws) C.row8.assign(P.n_slots, 0);
    if (P.B != 1) {   // a batch: the (shared) offsets only -- its values go through the value index
#pragma omp parallel for schedule(dynamic, 256)
        for (int64_t s = 0; s < n; ++s) {
            const int64_t q = s >> 5, e0 = P.slice_off[q] + (s & 31), l = P.row_of[s], r = own_off + l;
            for (int32_t t = 0; t < P.slice_w[q]; ++t)
                C.col16[e0 + 32 * t] = (int16_t)((int64_t)P.col[e0 + 32 * t] - r);
            if (ws) C.row8[s] = (uint8_t)(l - ((s >> ws) << ws));
        }
        return true;
    }
    C.val.assign(P.n_ell, 0.0);
    if (P.band_on) {
        C.lo.assign(P.n_slots, 0.0);
        C.up.assign(P.n_slots, 0.0);
    }
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t s = 0; s < n; ++s) {
        const int64_t q = s >> 5, e0 = P.slice_off[q] + (s & 31), l = P.row_of[s], r = own_off + l;
        const double dn = P.dneg[s];
        for (int32_t t = 0; t < P.slice_w[q]; ++t) {
            const int64_t e = e0 + 32 * t;
            C.val[e] = P.val[e] / dn;
            C.col16[e] = (int16_t)((int64_t)P.col[e] - r);
        }
        if (P.band_on) {
            C.lo[s] = P.lo[s] / dn;
            C.up[s] = P.up[s] / dn;
        }
        if (ws) C.row8[s] = (uint8_t)(l - ((s >> ws) << ws));
    }
    return true;
}

namespace {
// a stored entry's B-tuple of values (batch member b at w[b]), by bit pattern
struct VKey {
    uint64_t w[8];
    bool operator==(const VKey& o) const { return std::memcmp(w, o.w, sizeof(w)) == 0; }
};
struct VKeyHash {
    size_t operator()(const VKey& k) const {
        uint64_t h = 0x9E3779B97F4A7C15ull;
        for (uint64_t v : k.w) { h ^= v + 0x9E3779B97F4A7C15ull + (h << 6) + (h >> 2); }
        return (size_t)h;
    }
};
inline VKey vkey(const double* v, int B) {
    VKey k{};
    std::memcpy(k.w, v, sizeof(double) * B);
    return k;
}
}  // namespace

bool encode_value_index(const Packed& P, Compact& C) {
    C.vi_valid = false;
    C.dict.clear(); C.vidx.clear(); C.loi.clear(); C.upi.clear();
    const int B = P.B;
    if (!C.valid || B < 1 || B > 8) return false;
    constexpr size_t kMax = 65536;
    // distinct B-tuples (B = 1: distinct values) of the stored entries; all
    // stored values are finite and +0.0 or > 0
    std::unordered_set<VKey, VKeyHash> all;
    bool over = false;
#pragma omp parallel
    {
        std::unordered_set<VKey, VKeyHash> mine;
#pragma omp for schedule(static) nowait
        for (int64_t e = 0; e < P.n_ell; ++e) {
            if (mine.size() > kMax) continue;
            mine.insert(vkey(P.val.data() + (size_t)e * B, B));
        }
        if (P.band_on) {
#pragma omp for schedule(static) nowait
            for (int64_t s = 0; s < P.n_slots; ++s) {
                if (mine.size() > kMax) continue;
                mine.insert(vkey(P.lo.data() + (size_t)s * B, B));
                mine.insert(vkey(P.up.data() + (size_t)s * B, B));
            }
        }
#pragma omp critical
        {
            if (mine.size() > kMax) over = true;
            if (!over) all.insert(mine.begin(), mine.end());
            if (all.size() > kMax) over = true;
        }
    }
    if (over) return false;
    // ascending lexicographic order of the tuples (member 0 first)
    std::vector<VKey> keys(all.begin(), all.end());
    auto as_d = [](const VKey& k, int b) { double v; std::memcpy(&v, &k.w[b], 8); return v; };
    std::sort(keys.begin(), keys.end(), [&](const VKey& a, const VKey& b) {
        for (int m = 0; m < B; ++m) {
            const double x = as_d(a, m), y = as_d(b, m);
            if (x != y) return x < y;
        }
        return false;
    });
    std::unordered_map<VKey, uint16_t, VKeyHash> where;
    where.reserve(keys.size() * 2);
    std::vector<double> dict((size_t)keys.size() * B);
    for (size_t i = 0; i < keys.size(); ++i) {
        where[keys[i]] = (uint16_t)i;
        for (int m = 0; m < B; ++m) dict[i * B + m] = as_d(keys[i], m);
    }
    C.vidx.resize(P.n_ell);
#pragma omp parallel for schedule(static)
    for (int64_t e = 0; e < P.n_ell; ++e) C.vidx[e] = where.find(vkey(P.val.data() + (size_t)e * B, B))->second;
    if (P.band_on) {
        C.loi.resize(P.n_slots);
        C.upi.resize(P.n_slots);
#pragma omp parallel for schedule(static)
        for (int64_t s = 0; s < P.n_slots; ++s) {
            C.loi[s] = where.find(vkey(P.lo.data() + (size_t)s * B, B))->second;
            C.upi[s] = where.find(vkey(P.up.data() + (size_t)s * B, B))->second;
        }
    }
    C.dict = std::move(dict);
    C.vi_valid = true;
    return true;
}

void pack_csr_rows(const Csr& A, int64_t r0, int64_t r1, int64_t col_shift, Packed& P) {
    const int64_t n = r1 - r0;
    P = Packed();
    P.n = n;
    P.n_slots = (n + 31) / 32 * 32;
    P.n_slices = P.n_slots / 32;
    P.csr_rp.resize(n + 1);
    const int64_t base = A.rp[r0];
    for (int64_t l = 0; l <= n; ++l) P.csr_rp[l] = A.rp[r0 + l] - base;
    P.csr_ci.resize(P.csr_rp[n]);
    P.csr_v.assign(A.v.begin() + base, A.v.begin() + base + P.csr_rp[n]);  // (CSR arm: B = 1 only)
    for (int64_t p = 0; p < P.csr_rp[n]; ++p) P.csr_ci[p] = (int32_t)(A.ci[base + p] - col_shift);
    P.inv_d.assign(P.n_slots, 0.0);
    for (int64_t l = 0; l < n; ++l) P.inv_d[l] = 1.0 / (-A.d[r0 + l]);
    P.row_of.resize(P.n_slots);
    for (int64_t s = 0; s < P.n_slots; ++s) P.row_of[s] = (int32_t)s;
}

}  // namespace cme
