// Network enumerator: reachable microstates of a finitely buffered reaction
// network by DFS (after Cao & Liang [17]) and the off-diagonal rates
// A_k(x_j) = r_k prod_i C(x_i, c_i) (eq. 1).  Readings R7-R10 of
// DESIGN.md fix the buffer rule, the zero-outflow pruning, the DFS order and
// the propensity's index convention.  This is setup (not the hot path); it is
// checked bit-for-bit against the oracle's independent enumerator.
#include <cstring>
#include <memory>

#include "cme_internal.h"

struct cme_coo_s {
    int64_t n = 0, nnz = 0;
    int32_t m = 0;
    std::vector<int32_t> states, row, col;
    std::vector<double> rate;
};

namespace cme {
namespace {

struct Net {
    int m, R;
    const int32_t *x0, *reac, *change, *w;
    const double* rates;
    int64_t cap;
};

// exact binomial C(x, c), c small: product of c consecutive integers / c!
inline uint64_t choose(int64_t x, int32_t c) {
    if (c == 0) return 1;
    if (x < c) return 0;
    uint64_t num = 1;
    for (int32_t i = 0; i < c; ++i) num = num * (uint64_t)(x - i) / (uint64_t)(i + 1);
    return num;
}

inline double rate_of(const Net& N, const int32_t* x, int k) {
    uint64_t prod = 1;
    const int32_t* c = N.reac + (size_t)k * N.m;
    for (int i = 0; i < N.m; ++i) {
        if (c[i]) prod *= choose(x[i], c[i]);
    }
    return N.rates[k] * (double)prod;
}

// Target of reaction k at x (returns false when not enabled).
inline bool fire(const Net& N, const int32_t* x, int k, int32_t* y) {
    if (!(rate_of(N, x, k) > 0.0)) return false;
    const int32_t* nu = N.change + (size_t)k * N.m;
    int64_t load = 0;
    for (int i = 0; i < N.m; ++i) {
        y[i] = x[i] + nu[i];
        if (y[i] < 0) return false;
        load += (int64_t)N.w[i] * y[i];
    }
    return load <= N.cap;
}

class StateSet {
  public:
    explicit StateSet(int m) : m_(m) { rehash(1 << 20); }
    int64_t size() const { return n_; }
    const int32_t* at(int64_t s) const { return data_.data() + s * m_; }
    const std::vector<int32_t>& data() const { return data_; }
    int64_t find(const int32_t* x) const {
        const uint64_t h = hash(x);
        for (uint64_t p = h & mask_;; p = (p + 1) & mask_) {
            const int64_t s = slot_[p];
            if (s < 0) return -1;
            if (hv_[p] == h && std::memcmp(at(s), x, sizeof(int32_t) * m_) == 0) return s;
        }
    }
    int64_t insert(const int32_t* x) {  // caller checked absence
        if (2 * (n_ + 1) > (int64_t)slot_.size()) rehash(slot_.size() * 2);
        data_.insert(data_.end(), x, x + m_);
        place(n_, hash(x));
        return n_++;
    }

  private:
    uint64_t hash(const int32_t* x) const {
        uint64_t h = 0x9E3779B97F4A7C15ull;
        for (int i = 0; i < m_; ++i) {
            h ^= (uint32_t)x[i] + 0x632BE59BD9B4E019ull + (h << 6) + (h >> 2);
            h *= 0xFF51AFD7ED558CCDull;
        }
        return h ^ (h >> 33);
    }
    void place(int64_t s, uint64_t h) {
        uint64_t p = h & mask_;
        while (slot_[p] >= 0) p = (p + 1) & mask_;
        slot_[p] = s;
        hv_[p] = h;
    }
    void rehash(size_t sz) {
        slot_.assign(sz, -1);
        hv_.assign(sz, 0);
        mask_ = sz - 1;
        for (int64_t s = 0; s < n_; ++s) place(s, hash(at(s)));
    }
    int m_;
    int64_t n_ = 0;
    uint64_t mask_ = 0;
    std::vector<int64_t> slot_;
    std::vector<uint64_t> hv_;
    std::vector<int32_t> data_;
};

}  // namespace

cme_status enumerate_network(const Net& N, cme_coo_s& out) {
    StateSet S(N.m);
    std::vector<int32_t> y(N.m);
    S.insert(N.x0);
    // recursive-DFS preorder: (state, next reaction) frames
    std::vector<std::pair<int64_t, int32_t>> st{{0, 0}};
    while (!st.empty()) {
        auto& f = st.back();
        if (f.second == N.R) { st.pop_back(); continue; }
        const int k = f.second++;
        const int64_t j = f.first;
        if (!fire(N, S.at(j), k, y.data()) || S.find(y.data()) >= 0) continue;
        const int64_t id = S.insert(y.data());
        st.emplace_back(id, 0);
    }
    const int64_t n0 = S.size();
    const int R = N.R;
    std::vector<int32_t> tgt((size_t)n0 * R, -1);
    std::vector<int32_t> outdeg(n0, 0);
#pragma omp parallel
    {
        std::vector<int32_t> yy(N.m);
#pragma omp for schedule(static)
        for (int64_t j = 0; j < n0; ++j)
            for (int k = 0; k < R; ++k)
                if (fire(N, S.at(j), k, yy.data())) {
                    tgt[(size_t)j * R + k] = (int32_t)S.find(yy.data());
                    ++outdeg[j];
                }
    }
    // prune zero-outflow states (and edges into them) to the fixpoint with a
    // worklist over reverse edges
    std::vector<int64_t> rptr(n0 + 1, 0);
    for (int64_t e = 0; e < (int64_t)tgt.size(); ++e)
        if (tgt[e] >= 0) ++rptr[tgt[e] + 1];
    for (int64_t i = 0; i < n0; ++i) rptr[i + 1] += rptr[i];
    std::vector<int32_t> rsrc(rptr[n0]);
    {
        std::vector<int64_t> fill(rptr.begin(), rptr.end() - 1);
        for (int64_t e = 0; e < (int64_t)tgt.size(); ++e)
            if (tgt[e] >= 0) rsrc[fill[tgt[e]]++] = (int32_t)(e / R);
    }
    std::vector<char> dead(n0, 0);
    std::vector<int32_t> work;
    for (int64_t j = 0; j < n0; ++j)
        if (outdeg[j] == 0) { dead[j] = 1; work.push_back((int32_t)j); }
    while (!work.empty()) {
        const int32_t s = work.back();
        work.pop_back();
        for (int64_t p = rptr[s]; p < rptr[s + 1]; ++p) {
            const int32_t u = rsrc[p];
            if (!dead[u] && --outdeg[u] == 0) { dead[u] = 1; work.push_back(u); }
        }
    }
    std::vector<int32_t> nid(n0, -1);
    int64_t n = 0;
    for (int64_t j = 0; j < n0; ++j)
        if (!dead[j]) nid[j] = (int32_t)n++;
    out.m = N.m;
    out.n = n;
    out.states.resize((size_t)n * N.m);
    std::vector<int64_t> eoff(n0 + 1, 0);
    for (int64_t j = 0; j < n0; ++j) {
        int64_t c = 0;
        if (!dead[j])
            for (int k = 0; k < R; ++k) {
                const int32_t t = tgt[(size_t)j * R + k];
                c += t >= 0 && !dead[t];
            }
        eoff[j + 1] = eoff[j] + c;
    }
    out.nnz = eoff[n0];
    out.row.resize(out.nnz);
    out.col.resize(out.nnz);
    out.rate.resize(out.nnz);
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < n0; ++j) {
        if (dead[j]) continue;
        const int32_t* xj = S.at(j);
        std::memcpy(out.states.data() + (size_t)nid[j] * N.m, xj, sizeof(int32_t) * N.m);
        int64_t e = eoff[j];
        for (int k = 0; k < R; ++k) {
            const int32_t t = tgt[(size_t)j * R + k];
            if (t < 0 || dead[t]) continue;
            out.row[e] = nid[t];
            out.col[e] = nid[j];
            out.rate[e] = rate_of(N, xj, k);
            ++e;
        }
    }
    return CME_OK;
}

}  // namespace cme

extern "C" cme_status cme_network_enumerate(int m, const int32_t* x0, int R, const int32_t* reac,
                                            const int32_t* change, const double* rates,
                                            const int32_t* w, int64_t cap, cme_coo* out) {
    if (!out || m <= 0 || R <= 0 || !x0 || !reac || !change || !rates || !w) {
        cme::set_error("enumerate: bad arguments");
        return CME_ERR_INVALID_ARG;
    }
    *out = nullptr;
    int64_t load = 0;
    for (int i = 0; i < m; ++i) {
        if (x0[i] < 0) { cme::set_error("enumerate: negative x0"); return CME_ERR_INVALID_ARG; }
        load += (int64_t)w[i] * x0[i];
    }
    if (load > cap) { cme::set_error("enumerate: x0 violates the buffer"); return CME_ERR_INVALID_ARG; }
    for (int k = 0; k < R; ++k) {
        bool moves = false;
        for (int i = 0; i < m; ++i) moves |= change[(size_t)k * m + i] != 0;
        if (!moves || !(rates[k] >= 0.0)) {
            cme::set_error("enumerate: reaction " + std::to_string(k) + " has no net change or a bad rate");
            return CME_ERR_INVALID_ARG;
        }
    }
    try {
        auto c = std::make_unique<cme_coo_s>();
        cme::Net N{m, R, x0, reac, change, w, rates, cap};
        const cme_status st = cme::enumerate_network(N, *c);
        if (st != CME_OK) return st;
        *out = c.release();
        return CME_OK;
    } catch (const std::bad_alloc&) {
        cme::set_error("enumerate: out of host memory");
        return CME_ERR_OOM;
    }
}

extern "C" cme_status cme_coo_get(cme_coo c, int64_t* n, int64_t* nnz, int32_t m[1],
                                  const int32_t** states, const int32_t** row, const int32_t** col,
                                  const double** rate) {
    if (!c) return CME_ERR_INVALID_ARG;
    if (n) *n = c->n;
    if (nnz) *nnz = c->nnz;
    if (m) m[0] = c->m;
    if (states) *states = c->states.data();
    if (row) *row = c->row.data();
    if (col) *col = c->col.data();
    if (rate) *rate = c->rate.data();
    return CME_OK;
}

extern "C" void cme_coo_destroy(cme_coo c) { delete c; }
