// Network enumerator: reachable microstates of a finitely buffered reaction
// network by DFS (after Cao & Liang [17]) and the off-diagonal rates
// A_k(x_j) = r_k prod_i C(x_i, c_i) (eq. 1).  Readings R7-R10 of
// DESIGN.md fix the buffer rule, the zero-outflow pruning, the DFS order and
// the propensity's index convention.  This is setup (not the hot path); it is
// checked bit-for-bit against the oracle's independent enumerator.
#include <sys/mman.h>

#include <cstdlib>
#include <cstring>
#include <memory>

#include "cme_internal.h"

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

// Hash set of microstates.  States with m <= 8 species and counts < 2^16 are
// packed into a 128-bit key kept inside the slot, so a probe touches one cache
// line (the tables of 20M-state networks are GBs: every miss is a DRAM + TLB
// miss; the slot array asks for transparent huge pages).
class StateSet {
  public:
    explicit StateSet(int m) : m_(m), packed_(m <= 8) { rehash(1 << 20); }
    ~StateSet() { std::free(slot_); }
    StateSet(const StateSet&) = delete;
    StateSet& operator=(const StateSet&) = delete;
    int64_t size() const { return n_; }
    const int32_t* at(int64_t s) const { return data_.data() + s * m_; }
    bool packed() const { return packed_; }
    int64_t find(const int32_t* x) const {
        Key k;
        if (!make_key(x, k)) return -1;
        for (uint64_t p = k.h & mask_;; p = (p + 1) & mask_) {
            const Slot& e = slot_[p];
            if (e.s < 0) return -1;
            if (e.h == k.h && (packed_ ? (e.a == k.a && e.b == k.b)
                                       : std::memcmp(at(e.s), x, sizeof(int32_t) * m_) == 0))
                return e.s;
        }
    }
    // caller checked absence; returns -1 if the state cannot be packed (caller
    // then restarts in generic mode)
    int64_t insert(const int32_t* x) {
        Key k;
        if (!make_key(x, k)) return -1;
        if (2 * (n_ + 1) > (int64_t)(mask_ + 1)) rehash(2 * (mask_ + 1));
        data_.insert(data_.end(), x, x + m_);
        place(Slot{k.h, n_, k.a, k.b});
        return n_++;
    }
    void set_generic() { packed_ = false; }

  private:
    struct Key {
        uint64_t h, a, b;
    };
    struct Slot {
        uint64_t h;
        int64_t s;
        uint64_t a, b;
    };
    static uint64_t mix(uint64_t z) {
        z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
        z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
        return z ^ (z >> 31);
    }
    bool make_key(const int32_t* x, Key& k) const {
        if (packed_) {
            uint64_t a = 0, b = 0;
            for (int i = 0; i < m_; ++i) {
                if ((uint32_t)x[i] >= 65536u) return false;
                if (i < 4) a |= (uint64_t)x[i] << (16 * i);
                else b |= (uint64_t)x[i] << (16 * (i - 4));
            }
            k.a = a;
            k.b = b;
            k.h = mix(a ^ mix(b + 0x9E3779B97F4A7C15ull));
            return true;
        }
        uint64_t h = 0x9E3779B97F4A7C15ull;
        for (int i = 0; i < m_; ++i) h = mix(h ^ (uint32_t)x[i]);
        k.h = h;
        k.a = k.b = 0;
        return true;
    }
    void place(const Slot& e) {
        uint64_t p = e.h & mask_;
        while (slot_[p].s >= 0) p = (p + 1) & mask_;
        slot_[p] = e;
    }
    void rehash(size_t sz) {
        Slot* old = slot_;
        const size_t old_n = slot_ ? mask_ + 1 : 0;
        const size_t bytes = sz * sizeof(Slot);
        void* mem = nullptr;
        if (posix_memalign(&mem, 1 << 21, bytes) != 0) throw std::bad_alloc();
        madvise(mem, bytes, MADV_HUGEPAGE);
        slot_ = static_cast<Slot*>(mem);
        for (size_t i = 0; i < sz; ++i) slot_[i].s = -1;
        mask_ = sz - 1;
        for (size_t i = 0; i < old_n; ++i)
            if (old[i].s >= 0) place(old[i]);
        std::free(old);
    }
    int m_;
    bool packed_;
    int64_t n_ = 0;
    uint64_t mask_ = 0;
    Slot* slot_ = nullptr;
    std::vector<int32_t> data_;
};

struct Unpackable {};

}  // namespace

cme_status enumerate_network(const Net& N, cme_coo_s& out, bool generic);

cme_status enumerate_network(const Net& N, cme_coo_s& out) {
    try {
        return enumerate_network(N, out, false);
    } catch (const Unpackable&) {
        return enumerate_network(N, out, true);
    }
}

cme_status enumerate_network(const Net& N, cme_coo_s& out, bool generic) {
    StateSet S(N.m);
    if (generic) S.set_generic();
    const int R = N.R;
    std::vector<int32_t> y(N.m);
    std::vector<int32_t> tgt;                   // tgt[j*R + k]: target of reaction k at j, -1 = disabled
    std::vector<int32_t> outdeg;
    auto add = [&](const int32_t* x) {
        const int64_t id = S.insert(x);
        if (id < 0) throw Unpackable();
        tgt.resize((size_t)S.size() * R, -1);
        outdeg.resize(S.size(), 0);
        return id;
    };
    add(N.x0);
    // recursive-DFS preorder: (state, next reaction) frames; every (state,
    // reaction) pair is tried exactly once, so its target is recorded here
    std::vector<std::pair<int64_t, int32_t>> st{{0, 0}};
    while (!st.empty()) {
        auto& f = st.back();
        if (f.second == R) { st.pop_back(); continue; }
        const int k = f.second++;
        const int64_t j = f.first;
        if (!fire(N, S.at(j), k, y.data())) continue;
        int64_t id = S.find(y.data());   // (an unpackable y is "absent"; add() then restarts)
        const bool fresh = id < 0;
        if (fresh) id = add(y.data());
        tgt[(size_t)j * R + k] = (int32_t)id;
        ++outdeg[j];
        if (fresh) st.emplace_back(id, 0);
    }
    const int64_t n0 = S.size();
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
