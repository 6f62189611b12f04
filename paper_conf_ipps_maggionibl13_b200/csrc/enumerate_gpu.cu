// GPU state enumerator: the reachable microstates of a
// finitely buffered reaction network (after Cao & Liang [17]), their
// off-diagonal rates A_k(x_j) = r_k prod_i C(x_i, c_i) (eq. 1) and the
// zero-outflow pruning of reading R8 -- the same set, rates and pruning as the
// host DFS enumerator (enumerate.cpp), computed on the GPU:
//
//   1. level-synchronous BFS from x0: one thread per (frontier state,
//      reaction) fires the reaction (reading R7: enabled iff A_k(x) > 0,
//      x + nu >= 0 and w.(x + nu) <= cap) and inserts the target's 128-bit
//      key (16 bits per species, species 0 most significant) into an
//      open-addressing hash table with a 128-bit atomicCAS; a fresh insert
//      appends the key to the discovery list and the next frontier;
//   2. the discovered keys are radix-sorted (two stable 64-bit passes), so
//      state numbers follow the lexicographic order of (x_0, ..., x_{m-1}) --
//      deterministic, independent of the parallel discovery order;
//   3. one thread per (state, reaction) looks its target's number up in the
//      table (which now stores the sorted position);
//   4. zero-outflow states and the edges into them are removed to a fixpoint;
//   5. the survivors are compacted (order kept) and the COO triplets emitted
//      per source state in reaction order, rates by the same exact integer
//      binomials and one fp64 multiply as the host enumerator (bit-identical).
//
// The numbering differs from the host's DFS preorder; cme_reorder
// supplies DFS / RCM orderings of the resulting matrix.  Setup, not the
// Jacobi hot path.
#include <cub/device/device_radix_sort.cuh>
#include <cub/device/device_scan.cuh>

#include <memory>
#include <string>

#include "cme_internal.h"

namespace cme {
namespace {

constexpr int kMaxSpecies = 8;
constexpr int kMaxReactions = 64;
typedef unsigned __int128 u128;
constexpr uint32_t kMaxCount = 65534;   // 0xFFFF fields are reserved for the empty key

struct GNet {
    int m, R;
    int64_t cap;
    int32_t x0[kMaxSpecies];
    int32_t w[kMaxSpecies];
    int32_t reac[kMaxReactions * kMaxSpecies];
    int32_t change[kMaxReactions * kMaxSpecies];
    double rates[kMaxReactions];
};

__device__ __forceinline__ u128 empty_key() { return ~(u128)0; }

__device__ __forceinline__ u128 pack_key(const int32_t* x, int m) {
    u128 k = 0;
    for (int i = 0; i < kMaxSpecies; ++i) k = (k << 16) | (u128)(i < m ? (uint32_t)x[i] : 0u);
    return k;
}
__device__ __forceinline__ void unpack_key(u128 k, int m, int32_t* x) {
    for (int i = kMaxSpecies - 1; i >= 0; --i) {
        if (i < m) x[i] = (int32_t)(uint32_t)(k & 0xFFFF);
        k >>= 16;
    }
}
__device__ __forceinline__ uint64_t mix64(uint64_t z) {
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
__device__ __forceinline__ uint64_t hash_key(u128 k) {
    return mix64((uint64_t)k ^ mix64((uint64_t)(k >> 64) + 0x9E3779B97F4A7C15ull));
}

// exact binomial C(x, c) for small c (same recurrence as the host enumerator)
__device__ __forceinline__ uint64_t choose_d(int64_t x, int32_t c) {
    if (c == 0) return 1;
    if (x < c) return 0;
    uint64_t num = 1;
    for (int32_t i = 0; i < c; ++i) num = num * (uint64_t)(x - i) / (uint64_t)(i + 1);
    return num;
}
__device__ __forceinline__ double rate_d(const GNet& N, const int32_t* x, int k) {
    uint64_t prod = 1;
    for (int i = 0; i < N.m; ++i) {
        const int32_t c = N.reac[k * N.m + i];
        if (c) prod *= choose_d(x[i], c);
    }
    return N.rates[k] * (double)prod;
}
// target of reaction k at x; false when not enabled.  *over: a count beyond the key range
__device__ __forceinline__ bool fire_d(const GNet& N, const int32_t* x, int k, int32_t* y, int* over) {
    if (!(rate_d(N, x, k) > 0.0)) return false;
    int64_t load = 0;
    for (int i = 0; i < N.m; ++i) {
        y[i] = x[i] + N.change[k * N.m + i];
        if (y[i] < 0) return false;
        load += (int64_t)N.w[i] * y[i];
    }
    if (load > N.cap) return false;
    for (int i = 0; i < N.m; ++i)
        if ((uint32_t)y[i] > kMaxCount) { atomicExch(over, 1); return false; }
    return true;
}

struct Table {
    u128* key;
    int64_t* val;
    uint64_t mask;
};

// insert; true if this call inserted the key.  Slot ownership is decided by
// the 128-bit atomicCAS alone: a plain 128-bit load is not single-copy atomic
// in the PTX memory model, so a load racing another thread's insert could tear
// into a value that is neither empty nor k.  The plain load only short-cuts
// the common case "already here": a slot changes once, empty -> key, so a
// torn load mixes one half of a key with one all-ones half of the empty key,
// and no valid key has an all-ones half (counts <= kMaxCount < 0xFFFF).
__device__ __forceinline__ bool table_insert(const Table& T, u128 k) {
    for (uint64_t p = hash_key(k) & T.mask;; p = (p + 1) & T.mask) {
        if (T.key[p] == k) return false;
        const u128 old = atomicCAS(&T.key[p], empty_key(), k);
        if (old == empty_key()) return true;
        if (old == k) return false;
        // another key owns the slot (single-copy atomic CAS result): probe on
    }
}
__device__ __forceinline__ int64_t table_find(const Table& T, u128 k) {
    for (uint64_t p = hash_key(k) & T.mask;; p = (p + 1) & T.mask) {
        const u128 cur = T.key[p];
        if (cur == k) return T.val[p];
        if (cur == empty_key()) return -1;
    }
}

__global__ void fill_empty_kernel(u128* key, uint64_t n) {
    for (uint64_t i = blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
        key[i] = ~(u128)0;
}

__global__ void seed_kernel(const GNet N, Table T, u128* all, u128* front) {
    const u128 k = pack_key(N.x0, N.m);
    table_insert(T, k);
    all[0] = k;
    front[0] = k;
}

// one thread per (frontier state, reaction)
__global__ void expand_kernel(const GNet N, Table T, const u128* front, int64_t nfront, u128* next,
                              unsigned long long* nnext, u128* all, unsigned long long* nall, int* over) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < nfront * N.R;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t f = t / N.R;
        const int k = (int)(t % N.R);
        int32_t x[kMaxSpecies], y[kMaxSpecies];
        unpack_key(front[f], N.m, x);
        if (!fire_d(N, x, k, y, over)) continue;
        const u128 key = pack_key(y, N.m);
        if (table_insert(T, key)) {
            next[atomicAdd(nnext, 1ull)] = key;
            all[atomicAdd(nall, 1ull)] = key;
        }
    }
}

__global__ void reinsert_kernel(Table T, const u128* all, int64_t n) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x)
        table_insert(T, all[i]);
}

__global__ void split_kernel(const u128* k, int64_t n, uint64_t* hi, uint64_t* lo) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        hi[i] = (uint64_t)(k[i] >> 64);
        lo[i] = (uint64_t)k[i];
    }
}

// sorted position -> table value; states array
__global__ void number_kernel(const GNet N, Table T, const uint64_t* hi, const uint64_t* lo, int64_t n,
                              int32_t* states) {
    for (int64_t i = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; i < n; i += (int64_t)gridDim.x * blockDim.x) {
        const u128 k = ((u128)hi[i] << 64) | lo[i];
        for (uint64_t p = hash_key(k) & T.mask;; p = (p + 1) & T.mask)
            if (T.key[p] == k) { T.val[p] = i; break; }
        unpack_key(k, N.m, states + i * N.m);
    }
}

// tgt[j*R + k] = number of the target of reaction k at state j (or -1); outdeg[j]
__global__ void edges_kernel(const GNet N, Table T, const int32_t* states, int64_t n, int32_t* tgt, int32_t* outdeg) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n * N.R;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int64_t j = t / N.R;
        const int k = (int)(t % N.R);
        int32_t y[kMaxSpecies];
        int over = 0;
        int32_t id = -1;
        if (fire_d(N, states + j * N.m, k, y, &over)) id = (int32_t)table_find(T, pack_key(y, N.m));
        tgt[t] = id;
        if (id >= 0) atomicAdd(outdeg + j, 1);
    }
}

// one pruning round (reading R8): states with no outflow die; edges into the
// dead are removed from their sources' out-degrees.  *changed = 1 if a state died.
__global__ void prune_mark_kernel(int64_t n, const int32_t* outdeg, int8_t* dead, int* changed) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x)
        if (!dead[j] && outdeg[j] == 0) { dead[j] = 1; *changed = 1; }
}
__global__ void prune_edges_kernel(const GNet N, int64_t n, int32_t* tgt, int32_t* outdeg, const int8_t* dead) {
    for (int64_t t = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; t < n * N.R;
         t += (int64_t)gridDim.x * blockDim.x) {
        const int32_t d = tgt[t];
        if (d >= 0 && dead[d]) {
            tgt[t] = -1;
            if (!dead[t / N.R]) atomicSub(outdeg + t / N.R, 1);
        }
    }
}

__global__ void keep_counts_kernel(const GNet N, int64_t n, const int32_t* tgt, const int8_t* dead, int32_t* alive,
                                   int32_t* ecount) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        int32_t c = 0;
        if (!dead[j])
            for (int k = 0; k < N.R; ++k) c += tgt[j * N.R + k] >= 0;
        alive[j] = dead[j] ? 0 : 1;
        ecount[j] = c;
    }
}

__global__ void emit_kernel(const GNet N, int64_t n, const int32_t* states, const int32_t* tgt, const int8_t* dead,
                            const int64_t* nid, const int64_t* eoff, int32_t* out_states, int32_t* row, int32_t* col,
                            double* rate) {
    for (int64_t j = blockIdx.x * (int64_t)blockDim.x + threadIdx.x; j < n; j += (int64_t)gridDim.x * blockDim.x) {
        if (dead[j]) continue;
        const int32_t* xj = states + j * N.m;
        for (int i = 0; i < N.m; ++i) out_states[nid[j] * N.m + i] = xj[i];
        int64_t e = eoff[j];
        for (int k = 0; k < N.R; ++k) {
            const int32_t t = tgt[j * N.R + k];
            if (t < 0) continue;
            row[e] = (int32_t)nid[t];
            col[e] = (int32_t)nid[j];
            rate[e] = rate_d(N, xj, k);
            ++e;
        }
    }
}

// device allocations released on every exit path
struct DevBufs {
    std::vector<void*> p;
    ~DevBufs() {
        for (void* q : p) cudaFree(q);
    }
    template <typename T>
    cudaError_t get(T*& out, size_t count) {
        void* q = nullptr;
        const cudaError_t e = cudaMalloc(&q, std::max<size_t>(count, 1) * sizeof(T));
        if (e == cudaSuccess) p.push_back(q);
        out = static_cast<T*>(q);
        return e;
    }
    void release(void* q) {
        for (auto& x : p)
            if (x == q) { cudaFree(x); x = nullptr; }
    }
};

int blocks_for(int64_t n, int t = 256) { return (int)std::max<int64_t>(1, std::min<int64_t>((n + t - 1) / t, 1 << 20)); }

}  // namespace

cme_status enumerate_network_gpu(const GNet& N, int device, cme_coo_s& out) {
#define GTRY(expr)                                                                        \
    do {                                                                                  \
        cudaError_t _e = (expr);                                                          \
        if (_e != cudaSuccess) {                                                          \
            set_error(std::string("gpu enumerator: ") + #expr + ": " + cudaGetErrorString(_e)); \
            return _e == cudaErrorMemoryAllocation ? CME_ERR_OOM : CME_ERR_CUDA;          \
        }                                                                                 \
    } while (0)
    int count = 0;
    if (cudaGetDeviceCount(&count) != cudaSuccess || count == 0) {
        cudaGetLastError();
        set_error("gpu enumerator: no CUDA device visible");
        return CME_ERR_NO_DEVICE;
    }
    if (device >= 0) GTRY(cudaSetDevice(device));
    cudaStream_t s;
    GTRY(cudaStreamCreateWithFlags(&s, cudaStreamNonBlocking));
    std::unique_ptr<CUstream_st, void (*)(cudaStream_t)> sguard(s, [](cudaStream_t q) { cudaStreamDestroy(q); });
    DevBufs B;
    // --- 1. BFS --------------------------------------------------------------
    uint64_t cap_slots = uint64_t(1) << 22;
    int64_t cap_all = int64_t(1) << 21;     // discovery list / frontiers grow with the table
    Table T{};
    u128 *all = nullptr, *front = nullptr, *next = nullptr;
    unsigned long long* ctr = nullptr;      // [0] next count, [1] all count
    int* over = nullptr;
    GTRY(B.get(T.key, cap_slots));
    T.mask = cap_slots - 1;
    GTRY(B.get(all, cap_all));
    GTRY(B.get(front, cap_all));
    GTRY(B.get(next, cap_all));
    GTRY(B.get(ctr, 2));
    GTRY(B.get(over, 1));
    fill_empty_kernel<<<blocks_for(cap_slots), 256, 0, s>>>(T.key, cap_slots);
    GTRY(cudaMemsetAsync(over, 0, sizeof(int), s));
    unsigned long long h_ctr[2] = {0, 1};
    GTRY(cudaMemcpyAsync(ctr, h_ctr, sizeof(h_ctr), cudaMemcpyHostToDevice, s));
    seed_kernel<<<1, 1, 0, s>>>(N, T, all, front);
    int64_t nfront = 1, nall = 1;
    while (nfront > 0) {
        // worst case this level: every (state, reaction) inserts
        const int64_t grow = nfront * N.R;
        if ((uint64_t)(nall + grow) * 2 > cap_slots || nall + grow > cap_all) {
            uint64_t ns = cap_slots;
            while ((uint64_t)(nall + grow) * 2 > ns) ns *= 2;
            int64_t na = cap_all;
            while (nall + grow > na) na *= 2;
            if (ns != cap_slots) {   // rehash the table from the discovery list
                B.release(T.key);
                GTRY(B.get(T.key, ns));
                cap_slots = ns;
                T.mask = ns - 1;
                fill_empty_kernel<<<blocks_for(ns), 256, 0, s>>>(T.key, ns);
                reinsert_kernel<<<blocks_for(nall), 256, 0, s>>>(T, all, nall);
            }
            if (na != cap_all) {
                u128 *a2 = nullptr, *f2 = nullptr, *n2 = nullptr;
                GTRY(B.get(a2, na));
                GTRY(B.get(f2, na));
                GTRY(B.get(n2, na));
                GTRY(cudaMemcpyAsync(a2, all, nall * sizeof(u128), cudaMemcpyDeviceToDevice, s));
                GTRY(cudaMemcpyAsync(f2, front, nfront * sizeof(u128), cudaMemcpyDeviceToDevice, s));
                B.release(all); B.release(front); B.release(next);
                all = a2; front = f2; next = n2;
                cap_all = na;
            }
        }
        GTRY(cudaMemsetAsync(ctr, 0, sizeof(unsigned long long), s));
        expand_kernel<<<blocks_for(grow), 256, 0, s>>>(N, T, front, nfront, next, ctr, all, ctr + 1, over);
        GTRY(cudaGetLastError());
        GTRY(cudaMemcpyAsync(h_ctr, ctr, sizeof(h_ctr), cudaMemcpyDeviceToHost, s));
        GTRY(cudaStreamSynchronize(s));
        nfront = (int64_t)h_ctr[0];
        nall = (int64_t)h_ctr[1];
        std::swap(front, next);
    }
    int h_over = 0;
    GTRY(cudaMemcpy(&h_over, over, sizeof(int), cudaMemcpyDeviceToHost));
    if (h_over) {
        set_error("gpu enumerator: a species count exceeds 65534 (use cme_network_enumerate)");
        return CME_ERR_INVALID_ARG;
    }
    const int64_t n0 = nall;
    B.release(front);
    B.release(next);
    // --- 2. lexicographic numbering ------------------------------------------
    uint64_t *hi = nullptr, *lo = nullptr, *hi2 = nullptr, *lo2 = nullptr;
    GTRY(B.get(hi, n0));
    GTRY(B.get(lo, n0));
    GTRY(B.get(hi2, n0));
    GTRY(B.get(lo2, n0));
    split_kernel<<<blocks_for(n0), 256, 0, s>>>(all, n0, hi, lo);
    B.release(all);
    {
        size_t tmp_bytes = 0;
        GTRY(cub::DeviceRadixSort::SortPairs(nullptr, tmp_bytes, lo, lo2, hi, hi2, n0, 0, 64, s));
        char* tmp = nullptr;
        GTRY(B.get(tmp, tmp_bytes));
        // LSD over 128 bits: by the low word, then stably by the high word
        GTRY(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, lo, lo2, hi, hi2, n0, 0, 64, s));
        GTRY(cub::DeviceRadixSort::SortPairs(tmp, tmp_bytes, hi2, hi, lo2, lo, n0, 0, 64, s));
        B.release(tmp);
    }
    B.release(hi2);
    B.release(lo2);
    int32_t* states = nullptr;
    GTRY(B.get(T.val, cap_slots));
    GTRY(B.get(states, (size_t)n0 * N.m));
    number_kernel<<<blocks_for(n0), 256, 0, s>>>(N, T, hi, lo, n0, states);
    GTRY(cudaGetLastError());
    B.release(hi);
    B.release(lo);
    // --- 3. edges ------------------------------------------------------------
    int32_t *tgt = nullptr, *outdeg = nullptr;
    GTRY(B.get(tgt, (size_t)n0 * N.R));
    GTRY(B.get(outdeg, n0));
    GTRY(cudaMemsetAsync(outdeg, 0, n0 * sizeof(int32_t), s));
    edges_kernel<<<blocks_for(n0 * N.R), 256, 0, s>>>(N, T, states, n0, tgt, outdeg);
    GTRY(cudaGetLastError());
    B.release(T.key);
    B.release(T.val);
    // --- 4. zero-outflow pruning to the fixpoint -----------------------------
    int8_t* dead = nullptr;
    int* changed = nullptr;
    GTRY(B.get(dead, n0));
    GTRY(B.get(changed, 1));
    GTRY(cudaMemsetAsync(dead, 0, n0, s));
    for (;;) {
        GTRY(cudaMemsetAsync(changed, 0, sizeof(int), s));
        prune_mark_kernel<<<blocks_for(n0), 256, 0, s>>>(n0, outdeg, dead, changed);
        prune_edges_kernel<<<blocks_for(n0 * N.R), 256, 0, s>>>(N, n0, tgt, outdeg, dead);
        int h = 0;
        GTRY(cudaMemcpyAsync(&h, changed, sizeof(int), cudaMemcpyDeviceToHost, s));
        GTRY(cudaStreamSynchronize(s));
        if (!h) break;
    }
    // --- 5. compaction + COO -------------------------------------------------
    int32_t *alive = nullptr, *ecount = nullptr;
    int64_t *nid = nullptr, *eoff = nullptr;
    GTRY(B.get(alive, n0));
    GTRY(B.get(ecount, n0));
    GTRY(B.get(nid, n0));
    GTRY(B.get(eoff, n0));
    keep_counts_kernel<<<blocks_for(n0), 256, 0, s>>>(N, n0, tgt, dead, alive, ecount);
    {
        size_t tb = 0, tb2 = 0;
        GTRY(cub::DeviceScan::ExclusiveSum(nullptr, tb, alive, nid, n0, s));
        GTRY(cub::DeviceScan::ExclusiveSum(nullptr, tb2, ecount, eoff, n0, s));
        tb = std::max(tb, tb2);
        char* tmp = nullptr;
        GTRY(B.get(tmp, tb));
        GTRY(cub::DeviceScan::ExclusiveSum(tmp, tb, alive, nid, n0, s));
        GTRY(cub::DeviceScan::ExclusiveSum(tmp, tb, ecount, eoff, n0, s));
        B.release(tmp);
    }
    int64_t last_nid = 0, last_eoff = 0;
    int32_t last_alive = 0, last_ec = 0;
    GTRY(cudaMemcpyAsync(&last_nid, nid + n0 - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaMemcpyAsync(&last_eoff, eoff + n0 - 1, sizeof(int64_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaMemcpyAsync(&last_alive, alive + n0 - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaMemcpyAsync(&last_ec, ecount + n0 - 1, sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaStreamSynchronize(s));
    const int64_t n = last_nid + last_alive, nnz = last_eoff + last_ec;
    int32_t *o_states = nullptr, *o_row = nullptr, *o_col = nullptr;
    double* o_rate = nullptr;
    GTRY(B.get(o_states, (size_t)n * N.m));
    GTRY(B.get(o_row, nnz));
    GTRY(B.get(o_col, nnz));
    GTRY(B.get(o_rate, nnz));
    emit_kernel<<<blocks_for(n0), 256, 0, s>>>(N, n0, states, tgt, dead, nid, eoff, o_states, o_row, o_col, o_rate);
    GTRY(cudaGetLastError());
    out.m = N.m;
    out.n = n;
    out.nnz = nnz;
    out.states.resize((size_t)n * N.m);
    out.row.resize(nnz);
    out.col.resize(nnz);
    out.rate.resize(nnz);
    GTRY(cudaMemcpyAsync(out.states.data(), o_states, out.states.size() * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaMemcpyAsync(out.row.data(), o_row, nnz * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaMemcpyAsync(out.col.data(), o_col, nnz * sizeof(int32_t), cudaMemcpyDeviceToHost, s));
    GTRY(cudaMemcpyAsync(out.rate.data(), o_rate, nnz * sizeof(double), cudaMemcpyDeviceToHost, s));
    GTRY(cudaStreamSynchronize(s));
    return CME_OK;
#undef GTRY
}

}  // namespace cme

extern "C" cme_status cme_network_enumerate_gpu(int m, const int32_t* x0, int R, const int32_t* reac,
                                                const int32_t* change, const double* rates, const int32_t* w,
                                                int64_t cap, int device, cme_coo* out) {
    if (!out || m <= 0 || R <= 0 || !x0 || !reac || !change || !rates || !w) {
        cme::set_error("enumerate_gpu: bad arguments");
        return CME_ERR_INVALID_ARG;
    }
    *out = nullptr;
    if (m > cme::kMaxSpecies || R > cme::kMaxReactions) {
        cme::set_error("enumerate_gpu: at most 8 species and 64 reactions (use cme_network_enumerate)");
        return CME_ERR_INVALID_ARG;
    }
    cme::GNet N{};
    N.m = m;
    N.R = R;
    N.cap = cap;
    int64_t load = 0;
    for (int i = 0; i < m; ++i) {
        if (x0[i] < 0 || (uint32_t)x0[i] > cme::kMaxCount) {
            cme::set_error("enumerate_gpu: x0 out of range");
            return CME_ERR_INVALID_ARG;
        }
        load += (int64_t)w[i] * x0[i];
        N.x0[i] = x0[i];
        N.w[i] = w[i];
    }
    if (load > cap) { cme::set_error("enumerate_gpu: x0 violates the buffer"); return CME_ERR_INVALID_ARG; }
    for (int k = 0; k < R; ++k) {
        bool moves = false;
        for (int i = 0; i < m; ++i) {
            N.reac[k * m + i] = reac[(size_t)k * m + i];
            N.change[k * m + i] = change[(size_t)k * m + i];
            moves |= change[(size_t)k * m + i] != 0;
        }
        if (!moves || !(rates[k] >= 0.0)) {
            cme::set_error("enumerate_gpu: reaction " + std::to_string(k) + " has no net change or a bad rate");
            return CME_ERR_INVALID_ARG;
        }
        N.rates[k] = rates[k];
    }
    try {
        auto c = std::make_unique<cme_coo_s>();
        const cme_status st = cme::enumerate_network_gpu(N, device, *c);
        if (st != CME_OK) return st;
        *out = c.release();
        return CME_OK;
    } catch (const std::bad_alloc&) {
        cme::set_error("enumerate_gpu: out of host memory");
        return CME_ERR_OOM;
    }
}
