// State orderings and the directed-period test (host side of cme_reorder / cme_pack).
//
// DFS: "a DFS visit of the state space creates chains of reversible
// microstates" so the {-1,0,+1} band is dense.  RCM is the north star's second
// ordering (bandwidth ~4N on the toggle switch).  The exact tie
// rules are readings R11/R12 of DESIGN.md, frozen so that the oracle and this
// library agree bit for bit.
#include <algorithm>
#include <numeric>

#include "cme_internal.h"

namespace cme {

namespace {

// Column-wise pattern: out[j] = { i : A_ij != 0 } ascending (transitions j -> i).
void out_neighbours(const Csr& A, std::vector<int64_t>& ptr, std::vector<int32_t>& adj) {
    const int64_t n = A.n;
    ptr.assign(n + 1, 0);
    for (int32_t j : A.ci) ++ptr[j + 1];
    for (int64_t j = 0; j < n; ++j) ptr[j + 1] += ptr[j];
    adj.resize(A.nnz());
    std::vector<int64_t> fill(ptr.begin(), ptr.end() - 1);
    for (int64_t i = 0; i < n; ++i)
        for (int64_t p = A.rp[i]; p < A.rp[i + 1]; ++p) adj[fill[A.ci[p]]++] = (int32_t)i;
}

// Undirected pattern of A + A^T without the diagonal, neighbours ascending, no repeats.
void undirected(const Csr& A, std::vector<int64_t>& ptr, std::vector<int32_t>& adj) {
    std::vector<int64_t> tp;
    std::vector<int32_t> ta;
    out_neighbours(A, tp, ta);
    const int64_t n = A.n;
    ptr.assign(n + 1, 0);
    std::vector<int32_t> tmp;
    adj.clear();
    adj.reserve(2 * A.nnz());
    for (int64_t i = 0; i < n; ++i) {
        tmp.assign(A.ci.begin() + A.rp[i], A.ci.begin() + A.rp[i + 1]);
        tmp.insert(tmp.end(), ta.begin() + tp[i], ta.begin() + tp[i + 1]);
        std::sort(tmp.begin(), tmp.end());
        tmp.erase(std::unique(tmp.begin(), tmp.end()), tmp.end());
        for (int32_t v : tmp)
            if (v != i) adj.push_back(v);
        ptr[i + 1] = (int64_t)adj.size();
    }
}

struct Bfs {
    std::vector<int32_t> level;  // -1 = not reached
    std::vector<int32_t> queue;
    explicit Bfs(int64_t n) : level(n, -1) { queue.reserve(n); }
    // BFS over the undirected graph; returns eccentricity of s.
    int32_t run(int32_t s, const std::vector<int64_t>& ptr, const std::vector<int32_t>& adj) {
        for (int32_t v : queue) level[v] = -1;
        queue.clear();
        queue.push_back(s);
        level[s] = 0;
        int32_t ecc = 0;
        for (size_t h = 0; h < queue.size(); ++h) {
            const int32_t u = queue[h];
            for (int64_t p = ptr[u]; p < ptr[u + 1]; ++p) {
                const int32_t v = adj[p];
                if (level[v] < 0) {
                    level[v] = level[u] + 1;
                    ecc = std::max(ecc, level[v]);
                    queue.push_back(v);
                }
            }
        }
        return ecc;
    }
};

}  // namespace

void order_dfs(const Csr& A, int64_t root, std::vector<int32_t>& new_to_old) {
    const int64_t n = A.n;
    std::vector<int64_t> ptr;
    std::vector<int32_t> adj;
    out_neighbours(A, ptr, adj);
    new_to_old.clear();
    new_to_old.reserve(n);
    std::vector<char> seen(n, 0);
    std::vector<std::pair<int32_t, int64_t>> stack;  // (state, next out-edge)
    int64_t scan = 0;
    auto visit_from = [&](int32_t s) {
        seen[s] = 1;
        new_to_old.push_back(s);
        stack.emplace_back(s, ptr[s]);
        while (!stack.empty()) {
            auto& top = stack.back();
            if (top.second == ptr[top.first + 1]) { stack.pop_back(); continue; }
            const int32_t v = adj[top.second++];
            if (seen[v]) continue;
            seen[v] = 1;
            new_to_old.push_back(v);
            stack.emplace_back(v, ptr[v]);
        }
    };
    visit_from((int32_t)root);
    while ((int64_t)new_to_old.size() < n) {
        while (seen[scan]) ++scan;
        visit_from((int32_t)scan);
    }
}

void order_rcm(const Csr& A, std::vector<int32_t>& new_to_old) {
    const int64_t n = A.n;
    std::vector<int64_t> ptr;
    std::vector<int32_t> adj;
    undirected(A, ptr, adj);
    auto deg = [&](int32_t v) { return ptr[v + 1] - ptr[v]; };
    auto lighter = [&](int32_t a, int32_t b) {  // (degree, index) order
        return deg(a) != deg(b) ? deg(a) < deg(b) : a < b;
    };
    Bfs bfs(n);
    std::vector<char> placed(n, 0);
    std::vector<int32_t> cm;
    cm.reserve(n);
    std::vector<int32_t> nb;
    for (int32_t v0 = 0; v0 < n; ++v0) {
        if (placed[v0]) continue;
        // start: minimum-degree vertex of the component (ties: smallest index) ...
        bfs.run(v0, ptr, adj);
        int32_t s = *std::min_element(bfs.queue.begin(), bfs.queue.end(), lighter);
        // ... then George-Liu: hop to the lightest vertex of the last BFS level
        // while the eccentricity keeps growing.
        int32_t ecc = bfs.run(s, ptr, adj);
        for (;;) {
            int32_t cand = -1;
            for (int32_t u : bfs.queue)
                if (bfs.level[u] == ecc && (cand < 0 || lighter(u, cand))) cand = u;
            const int32_t e2 = bfs.run(cand, ptr, adj);
            if (e2 <= ecc) break;
            ecc = e2;
            s = cand;
        }
        // Cuthill-McKee sweep from s
        const size_t head0 = cm.size();
        cm.push_back(s);
        placed[s] = 1;
        for (size_t h = head0; h < cm.size(); ++h) {
            const int32_t u = cm[h];
            nb.clear();
            for (int64_t p = ptr[u]; p < ptr[u + 1]; ++p)
                if (!placed[adj[p]]) { placed[adj[p]] = 1; nb.push_back(adj[p]); }
            std::sort(nb.begin(), nb.end(), lighter);
            cm.insert(cm.end(), nb.begin(), nb.end());
        }
    }
    new_to_old.assign(cm.rbegin(), cm.rend());
}

int64_t directed_period(const Csr& A, int64_t root) {
    const int64_t n = A.n;
    std::vector<int64_t> ptr;
    std::vector<int32_t> adj;
    out_neighbours(A, ptr, adj);
    std::vector<int64_t> lvl(n, -1);
    std::vector<int32_t> q;
    q.reserve(n);
    int64_t scan = 0;
    int64_t s = root;
    for (;;) {
        if (s < 0) {
            while (scan < n && lvl[scan] >= 0) ++scan;
            if (scan == n) break;
            s = scan;
        }
        q.clear();
        q.push_back((int32_t)s);
        lvl[s] = 0;
        for (size_t h = 0; h < q.size(); ++h) {
            const int32_t u = q[h];
            for (int64_t p = ptr[u]; p < ptr[u + 1]; ++p)
                if (lvl[adj[p]] < 0) { lvl[adj[p]] = lvl[u] + 1; q.push_back(adj[p]); }
        }
        s = -1;
    }
    int64_t g = 0;
    for (int64_t u = 0; u < n; ++u)
        for (int64_t p = ptr[u]; p < ptr[u + 1]; ++p) g = std::gcd(g, std::abs(lvl[u] + 1 - lvl[adj[p]]));
    return g;
}

void permute(const Csr& A, const std::vector<int32_t>& p, Csr& B) {
    const int64_t n = A.n;
    const int32_t nb = A.B;
    std::vector<int32_t> inv(n);
    for (int64_t r = 0; r < n; ++r) inv[p[r]] = (int32_t)r;
    B.n = n;
    B.B = nb;
    B.rp.assign(n + 1, 0);
    for (int64_t r = 0; r < n; ++r) B.rp[r + 1] = B.rp[r] + (A.rp[p[r] + 1] - A.rp[p[r]]);
    B.ci.resize(A.nnz());
    B.v.resize((size_t)A.nnz() * nb);
    B.d.resize((size_t)n * nb);
#pragma omp parallel
    {
        std::vector<std::pair<int32_t, int64_t>> row;  // (new column, old position)
#pragma omp for schedule(dynamic, 4096)
        for (int64_t r = 0; r < n; ++r) {
            const int64_t o = p[r];
            for (int32_t b = 0; b < nb; ++b) B.d[(size_t)r * nb + b] = A.d[(size_t)o * nb + b];
            row.clear();
            for (int64_t q = A.rp[o]; q < A.rp[o + 1]; ++q) row.emplace_back(inv[A.ci[q]], q);
            std::sort(row.begin(), row.end(),
                      [](const auto& a, const auto& b) { return a.first < b.first; });
            int64_t w = B.rp[r];
            for (auto& e : row) {
                B.ci[w] = e.first;
                for (int32_t b = 0; b < nb; ++b) B.v[(size_t)w * nb + b] = A.v[(size_t)e.second * nb + b];
                ++w;
            }
        }
    }
}

}  // namespace cme
