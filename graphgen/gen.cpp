// graphgen/gen.cpp -- seeded synthetic graph / feature generators.
//
// Shared by the tests, the bench and smoke() on BOTH sides of the parity check: the
// CUDA path and the CPU oracle receive the same arrays from here.  This module holds
// none of MergePath-SpMM's arithmetic (no partition, no product, no fix-up): it only
// builds inputs with the shapes, sizes and skew of the paper's workloads (Table II,
// P:202-228) as restated in DESIGN.md "Input recipe".
//
// Randomness is a counter-based generator (splitmix64 of (seed, stream, index)), so
// every value depends only on its counter, never on thread count or schedule.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <vector>
#include <omp.h>

namespace {

inline uint64_t mix64(uint64_t z) {
    z += 0x9E3779B97F4A7C15ull;
    z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
    z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
    return z ^ (z >> 31);
}
inline uint64_t rng(uint64_t seed, uint64_t stream, uint64_t idx) {
    return mix64(mix64(seed * 0xD1B54A32D192ED03ull + stream) ^ (idx * 0x9E3779B97F4A7C15ull));
}
inline double u01(uint64_t seed, uint64_t stream, uint64_t idx) {
    return (double)(rng(seed, stream, idx) >> 11) * (1.0 / 9007199254740992.0);
}

enum : uint64_t { S_EDGE = 1, S_PERM = 2, S_RMAT = 3, S_EVIL = 4, S_VAL = 5, S_DENSE = 6 };

struct Graph {
    int64_t m = 0, n = 0;
    std::vector<int32_t> rp;
    std::vector<int32_t> ci;
};

// Continuous power law p(x) ~ (x + i0)^-alpha on [0, n): inverse CDF.
struct PowerLaw {
    double alpha, i0, a, S;
    int64_t n;
    PowerLaw(int64_t n_, double alpha_, double i0_) : alpha(alpha_), i0(i0_), n(n_) {
        double e = 1.0 - alpha;
        a = std::pow(i0, e);
        S = std::pow((double)n + i0, e) - a;
    }
    int32_t sample(double u) const {
        double x = std::pow(a + u * S, 1.0 / (1.0 - alpha)) - i0;
        int64_t k = (int64_t)x;
        if (k < 0) k = 0;
        if (k >= n) k = n - 1;
        return (int32_t)k;
    }
    double p0() const { return (std::pow(1.0 + i0, 1.0 - alpha) - a) / S; }
};

// Solve i0 so that the expected (pre-dedup) degree of the heaviest node is dmax.
PowerLaw fit_power_law(int64_t n, int64_t E, double alpha, double dmax) {
    double lo = 1e-3, hi = 1e12;
    for (int it = 0; it < 200; ++it) {
        double mid = std::sqrt(lo * hi);
        PowerLaw pl(n, alpha, mid);
        double d0 = 2.0 * (double)E * pl.p0();
        if (d0 > dmax) lo = mid; else hi = mid;
    }
    return PowerLaw(n, alpha, std::sqrt(lo * hi));
}

// Random permutation of [0, n): order nodes by a 64-bit hash of their id.
std::vector<int32_t> random_perm(int64_t n, uint64_t seed) {
    std::vector<uint64_t> key(n);
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < n; ++i) key[i] = (rng(seed, S_PERM, i) & ~0xFFFFFFFFFull) | (uint64_t)i;
    std::sort(key.begin(), key.end());
    std::vector<int32_t> perm(n);
    // perm[old] = new
#pragma omp parallel for schedule(static)
    for (int64_t r = 0; r < n; ++r) perm[key[r] & 0xFFFFFFFFFull] = (int32_t)r;
    return perm;
}

// Build a CSR from per-row lists given as (row, col) pairs with sorted, de-duplicated
// columns.  rows/cols: entries; relabel through perm (may be empty = identity).
void build_csr(Graph &g, int64_t m, int64_t n, const std::vector<int32_t> &rows,
               const std::vector<int32_t> &cols, const std::vector<int32_t> &perm, bool dedup) {
    g.m = m;
    g.n = n;
    int64_t ne = (int64_t)rows.size();
    std::vector<int64_t> cnt(m + 1, 0);
    for (int64_t e = 0; e < ne; ++e) cnt[(perm.empty() ? rows[e] : perm[rows[e]]) + 1]++;
    for (int64_t i = 0; i < m; ++i) cnt[i + 1] += cnt[i];
    std::vector<int32_t> tmp(ne);
    std::vector<int64_t> cur(cnt.begin(), cnt.end() - 1);
    for (int64_t e = 0; e < ne; ++e) {
        int32_t r = perm.empty() ? rows[e] : perm[rows[e]];
        tmp[cur[r]++] = perm.empty() ? cols[e] : perm[cols[e]];
    }
    std::vector<int64_t> keep(m, 0);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < m; ++i) {
        auto b = tmp.begin() + cnt[i], e = tmp.begin() + cnt[i + 1];
        std::sort(b, e);
        keep[i] = dedup ? (int64_t)(std::unique(b, e) - b) : (int64_t)(e - b);
    }
    g.rp.assign(m + 1, 0);
    for (int64_t i = 0; i < m; ++i) g.rp[i + 1] = (int32_t)(g.rp[i] + keep[i]);
    g.ci.resize(g.rp[m]);
#pragma omp parallel for schedule(dynamic, 1024)
    for (int64_t i = 0; i < m; ++i)
        std::copy(tmp.begin() + cnt[i], tmp.begin() + cnt[i] + keep[i], g.ci.begin() + g.rp[i]);
}

// Chung-Lu undirected graph with exactly E distinct undirected edges (if reachable),
// symmetrised (nnz = 2E), no self loops, node ids randomly permuted, columns sorted.
Graph chung_lu(int64_t n, int64_t E, double alpha, double dmax, uint64_t seed) {
    PowerLaw pl = fit_power_law(n, E, alpha, dmax);
    double over = 1.10;
    for (int attempt = 0; attempt < 8; ++attempt, over *= 1.35) {
        int64_t Es = (int64_t)((double)E * over) + 64;
        std::vector<int32_t> u(Es), v(Es);
#pragma omp parallel for schedule(static)
        for (int64_t s = 0; s < Es; ++s) {
            u[s] = pl.sample(u01(seed, S_EDGE, 2 * s));
            v[s] = pl.sample(u01(seed, S_EDGE, 2 * s + 1));
        }
        // per-row keys (col << 32 | sample) for both directions
        std::vector<int64_t> off(n + 1, 0);
        for (int64_t s = 0; s < Es; ++s)
            if (u[s] != v[s]) { off[u[s] + 1]++; off[v[s] + 1]++; }
        for (int64_t i = 0; i < n; ++i) off[i + 1] += off[i];
        std::vector<uint64_t> key(off[n]);
        std::vector<int64_t> cur(off.begin(), off.end() - 1);
        for (int64_t s = 0; s < Es; ++s)
            if (u[s] != v[s]) {
                key[cur[u[s]]++] = ((uint64_t)(uint32_t)v[s] << 32) | (uint64_t)s;
                key[cur[v[s]]++] = ((uint64_t)(uint32_t)u[s] << 32) | (uint64_t)s;
            }
        // sort rows, keep the first sample of every distinct column
        std::vector<int64_t> uniq(n, 0);
#pragma omp parallel for schedule(dynamic, 256)
        for (int64_t i = 0; i < n; ++i) {
            auto b = key.begin() + off[i], e = key.begin() + off[i + 1];
            std::sort(b, e);
            int64_t w = 0;
            for (auto it = b; it != e; ++it)
                if (w == 0 || (*(b + w - 1) >> 32) != (*it >> 32)) *(b + (w++)) = *it;
            uniq[i] = w;
        }
        // first-sample ids of the distinct undirected edges (row < col side)
        std::vector<uint32_t> first;
        first.reserve(E + E / 4);
        for (int64_t i = 0; i < n; ++i)
            for (int64_t t = 0; t < uniq[i]; ++t) {
                uint64_t k = key[off[i] + t];
                if ((int64_t)(k >> 32) > i) first.push_back((uint32_t)k);
            }
        if ((int64_t)first.size() < E && attempt < 7) continue;
        uint64_t tau = UINT64_MAX;
        if ((int64_t)first.size() > E) {
            std::nth_element(first.begin(), first.begin() + (E - 1), first.end());
            tau = first[E - 1];
        }
        std::vector<int32_t> rows, cols;
        rows.reserve(2 * E);
        cols.reserve(2 * E);
        for (int64_t i = 0; i < n; ++i)
            for (int64_t t = 0; t < uniq[i]; ++t) {
                uint64_t k = key[off[i] + t];
                if ((uint64_t)(uint32_t)k <= tau) {
                    rows.push_back((int32_t)i);
                    cols.push_back((int32_t)(k >> 32));
                }
            }
        std::vector<int32_t> perm = random_perm(n, seed);
        Graph g;
        build_csr(g, n, n, rows, cols, perm, true);
        return g;
    }
    return Graph();
}

// "Structured" graph (Table II type II: batches of small molecule/protein graphs):
// block-diagonal, blocks of `block` consecutive nodes, E distinct undirected edges drawn
// uniformly inside the blocks (first E distinct samples), symmetrised, no self loops.
// Node ids are NOT permuted: these datasets keep each small graph contiguous.
Graph block_diag(int64_t n, int64_t E, int64_t block, uint64_t seed) {
    const int64_t nblk = (n + block - 1) / block;
    double over = 1.10;
    for (int attempt = 0; attempt < 8; ++attempt, over *= 1.35) {
        int64_t Es = (int64_t)((double)E * over) + 64;
        std::vector<int32_t> u(Es), v(Es);
#pragma omp parallel for schedule(static)
        for (int64_t s = 0; s < Es; ++s) {
            const int64_t b = (int64_t)(rng(seed, S_EDGE, 3 * s) % (uint64_t)nblk);
            const int64_t lo = b * block, sz = std::min(block, n - lo);
            u[s] = (int32_t)(lo + (int64_t)(rng(seed, S_EDGE, 3 * s + 1) % (uint64_t)sz));
            v[s] = (int32_t)(lo + (int64_t)(rng(seed, S_EDGE, 3 * s + 2) % (uint64_t)sz));
        }
        // canonical (min, max) keys with the first sample id, sorted and de-duplicated
        std::vector<std::pair<uint64_t, uint32_t>> key;
        key.reserve(Es);
        for (int64_t s = 0; s < Es; ++s)
            if (u[s] != v[s]) {
                const uint32_t a = (uint32_t)std::min(u[s], v[s]), b = (uint32_t)std::max(u[s], v[s]);
                key.push_back({((uint64_t)a << 32) | b, (uint32_t)s});
            }
        std::sort(key.begin(), key.end());
        std::vector<std::pair<uint32_t, uint64_t>> first;   // (sample, edge)
        for (size_t i = 0; i < key.size(); ++i)
            if (i == 0 || key[i].first != key[i - 1].first) first.push_back({key[i].second, key[i].first});
        if ((int64_t)first.size() < E && attempt < 7) continue;
        if ((int64_t)first.size() > E) {
            std::nth_element(first.begin(), first.begin() + E, first.end());
            first.resize(E);
        }
        std::vector<int32_t> rows, cols;
        rows.reserve(2 * first.size());
        cols.reserve(2 * first.size());
        for (auto &f : first) {
            const int32_t a = (int32_t)(f.second >> 32), b = (int32_t)(f.second & 0xffffffffu);
            rows.push_back(a); cols.push_back(b);
            rows.push_back(b); cols.push_back(a);
        }
        Graph g;
        build_csr(g, n, n, rows, cols, std::vector<int32_t>(), true);
        return g;
    }
    return Graph();
}

// R-MAT (Chakrabarti et al.) directed graph, de-duplicated, no self loops, ids
// permuted; then `n_evil` rows (row 0, row n-1 and seeded-random rows) replaced by
// `evil_len` distinct columns each ("evil rows").
Graph rmat(int scale, int64_t edge_factor, double a, double b, double c, int n_evil,
           int64_t evil_len, uint64_t seed) {
    int64_t n = (int64_t)1 << scale;
    int64_t Es = edge_factor * n;
    std::vector<int32_t> u(Es), v(Es);
#pragma omp parallel for schedule(static)
    for (int64_t s = 0; s < Es; ++s) {
        int64_t x = 0, y = 0;
        for (int l = 0; l < scale; ++l) {
            double r = u01(seed, S_RMAT, s * scale + l);
            int bx = 0, by = 0;
            if (r < a) {
            } else if (r < a + b) {
                by = 1;
            } else if (r < a + b + c) {
                bx = 1;
            } else {
                bx = 1;
                by = 1;
            }
            x = (x << 1) | bx;
            y = (y << 1) | by;
        }
        u[s] = (int32_t)x;
        v[s] = (int32_t)y;
    }
    std::vector<int32_t> perm = random_perm(n, seed);
    // choose evil rows (post-permutation ids)
    std::vector<int32_t> evil;
    if (n_evil > 0) evil.push_back(0);
    if (n_evil > 1) evil.push_back((int32_t)(n - 1));
    for (uint64_t t = 0; (int)evil.size() < n_evil && t < 1000000; ++t) {
        int32_t r = (int32_t)(rng(seed, S_EVIL, t) % (uint64_t)n);
        if (std::find(evil.begin(), evil.end(), r) == evil.end()) evil.push_back(r);
    }
    std::vector<char> is_evil(n, 0);
    for (int32_t r : evil) is_evil[r] = 1;
    std::vector<int32_t> rows, cols;
    rows.reserve(Es + evil.size() * evil_len);
    cols.reserve(Es + evil.size() * evil_len);
    for (int64_t s = 0; s < Es; ++s) {
        if (u[s] == v[s]) continue;
        int32_t pr = perm[u[s]], pc = perm[v[s]];
        if (is_evil[pr]) continue;
        rows.push_back(pr);
        cols.push_back(pc);
    }
    for (size_t t = 0; t < evil.size(); ++t) {
        // distinct columns: an affine bijection of Z_{2^scale}, skipping the diagonal
        uint64_t mul = (rng(seed, S_EVIL, 1000000 + 2 * t) | 1ull) & (uint64_t)(n - 1);
        uint64_t add = rng(seed, S_EVIL, 1000001 + 2 * t) & (uint64_t)(n - 1);
        int64_t taken = 0;
        for (int64_t i = 0; taken < evil_len && i < n; ++i) {
            int32_t col = (int32_t)((mul * (uint64_t)i + add) & (uint64_t)(n - 1));
            if (col == evil[t]) continue;
            rows.push_back(evil[t]);
            cols.push_back(col);
            ++taken;
        }
    }
    Graph g;
    build_csr(g, n, n, rows, cols, std::vector<int32_t>(), true);
    return g;
}

}  // namespace

extern "C" {

int gen_abi_version(void) { return 1; }

void *gen_chung_lu(int64_t n, int64_t E, double alpha, double dmax, uint64_t seed) {
    Graph *g = new Graph(chung_lu(n, E, alpha, dmax, seed));
    return g;
}

void *gen_rmat(int32_t scale, int64_t edge_factor, double a, double b, double c, int32_t n_evil,
               int64_t evil_len, uint64_t seed) {
    return new Graph(rmat(scale, edge_factor, a, b, c, n_evil, evil_len, seed));
}

void *gen_block_diag(int64_t n, int64_t E, int64_t block, uint64_t seed) {
    return new Graph(block_diag(n, E, block, seed));
}

// Arbitrary CSR from explicit per-row lengths with uniformly random columns in
// [0, n) (duplicates and unsorted columns allowed when `canonical` is 0).
void *gen_random_csr(int64_t m, int64_t n, const int32_t *row_len, int32_t canonical,
                     uint64_t seed) {
    Graph *g = new Graph();
    g->m = m;
    g->n = n;
    g->rp.assign(m + 1, 0);
    for (int64_t i = 0; i < m; ++i) g->rp[i + 1] = g->rp[i] + row_len[i];
    g->ci.resize(g->rp[m]);
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < m; ++i) {
        for (int64_t j = g->rp[i]; j < g->rp[i + 1]; ++j)
            g->ci[j] = n > 0 ? (int32_t)(rng(seed, S_EDGE, j) % (uint64_t)n) : 0;
        if (canonical) std::sort(g->ci.begin() + g->rp[i], g->ci.begin() + g->rp[i + 1]);
    }
    return g;
}

int64_t gen_rows(void *h) { return ((Graph *)h)->m; }
int64_t gen_cols(void *h) { return ((Graph *)h)->n; }
int64_t gen_nnz(void *h) { return ((Graph *)h)->rp.empty() ? 0 : ((Graph *)h)->rp.back(); }
void gen_copy(void *h, int32_t *rp, int32_t *ci) {
    Graph *g = (Graph *)h;
    std::memcpy(rp, g->rp.data(), sizeof(int32_t) * g->rp.size());
    std::memcpy(ci, g->ci.data(), sizeof(int32_t) * g->ci.size());
}
void gen_free(void *h) { delete (Graph *)h; }

// GCN-normalised edge values 1/sqrt(d_i * d_j) with d = row length (>= 1).
void gen_values_gcn(int64_t m, const int32_t *rp, const int32_t *ci, float *val) {
#pragma omp parallel for schedule(dynamic, 256)
    for (int64_t i = 0; i < m; ++i) {
        double di = std::max<int64_t>(1, rp[i + 1] - rp[i]);
        for (int64_t j = rp[i]; j < rp[i + 1]; ++j) {
            int64_t c = ci[j];
            double dj = (c < m) ? std::max<int64_t>(1, rp[c + 1] - rp[c]) : 1.0;
            val[j] = (float)(1.0 / std::sqrt(di * dj));
        }
    }
}

// Integer edge values in {1, 2, 3} (exact-arithmetic parity runs).
void gen_values_int(int64_t nnz, uint64_t seed, float *val) {
#pragma omp parallel for schedule(static)
    for (int64_t j = 0; j < nnz; ++j) val[j] = (float)(1 + rng(seed, S_VAL, j) % 3);
}

// Dense rows x K (leading dimension ld) with U[-1, 1) entries; padding left as is.
void gen_dense_uniform(int64_t rows, int32_t K, int64_t ld, uint64_t seed, float *B) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < rows; ++i)
        for (int32_t k = 0; k < K; ++k)
            B[i * ld + k] = (float)(2.0 * u01(seed, S_DENSE, (uint64_t)i * (uint64_t)K + k) - 1.0);
}

// Dense rows x K with integer entries in {-4, ..., 4}.
void gen_dense_int(int64_t rows, int32_t K, int64_t ld, uint64_t seed, float *B) {
#pragma omp parallel for schedule(static)
    for (int64_t i = 0; i < rows; ++i)
        for (int32_t k = 0; k < K; ++k)
            B[i * ld + k] = (float)((int)(rng(seed, S_DENSE, (uint64_t)i * (uint64_t)K + k) % 9) - 4);
}

}  // extern "C"
