// graphgen.cpp -- seeded synthetic input generators shared by tests, bench and oracle runs.
//
// This module holds NONE of the SCC method's arithmetic: it only emits CSR graphs.  Both
// the CUDA path and the oracle consume the very same arrays.  Every random draw is a
// counter-based splitmix64 hash of (seed, item, draw), so the output is bit-reproducible
// and independent of thread count and schedule.  Compiled with -ffp-contract=off and no
// fast-math so the floating-point sign tests of the mesh generator are reproducible.
//
//  * gen_mesh  -- directed sweep graph of a Kuhn-6 tetrahedralisation of an N^3 cube grid
//                 (after P:265-269, Sec. 4.1: one vertex per element, one edge per interior
//                 face and quadrature point orientation; re-entrant curved faces give both
//                 directions).  Curvature is modelled by perturbing the face normal at Q
//                 points: n_i = n_face + kappa * xi_i, xi_i ~ N(0, I3).
//  * gen_rmat  -- Graph500-style R-MAT (a,b,c,d), random vertex relabelling, self-loops and
//                 duplicates dropped (shaped like the power-law inputs of Table 3).
//  * gen_gnm   -- uniform G(n, m): m distinct ordered pairs u != v.
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <unordered_set>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {

inline uint64_t splitmix64(uint64_t x) {
    x += 0x9E3779B97F4A7C15ull;
    x = (x ^ (x >> 30)) * 0xBF58476D1CE4E5B9ull;
    x = (x ^ (x >> 27)) * 0x94D049BB133111EBull;
    return x ^ (x >> 31);
}
inline uint64_t hash3(uint64_t seed, uint64_t a, uint64_t b) {
    return splitmix64(splitmix64(splitmix64(seed) ^ a) ^ b);
}
// uniform in (0,1), 53 bits
inline double unit(uint64_t r) { return ((double)(r >> 11) + 0.5) * (1.0 / 9007199254740992.0); }

// ---------------------------------------------------------------- mesh
const int PERM[6][3] = {{0, 1, 2}, {0, 2, 1}, {1, 0, 2}, {1, 2, 0}, {2, 0, 1}, {2, 1, 0}};
inline int perm_index(int a, int b, int c) {
    for (int p = 0; p < 6; p++)
        if (PERM[p][0] == a && PERM[p][1] == b && PERM[p][2] == c) return p;
    return -1;
}

struct MeshSpec {
    int64_t N;
    int order;  // 0 = lexicographic (x-major), 1 = 8^3-blocked (block-major, lex inside)
    int64_t nb;
};

inline int64_t cube_index(const MeshSpec& s, int64_t x, int64_t y, int64_t z) {
    const int64_t N = s.N;
    if (s.order == 0) return (x * N + y) * N + z;
    const int64_t B = 8;
    int64_t bx = x / B, by = y / B, bz = z / B;
    int64_t bsx = std::min(B, N - bx * B), bsy = std::min(B, N - by * B), bsz = std::min(B, N - bz * B);
    int64_t off = (bx * B) * N * N + bsx * (by * B) * N + bsx * bsy * (bz * B);
    int64_t lx = x - bx * B, ly = y - by * B, lz = z - bz * B;
    return off + (lx * bsy + ly) * bsz + lz;
}

}  // namespace

extern "C" {

// Directed mesh sweep graph.  n = 6*N^3 vertices.
//   omega[3]   the ordinate (need not be normalised)
//   kappa      curvature noise amplitude; kappa_hot applies in 8^3-cube blocks with
//              (bx+by+bz) % hot_mod == 0 (hot_mod <= 0 disables hot spots)
//   Q          quadrature points per face
//   row_ptr    out, n+1 entries;  col_idx  out, capacity 4*n
// returns nnz.  Each row is sorted ascending.
int64_t gen_mesh(int64_t N, int order, const double* omega, double kappa, double kappa_hot,
                 int hot_mod, int Q, uint64_t seed, int32_t* row_ptr, int32_t* col_idx) {
    MeshSpec s{N, order, (N + 7) / 8};
    const int64_t n = 6 * N * N * N;
    std::vector<uint8_t> deg(n);
    std::vector<int32_t> slots((size_t)n * 4);
    const double ox = omega[0], oy = omega[1], oz = omega[2];

#pragma omp parallel for schedule(static)
    for (int64_t xyz = 0; xyz < N * N * N; xyz++) {
        const int64_t x = xyz / (N * N), y = (xyz / N) % N, z = xyz % N;
        const int64_t c[3] = {x, y, z};
        const int64_t cid = cube_index(s, x, y, z);
        const int64_t clex = (x * N + y) * N + z;   // numbering-independent cube key
        for (int p = 0; p < 6; p++) {
            const int a = PERM[p][0], b = PERM[p][1], cc = PERM[p][2];
            const int64_t e = 6 * cid + p;
            const int64_t elex = 6 * clex + p;
            // tet vertices (integer coordinates)
            int64_t V[4][3];
            for (int d = 0; d < 3; d++) {
                V[0][d] = c[d];
                V[1][d] = c[d] + (d == a);
                V[2][d] = c[d] + (d == a) + (d == b);
                V[3][d] = c[d] + 1;
            }
            int outs[4];
            int nout = 0;
            for (int k = 0; k < 4; k++) {  // face opposite vertex k
                int64_t nc[3] = {c[0], c[1], c[2]};
                int np_;
                if (k == 3) { nc[cc] -= 1; np_ = perm_index(cc, a, b); }
                else if (k == 0) { nc[a] += 1; np_ = perm_index(b, cc, a); }
                else if (k == 1) { np_ = perm_index(b, a, cc); }
                else { np_ = perm_index(a, cc, b); }
                if (nc[0] < 0 || nc[1] < 0 || nc[2] < 0 || nc[0] >= N || nc[1] >= N || nc[2] >= N)
                    continue;  // boundary face
                const int64_t e2 = 6 * cube_index(s, nc[0], nc[1], nc[2]) + np_;
                const int64_t e2lex = 6 * ((nc[0] * N + nc[1]) * N + nc[2]) + np_;
                // exact integer outward normal of e on this face
                int64_t f[3][3];
                int t = 0;
                for (int j = 0; j < 4; j++)
                    if (j != k) { for (int d = 0; d < 3; d++) f[t][d] = V[j][d]; t++; }
                int64_t u1[3], u2[3], w[3];
                for (int d = 0; d < 3; d++) { u1[d] = f[1][d] - f[0][d]; u2[d] = f[2][d] - f[0][d]; }
                int64_t cr[3] = {u1[1] * u2[2] - u1[2] * u2[1], u1[2] * u2[0] - u1[0] * u2[2],
                                 u1[0] * u2[1] - u1[1] * u2[0]};
                for (int d = 0; d < 3; d++) w[d] = V[k][d] - f[0][d];
                if (cr[0] * w[0] + cr[1] * w[1] + cr[2] * w[2] > 0)
                    for (int d = 0; d < 3; d++) cr[d] = -cr[d];
                // canonical orientation: e1 = lower LEXICOGRAPHIC element key, normal points
                // from e1 into e2.  The face's RNG stream, its orientation and its
                // hot-spot test depend only on lexicographic keys, so every element order
                // yields the same graph up to a relabelling of the vertices.
                const bool lo_is_e = elex < e2lex;
                const int64_t lo = lo_is_e ? elex : e2lex, hi = lo_is_e ? e2lex : elex;
                if (!lo_is_e) for (int d = 0; d < 3; d++) cr[d] = -cr[d];
                const double nn = std::sqrt((double)(cr[0] * cr[0] + cr[1] * cr[1] + cr[2] * cr[2]));
                const double n0 = (double)cr[0] / nn, n1 = (double)cr[1] / nn, n2 = (double)cr[2] / nn;
                // curvature of the face: hot spot decided by the cube of e1 = lo
                const int64_t* lc = lo_is_e ? c : nc;
                double kap = kappa;
                if (hot_mod > 0 && ((lc[0] / 8 + lc[1] / 8 + lc[2] / 8) % hot_mod) == 0) kap = kappa_hot;
                bool fwd = false, bwd = false;
                const uint64_t h = hash3(seed, (uint64_t)lo, (uint64_t)hi);
                for (int i = 0; i < Q; i++) {
                    double g[4];
                    for (int j = 0; j < 2; j++) {
                        const double u = unit(splitmix64(h + (uint64_t)(4 * i + 2 * j)));
                        const double v = unit(splitmix64(h + (uint64_t)(4 * i + 2 * j + 1)));
                        const double r = std::sqrt(-2.0 * std::log(u));
                        g[2 * j] = r * std::cos(6.283185307179586 * v);
                        g[2 * j + 1] = r * std::sin(6.283185307179586 * v);
                    }
                    const double d = ox * (n0 + kap * g[0]) + oy * (n1 + kap * g[1]) + oz * (n2 + kap * g[2]);
                    if (d > 0) fwd = true; else bwd = true;  // Omega.n > 0 -> e1->e2, else e2->e1
                }
                if (lo_is_e ? fwd : bwd) outs[nout++] = (int32_t)e2;
            }
            std::sort(outs, outs + nout);
            deg[e] = (uint8_t)nout;
            for (int j = 0; j < nout; j++) slots[(size_t)e * 4 + j] = outs[j];
        }
    }
    int64_t acc = 0;
    row_ptr[0] = 0;
    for (int64_t v = 0; v < n; v++) { acc += deg[v]; row_ptr[v + 1] = (int32_t)acc; }
#pragma omp parallel for schedule(static)
    for (int64_t v = 0; v < n; v++)
        for (int j = 0; j < deg[v]; j++) col_idx[row_ptr[v] + j] = slots[(size_t)v * 4 + j];
    return acc;
}

// ---------------------------------------------------------------- sorting helper
static void radix_sort_u64(std::vector<uint64_t>& a) {
    std::vector<uint64_t> tmp(a.size());
    for (int shift = 0; shift < 64; shift += 16) {
        std::vector<int64_t> cnt(65537, 0);
        for (uint64_t x : a) cnt[((x >> shift) & 0xFFFF) + 1]++;
        for (int i = 0; i < 65536; i++) cnt[i + 1] += cnt[i];
        for (uint64_t x : a) tmp[cnt[(x >> shift) & 0xFFFF]++] = x;
        a.swap(tmp);
    }
}

static int64_t keys_to_csr(std::vector<uint64_t>& keys, int64_t n, int32_t* row_ptr, int32_t* col_idx) {
    radix_sort_u64(keys);
    keys.erase(std::unique(keys.begin(), keys.end()), keys.end());
    std::fill(row_ptr, row_ptr + n + 1, 0);
    for (uint64_t k : keys) row_ptr[(k >> 32) + 1]++;
    for (int64_t v = 0; v < n; v++) row_ptr[v + 1] += row_ptr[v];
    for (size_t i = 0; i < keys.size(); i++) col_idx[i] = (int32_t)(keys[i] & 0xFFFFFFFFu);
    return (int64_t)keys.size();
}

// R-MAT (Graph500 bit sampling).  n = 2^scale, samples = edge_factor * n.
//   col_idx capacity: samples.  Returns nnz after dropping self-loops and duplicates.
int64_t gen_rmat(int scale, int64_t edge_factor, double a, double b, double c, uint64_t seed,
                 int permute, int32_t* row_ptr, int32_t* col_idx) {
    const int64_t n = (int64_t)1 << scale;
    const int64_t samples = edge_factor * n;
    // random relabelling (Fisher-Yates driven by a counter-based hash)
    std::vector<uint32_t> perm(n);
    for (int64_t i = 0; i < n; i++) perm[i] = (uint32_t)i;
    if (permute)
        for (int64_t i = n - 1; i > 0; i--) {
            int64_t j = (int64_t)(splitmix64(splitmix64(seed ^ 0xABCDEF) + (uint64_t)i) % (uint64_t)(i + 1));
            std::swap(perm[i], perm[j]);
        }
    std::vector<uint64_t> keys(samples);
    const double ab = a + b, abc = a + b + c;
#pragma omp parallel for schedule(static)
    for (int64_t k = 0; k < samples; k++) {
        uint64_t u = 0, v = 0;
        const uint64_t h = hash3(seed, 0x524D4154ull, (uint64_t)k);
        for (int l = 0; l < scale; l++) {
            const double r = unit(splitmix64(h + (uint64_t)l));
            uint64_t ub, vb;
            if (r < a) { ub = 0; vb = 0; }
            else if (r < ab) { ub = 0; vb = 1; }
            else if (r < abc) { ub = 1; vb = 0; }
            else { ub = 1; vb = 1; }
            u = (u << 1) | ub;
            v = (v << 1) | vb;
        }
        u = perm[u]; v = perm[v];
        keys[k] = (u == v) ? ~0ull : ((u << 32) | v);
    }
    // drop self-loops (marked ~0)
    int64_t w = 0;
    for (int64_t k = 0; k < samples; k++) if (keys[k] != ~0ull) keys[w++] = keys[k];
    keys.resize(w);
    return keys_to_csr(keys, n, row_ptr, col_idx);
}

// G(n, m): m distinct ordered pairs (u, v), u != v.  col_idx capacity m.  Returns m (or
// fewer if m > n(n-1)).
int64_t gen_gnm(int64_t n, int64_t m, uint64_t seed, int32_t* row_ptr, int32_t* col_idx) {
    const int64_t maxm = n * (n - 1);
    if (m > maxm) m = maxm;
    std::unordered_set<uint64_t> seen;
    std::vector<uint64_t> keys;
    keys.reserve(m);
    for (uint64_t k = 0; (int64_t)keys.size() < m; k++) {
        const uint64_t r = hash3(seed, 0x474E4Dull, k);
        const uint64_t u = (r >> 32) % (uint64_t)n, v = (r & 0xFFFFFFFFu) % (uint64_t)n;
        if (u == v) continue;
        const uint64_t key = (u << 32) | v;
        if (seen.insert(key).second) keys.push_back(key);
    }
    return keys_to_csr(keys, n, row_ptr, col_idx);
}

// FNV-1a hash of a CSR (to pin generator reproducibility across machines).
uint64_t csr_hash(int64_t n, const int32_t* row_ptr, int64_t nnz, const int32_t* col_idx) {
    uint64_t h = 1469598103934665603ull;
    auto mix = [&](const void* p, size_t bytes) {
        const unsigned char* c = (const unsigned char*)p;
        for (size_t i = 0; i < bytes; i++) { h ^= c[i]; h *= 1099511628211ull; }
    };
    mix(row_ptr, sizeof(int32_t) * (size_t)(n + 1));
    mix(col_idx, sizeof(int32_t) * (size_t)nnz);
    return h;
}

}  // extern "C"
