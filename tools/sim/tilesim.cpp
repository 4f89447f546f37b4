// tilesim.cpp -- CPU model of Phase 2 (one outer iteration) with tile-local fixed points
// and synchronous passes between tiles (development tool: evaluates tile shapes and
// priority choices without a GPU).  Jacobi across tiles (a tile reads the other tiles'
// values from the previous pass), exact local fixed point inside a tile (worklist),
// dirty-tile skipping.  Counts passes, tile visits, visited vertices and value raises.
#include <cstdint>
#include <cstring>
#include <vector>
#include <deque>
#include <algorithm>

#include <queue>
extern "C" int64_t tilesim(int32_t n, const int32_t* rp, const int32_t* ci, const int32_t* tile_of, int32_t ntiles,
                           const int32_t* prio, int64_t* out /* passes, visits, visited_vertices, raises */, int heap,
                           int gs /* 1: Gauss-Seidel across tiles, alternating order */,
                           const int32_t* order /* tile dispatch order (nullptr: index) */, int32_t window,
                           int32_t kround /* >0: exactly kround Jacobi rounds inside a tile instead of its fixed point */) {
    // CSC
    std::vector<int32_t> cp(n + 1, 0), cr(rp[n]);
    for (int64_t e = 0; e < rp[n]; e++) cp[ci[e] + 1]++;
    for (int v = 0; v < n; v++) cp[v + 1] += cp[v];
    {
        std::vector<int32_t> cur(cp.begin(), cp.end() - 1);
        for (int u = 0; u < n; u++)
            for (int e = rp[u]; e < rp[u + 1]; e++) cr[cur[ci[e]]++] = u;
    }
    std::vector<std::vector<int32_t>> members(ntiles);
    for (int v = 0; v < n; v++) members[tile_of[v]].push_back(v);
    std::vector<int32_t> vin(prio, prio + n), vout(prio, prio + n), sin(n), sout(n), start_in(n), start_out(n);
    std::vector<char> dirty(ntiles, 1), ndirty(ntiles, 0), inq_in(n, 0), inq_out(n, 0);
    std::vector<int64_t> done_at(ntiles, -1);   // dispatch position of the tile in this pass
    std::vector<std::vector<int32_t>> pending(1);
    int64_t pos = 0;
    int64_t passes = 0, visits = 0, vv = 0, raises = 0;
    for (;;) {
        sin = vin; sout = vout;                     // Jacobi snapshot across tiles
        start_in = vin; start_out = vout;
        std::fill(ndirty.begin(), ndirty.end(), 0);
        bool changed = false;
        std::fill(done_at.begin(), done_at.end(), -1);
        int64_t pos0 = pos;
        for (int ti = 0; ti < ntiles; ti++) {
            const int oi = (gs && (passes & 1)) ? ntiles - 1 - ti : ti;
            const int t = order ? order[oi] : oi;
            if (!dirty[t]) continue;
            const int64_t my = pos++;
            if (gs) {   // live values of tiles finished at least `window` dispatches earlier
                for (int v : members[t]) {
                    for (int e = cp[v]; e < cp[v + 1]; e++) {
                        const int u = cr[e], tu = tile_of[u];
                        if (tu != t && done_at[tu] >= 0 && (window < 0 ? (tu / -window == t / -window) : done_at[tu] <= my - window)) sin[u] = vin[u];
                    }
                    for (int e = rp[v]; e < rp[v + 1]; e++) {
                        const int w = ci[e], tw = tile_of[w];
                        if (tw != t && done_at[tw] >= 0 && (window < 0 ? (tw / -window == t / -window) : done_at[tw] <= my - window)) sout[w] = vout[w];
                    }
                }
            }
            visits++; vv += members[t].size();
            std::deque<int32_t> qi, qo;
            // step 1: external pulls, intra-tile initial state
            for (int v : members[t]) {
                int x = vin[v], y = vout[v];
                for (int e = cp[v]; e < cp[v + 1]; e++) { int u = cr[e]; if (tile_of[u] != t) x = std::max(x, sin[u]); }
                for (int e = rp[v]; e < rp[v + 1]; e++) { int w = ci[e]; if (tile_of[w] != t) y = std::max(y, sout[w]); }
                if (x > vin[v]) { vin[v] = x; raises++; }
                if (y > vout[v]) { vout[v] = y; raises++; }
                qi.push_back(v); qo.push_back(v); inq_in[v] = inq_out[v] = 1;
            }
            // step 2: local fixed point by pushes (FIFO, or max-value-first with heap=1)
            if (kround > 0) {
                qi.clear(); qo.clear();
                for (int v : members[t]) inq_in[v] = inq_out[v] = 0;
                std::vector<int32_t> ti, to;
                for (int r = 0; r < kround; r++) {
                    ti.clear(); to.clear();
                    for (int v : members[t]) {
                        int x = vin[v], y = vout[v];
                        for (int e = cp[v]; e < cp[v + 1]; e++) { int u = cr[e]; if (tile_of[u] == t) x = std::max(x, vin[u]); }
                        for (int e = rp[v]; e < rp[v + 1]; e++) { int w = ci[e]; if (tile_of[w] == t) y = std::max(y, vout[w]); }
                        ti.push_back(x); to.push_back(y);
                    }
                    size_t k = 0;
                    for (int v : members[t]) { if (ti[k] > vin[v]) { vin[v] = ti[k]; raises++; } if (to[k] > vout[v]) { vout[v] = to[k]; raises++; } k++; }
                }
            } else if (heap) {
                std::priority_queue<std::pair<int,int>> hi, ho;
                for (int v : members[t]) { hi.push({vin[v], v}); ho.push({vout[v], v}); }
                qi.clear(); qo.clear();
                for (int v : members[t]) inq_in[v] = inq_out[v] = 0;
                while (!hi.empty()) {
                    auto [val, v] = hi.top(); hi.pop();
                    if (val != vin[v]) continue;
                    for (int e = rp[v]; e < rp[v + 1]; e++) {
                        int w = ci[e];
                        if (tile_of[w] == t && vin[w] < val) { vin[w] = val; raises++; hi.push({val, w}); }
                    }
                }
                while (!ho.empty()) {
                    auto [val, v] = ho.top(); ho.pop();
                    if (val != vout[v]) continue;
                    for (int e = cp[v]; e < cp[v + 1]; e++) {
                        int u = cr[e];
                        if (tile_of[u] == t && vout[u] < val) { vout[u] = val; raises++; ho.push({val, u}); }
                    }
                }
            }
            while (!qi.empty()) {
                int v = qi.front(); qi.pop_front(); inq_in[v] = 0;
                for (int e = rp[v]; e < rp[v + 1]; e++) {
                    int w = ci[e];
                    if (tile_of[w] == t && vin[w] < vin[v]) { vin[w] = vin[v]; raises++; if (!inq_in[w]) { inq_in[w] = 1; qi.push_back(w); } }
                }
            }
            while (!qo.empty()) {
                int v = qo.front(); qo.pop_front(); inq_out[v] = 0;
                for (int e = cp[v]; e < cp[v + 1]; e++) {
                    int u = cr[e];
                    if (tile_of[u] == t && vout[u] < vout[v]) { vout[u] = vout[v]; raises++; if (!inq_out[u]) { inq_out[u] = 1; qo.push_back(u); } }
                }
            }
            done_at[t] = my;
            // step 3: dirty marking for raised vertices
            for (int v : members[t]) {
                if (vin[v] > start_in[v]) { changed = true; for (int e = rp[v]; e < rp[v + 1]; e++) if (tile_of[ci[e]] != t) ndirty[tile_of[ci[e]]] = 1; }
                if (vout[v] > start_out[v]) { changed = true; for (int e = cp[v]; e < cp[v + 1]; e++) if (tile_of[cr[e]] != t) ndirty[tile_of[cr[e]]] = 1; }
            }
        }
        passes++;
        if (!changed) break;
        dirty.swap(ndirty);
    }
    out[0] = passes; out[1] = visits; out[2] = vv; out[3] = raises;
    return passes;
}
