// asyncsim.cpp -- CPU model of the asynchronous Phase 2 (one outer iteration): W tiles in
// flight per round (they read a common snapshot of the other tiles' values), tile-local
// fixed points, neighbour marks.  Policies for choosing the next tiles:
//   0  sweep cursor over the tile indices, alternating direction (k_prop_async)
//   1  highest trigger value first (the largest value that dirtied the tile)
// Counts rounds, tile visits and value raises (development tool).
#include <algorithm>
#include <cmath>
#include <cstdint>
#include <cstring>
#include <deque>
#include <vector>

extern "C" int64_t asyncsim(int32_t n, const int32_t* rp, const int32_t* ci, const int32_t* tile_of, int32_t ntiles,
                            const int32_t* prio, int32_t window, int32_t policy, int64_t* out) {
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
    std::vector<int32_t> vin(prio, prio + n), vout(prio, prio + n), sin(n), sout(n);
    std::vector<char> dirty(ntiles, 1), inq_in(n, 0), inq_out(n, 0);
    std::vector<int64_t> trig(ntiles, 0);
    for (int t = 0; t < ntiles; t++)
        for (int v : members[t]) trig[t] = std::max<int64_t>(trig[t], prio[v]);
    int64_t rounds = 0, visits = 0, raises = 0, cursor = 0;
    std::vector<int> pick;
    for (;;) {
        pick.clear();
        if (policy == 0) {
            for (int64_t k = 0; k < ntiles && (int)pick.size() < window; k++, cursor++) {
                const int64_t sweep = cursor / ntiles, off = cursor % ntiles;
                const int t = (int)((sweep & 1) ? ntiles - 1 - off : off);
                if (dirty[t]) pick.push_back(t);
            }
        } else if (policy >= 2) {
            // sweep cursor, but only tiles whose trigger bucket is within `slack` of the best
            // dirty bucket (bucket = floor(2 log2(n - trig)): half-octaves below the top)
            const int slack = policy - 2;
            auto bucket = [&](int64_t tr) { double k = (double)n - (double)tr; return (int)(2.0 * std::log2(k)); };
            int best = 1 << 30;
            for (int t = 0; t < ntiles; t++)
                if (dirty[t]) best = std::min(best, bucket(trig[t]));
            for (int64_t k = 0; k < ntiles && (int)pick.size() < window; k++, cursor++) {
                const int64_t sweep = cursor / ntiles, off = cursor % ntiles;
                const int t = (int)((sweep & 1) ? ntiles - 1 - off : off);
                if (dirty[t] && bucket(trig[t]) <= best + slack) pick.push_back(t);
            }
        } else {
            std::vector<std::pair<int64_t, int>> cand;
            for (int t = 0; t < ntiles; t++)
                if (dirty[t]) cand.push_back({trig[t], t});
            const size_t k = std::min<size_t>(cand.size(), (size_t)window);
            std::partial_sort(cand.begin(), cand.begin() + k, cand.end(), std::greater<>());
            for (size_t i = 0; i < k; i++) pick.push_back(cand[i].second);
        }
        if (pick.empty()) {
            bool any = false;
            for (int t = 0; t < ntiles; t++) any |= dirty[t];
            if (!any) break;
            continue;
        }
        rounds++;
        sin = vin;
        sout = vout;
        for (int t : pick) { dirty[t] = 0; trig[t] = 0; }
        for (int t : pick) {
            visits++;
            std::deque<int32_t> qi, qo;
            std::vector<int32_t> x0, y0;
            for (int v : members[t]) {
                x0.push_back(vin[v]);
                y0.push_back(vout[v]);
                int x = vin[v], y = vout[v];
                for (int e = cp[v]; e < cp[v + 1]; e++) { int u = cr[e]; if (tile_of[u] != t) x = std::max(x, sin[u]); }
                for (int e = rp[v]; e < rp[v + 1]; e++) { int w = ci[e]; if (tile_of[w] != t) y = std::max(y, sout[w]); }
                if (x > vin[v]) { vin[v] = x; raises++; }
                if (y > vout[v]) { vout[v] = y; raises++; }
                qi.push_back(v); qo.push_back(v); inq_in[v] = inq_out[v] = 1;
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
            size_t k = 0;
            for (int v : members[t]) {
                if (vin[v] > x0[k])
                    for (int e = rp[v]; e < rp[v + 1]; e++) { int tw = tile_of[ci[e]]; if (tw != t) { dirty[tw] = 1; trig[tw] = std::max<int64_t>(trig[tw], vin[v]); } }
                if (vout[v] > y0[k])
                    for (int e = cp[v]; e < cp[v + 1]; e++) { int tu = tile_of[cr[e]]; if (tu != t) { dirty[tu] = 1; trig[tu] = std::max<int64_t>(trig[tu], vout[v]); } }
                k++;
            }
        }
    }
    out[0] = rounds; out[1] = visits; out[2] = raises;
    return rounds;
}
