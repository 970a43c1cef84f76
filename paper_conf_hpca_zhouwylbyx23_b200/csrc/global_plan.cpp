// NEXT-1: joint plan of several exporters (include/mpress.h:
// mpress_plan_global).
//
// Fig. 6 enumerates, per importer, every way to distribute its
// spare memory among the overflowed exporters that are its NVLink neighbours
// (lines 2-8), combines the single-GPU plans (line 20) and keeps the one with
// the best score, the reciprocal of the maximal D2D swap time (R1).
// The enumeration is exponential; here the same optimum is found exactly in
// polynomial time (reading R23):
//
//   * for a time bound T the question "can every unit be placed?" is a
//     max-flow: source -> exporter s (K_s units), s -> importer p
//     (floor(T * B_sp) units, the link), p -> sink (min(cap_p, floor(T * I_p))),
//     plus K_s <= T * E_s for the exporter's egress port;
//   * feasibility is monotone in T and the optimum T* is one of the values
//     k / w (k integer, w one of the model's weights), so for every weight w
//     a binary search finds the least feasible k; T* = min_w k_w / w;
//   * the integral max-flow at T* is the assignment (Dinic, deterministic:
//     every rank computes the same units).
// All comparisons are exact (128-bit integer cross products).
#include <algorithm>
#include <limits>
#include <new>
#include <vector>

#include "common.h"

namespace mpress {
namespace {

using u128 = unsigned __int128;
constexpr uint64_t kInf = std::numeric_limits<uint64_t>::max();

struct Dinic {
  struct Edge {
    int to;
    uint64_t cap;
  };
  std::vector<Edge> e;
  std::vector<std::vector<int>> g;
  std::vector<int> level, it;
  explicit Dinic(int n) : g(n), level(n), it(n) {}
  int add(int u, int v, uint64_t c) {
    e.push_back({v, c});
    g[u].push_back((int)e.size() - 1);
    e.push_back({u, 0});
    g[v].push_back((int)e.size() - 1);
    return (int)e.size() - 2;
  }
  bool bfs(int s, int t) {
    std::fill(level.begin(), level.end(), -1);
    std::vector<int> q{s};
    level[s] = 0;
    for (size_t h = 0; h < q.size(); ++h)
      for (int id : g[q[h]])
        if (e[id].cap > 0 && level[e[id].to] < 0) {
          level[e[id].to] = level[q[h]] + 1;
          q.push_back(e[id].to);
        }
    return level[t] >= 0;
  }
  uint64_t dfs(int u, int t, uint64_t f) {
    if (u == t) return f;
    for (int& i = it[u]; i < (int)g[u].size(); ++i) {
      Edge& ed = e[g[u][i]];
      if (ed.cap > 0 && level[ed.to] == level[u] + 1) {
        uint64_t d = dfs(ed.to, t, std::min(f, ed.cap));
        if (d > 0) {
          ed.cap -= d;
          e[g[u][i] ^ 1].cap += d;
          return d;
        }
      }
    }
    return 0;
  }
  u128 run(int s, int t) {
    u128 flow = 0;
    while (bfs(s, t)) {
      std::fill(it.begin(), it.end(), 0);
      while (uint64_t f = dfs(s, t, kInf)) flow += f;
    }
    return flow;
  }
};

struct Problem {
  int world;
  std::vector<int> src;            // exporters
  std::vector<uint64_t> K;         // units per exporter
  std::vector<uint64_t> cap;       // units per importer
  const uint64_t* bw;              // [world*world]
  const uint64_t* egress;          // [world] or null
  const uint64_t* ingress;         // [world] or null
};

inline bool link(const Problem& P, int s, int p) { return p != s && P.bw[(size_t)s * P.world + p] > 0 && P.cap[p] > 0; }

// floor(k * B / w), saturated to 64 bits
inline uint64_t scaled(uint64_t k, uint64_t B, uint64_t w) {
  u128 v = (u128)k * B / w;
  return v > kInf ? kInf : (uint64_t)v;
}

// Can every unit be routed within time k / w?  Fills x[si*world+p] if asked.
bool feasible(const Problem& P, uint64_t k, uint64_t w, std::vector<uint64_t>* x) {
  const int S = (int)P.src.size(), W = P.world;
  u128 total = 0;
  for (int si = 0; si < S; ++si) {
    total += P.K[si];
    const int s = P.src[si];
    if (P.egress && P.egress[s] > 0 && (u128)P.K[si] * w > (u128)k * P.egress[s]) return false;
  }
  Dinic d(2 + S + W);
  const int so = 0, si_ = 1;
  std::vector<int> eid((size_t)S * W, -1);
  for (int i = 0; i < S; ++i) {
    d.add(so, 2 + i, P.K[i]);
    const int s = P.src[i];
    for (int p = 0; p < W; ++p)
      if (link(P, s, p)) eid[(size_t)i * W + p] = d.add(2 + i, 2 + S + p, scaled(k, P.bw[(size_t)s * W + p], w));
  }
  for (int p = 0; p < W; ++p) {
    uint64_t c = P.cap[p];
    if (P.ingress && P.ingress[p] > 0) c = std::min(c, scaled(k, P.ingress[p], w));
    if (c) d.add(2 + S + p, si_, c);
  }
  if (d.run(so, si_) != total) return false;
  if (x) {
    x->assign((size_t)S * W, 0);
    for (size_t j = 0; j < eid.size(); ++j)
      if (eid[j] >= 0) (*x)[j] = d.e[eid[j] ^ 1].cap;  // flow = reverse residual
  }
  return true;
}

// T* = min over the model's weights w of (least k with feasible(k / w)) / w.
// Returns false when no T places every unit (capacity).
bool solve(const Problem& P, uint64_t* best_k, uint64_t* best_w) {
  const int world = P.world;
  u128 total = 0;
  for (uint64_t k : P.K) total += k;
  std::vector<uint64_t> weights;  // every usable link, egress and ingress port
  for (int s : P.src)
    for (int p = 0; p < world; ++p)
      if (link(P, s, p)) weights.push_back(P.bw[(size_t)s * world + p]);
  for (int s : P.src)
    if (P.egress && P.egress[s] > 0) weights.push_back(P.egress[s]);
  for (int p = 0; p < world; ++p)
    if (P.ingress && P.ingress[p] > 0) weights.push_back(P.ingress[p]);
  std::sort(weights.begin(), weights.end());
  weights.erase(std::unique(weights.begin(), weights.end()), weights.end());
  if (weights.empty() || !feasible(P, (uint64_t)total * weights.back() + 1, 1, nullptr)) return false;
  *best_k = 0;
  *best_w = 0;
  for (uint64_t w : weights) {
    // a smaller k/w than the best so far is all that matters: start there
    uint64_t hi = *best_w ? (uint64_t)(((u128)*best_k * w) / *best_w) + 1 : (uint64_t)total;
    if (*best_w && !feasible(P, hi, w, nullptr)) continue;  // cannot beat the best
    uint64_t lo = 0;
    while (!*best_w && !feasible(P, hi, w, nullptr)) {
      if (hi > kInf / 2) { hi = 0; break; }
      lo = hi;
      hi *= 2;
    }
    if (hi == 0) continue;
    while (hi - lo > 1) {  // invariant: lo infeasible (or 0), hi feasible
      const uint64_t mid = lo + (hi - lo) / 2;
      if (feasible(P, mid, w, nullptr)) hi = mid; else lo = mid;
    }
    if (*best_w == 0 || (u128)hi * *best_w < (u128)*best_k * w) {
      *best_k = hi;
      *best_w = w;
    }
  }
  return *best_w != 0;
}

}  // namespace
}  // namespace mpress

using namespace mpress;

extern "C" int mpress_map_search(int n, const uint64_t* demand, const uint64_t* spare, const uint64_t* link,
                                 const uint64_t* egress, const uint64_t* ingress, uint64_t granule,
                                 int32_t* stage_to_gpu, uint64_t* makespan_num, uint64_t* makespan_den,
                                 uint64_t* evaluated) {
  if (n < 1 || n > 10 || !demand || !spare || !link || !stage_to_gpu)
    return fail(MPRESS_ERR_ARG, "mpress_map_search: bad argument (1 <= n <= 10)");
  const uint64_t G = granule ? granule : MPRESS_DEFAULT_GRANULE;
  if (G % MPRESS_ALIGN != 0) return fail(MPRESS_ERR_ARG, "mpress_map_search: granule not a multiple of 256");
  std::vector<uint64_t> units(n, 0);
  bool any = false;
  for (int s = 0; s < n; ++s) {
    if (demand[s] == 0) continue;
    uint64_t V;
    if (demand[s] > UINT64_MAX - 255) return fail(MPRESS_ERR_ARG, "mpress_map_search: demand too large");
    V = roundup(demand[s], MPRESS_ALIGN);
    units[s] = V / G + (V % G != 0);
    any = true;
  }
  if (!any) return fail(MPRESS_ERR_ARG, "mpress_map_search: no stage overflows");
  std::vector<int> perm(n);
  for (int i = 0; i < n; ++i) perm[i] = i;
  uint64_t best_k = 0, best_w = 0, count = 0;
  std::vector<int> best_perm;
  Problem P;
  P.world = n;
  P.bw = link;
  P.egress = egress;
  P.ingress = ingress;
  try {
    do {  // lexicographic order of (gpu of stage 0, gpu of stage 1, ...)
      ++count;
      P.src.clear();
      P.K.clear();
      P.cap.assign(n, 0);
      for (int s = 0; s < n; ++s) {
        if (demand[s] > 0) {
          P.src.push_back(perm[s]);
          P.K.push_back(units[s]);
        } else {
          P.cap[perm[s]] = spare[s] / G;
        }
      }
      uint64_t k, w;
      if (!solve(P, &k, &w)) continue;
      if (best_w == 0 || (u128)k * best_w < (u128)best_k * w) {
        best_k = k;
        best_w = w;
        best_perm = perm;
      }
    } while (std::next_permutation(perm.begin(), perm.end()));
  } catch (const std::bad_alloc&) {
    return fail(MPRESS_ERR_ARG, "mpress_map_search: out of host memory");
  }
  if (evaluated) *evaluated = count;
  if (best_w == 0) return fail(MPRESS_ERR_NO_SPACE, "mpress_map_search: no mapping fits the demand");
  for (int s = 0; s < n; ++s) stage_to_gpu[s] = best_perm[s];
  if (makespan_num) *makespan_num = best_k;
  if (makespan_den) *makespan_den = best_w;
  return MPRESS_OK;
}

extern "C" int mpress_plan_global(int world, uint32_t n_sources, const int32_t* sources,
                                  const uint32_t* n_tensors, const uint64_t* sizes_flat,
                                  const uint64_t* spare_bytes, const uint64_t* bw_matrix,
                                  const uint64_t* egress, const uint64_t* ingress, uint64_t granule,
                                  uint64_t* units_out, uint64_t* makespan_num, uint64_t* makespan_den) {
  if (world < 1 || n_sources == 0 || !sources || !n_tensors || !sizes_flat || !spare_bytes || !bw_matrix ||
      !units_out)
    return fail(MPRESS_ERR_ARG, "mpress_plan_global: null argument");
  const uint64_t G = granule ? granule : MPRESS_DEFAULT_GRANULE;
  if (G % MPRESS_ALIGN != 0) return fail(MPRESS_ERR_ARG, "mpress_plan_global: granule not a multiple of 256");
  Problem P;
  P.world = world;
  P.bw = bw_matrix;
  P.egress = egress;
  P.ingress = ingress;
  P.cap.resize(world);
  for (int p = 0; p < world; ++p) P.cap[p] = spare_bytes[p] / G;
  std::vector<char> seen(world, 0);
  size_t off = 0;
  u128 total = 0;
  for (uint32_t i = 0; i < n_sources; ++i) {
    const int s = sources[i];
    if (s < 0 || s >= world || seen[s])
      return fail(MPRESS_ERR_ARG, "mpress_plan_global: bad or repeated source %d", s);
    seen[s] = 1;
    if (n_tensors[i] == 0) return fail(MPRESS_ERR_ARG, "mpress_plan_global: source %d has no tensors", s);
    uint64_t V = 0;
    for (uint32_t j = 0; j < n_tensors[i]; ++j) {
      const uint64_t b = sizes_flat[off + j];
      if (b == 0 || b > UINT64_MAX - 255 || !add_ok(V, roundup(b, MPRESS_ALIGN), &V))
        return fail(MPRESS_ERR_ARG, "mpress_plan_global: bad tensor size");
    }
    off += n_tensors[i];
    P.src.push_back(s);
    P.K.push_back(V / G + (V % G != 0));
    total += P.K.back();
  }
  if (total > kInf) return fail(MPRESS_ERR_ARG, "mpress_plan_global: too many units");
  uint64_t best_k = 0, best_w = 0;
  if (!solve(P, &best_k, &best_w))
    return fail(MPRESS_ERR_NO_SPACE, "mpress_plan_global: the importers' spare memory cannot hold all batches");
  std::vector<uint64_t> x;
  feasible(P, best_k, best_w, &x);
  for (size_t i = 0; i < (size_t)n_sources * world; ++i) units_out[i] = x[i];
  if (makespan_num) *makespan_num = best_k;
  if (makespan_den) *makespan_den = best_w;
  return MPRESS_OK;
}
