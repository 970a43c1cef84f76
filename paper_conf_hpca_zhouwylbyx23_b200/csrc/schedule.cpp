// NEXT-2: 1F1B swap schedule with the live-interval check
// (include/mpress.h: mpress_schedule_1f1b; reading R24).
//
// Paper: P:62-77 / P:87-89 (1F1B pipelines keep more micro-batches alive on
// early stages), P:145 + P:236 (swap-out and swap-in operators on their own
// streams beside compute), P:219 + fn.1 P:226 (a swap is free when the live
// interval -- backward timestamp minus forward timestamp -- covers it),
// P:281 (computation-balanced stages).
//
// The timeline is a DAG: every resource (S compute stages; one or two swap
// streams) runs its ops in a fixed order, and an op starts when its
// resource predecessor and its data dependencies have ended.  Start times are
// longest paths, computed here by a topological (Kahn) pass over an explicit
// edge list; the oracle evaluates the same definition by sweeping resources.
#include <algorithm>
#include <new>
#include <vector>

#include "common.h"

namespace mpress {
namespace {

struct Graph {
  std::vector<uint64_t> dur;
  std::vector<std::vector<int>> succ;
  std::vector<int> indeg;
  int add(uint64_t d) {
    dur.push_back(d);
    succ.emplace_back();
    indeg.push_back(0);
    return (int)dur.size() - 1;
  }
  void edge(int a, int b) {
    if (a < 0 || b < 0) return;
    succ[a].push_back(b);
    ++indeg[b];
  }
  // start/end of every node; false if the graph has a cycle
  bool longest(std::vector<uint64_t>* st, std::vector<uint64_t>* en) {
    const size_t n = dur.size();
    st->assign(n, 0);
    en->assign(n, 0);
    std::vector<int> deg = indeg, q;
    for (size_t i = 0; i < n; ++i)
      if (deg[i] == 0) q.push_back((int)i);
    size_t seen = 0;
    for (size_t h = 0; h < q.size(); ++h) {
      const int u = q[h];
      ++seen;
      (*en)[u] = (*st)[u] + dur[u];
      for (int v : succ[u]) {
        (*st)[v] = std::max((*st)[v], (*en)[u]);
        if (--deg[v] == 0) q.push_back(v);
      }
    }
    return seen == n;
  }
};

// op j of stage k in 1F1B order: kind (0 = F, 1 = B) and micro-batch
struct Op {
  int kind, m;
};

std::vector<Op> stage_ops(uint32_t S, uint32_t k, uint32_t M) {
  const uint32_t W = std::min(S - 1 - k, M);
  std::vector<Op> ops;
  for (uint32_t m = 0; m < W; ++m) ops.push_back({0, (int)m});
  for (uint32_t i = 0; i < M; ++i) {
    if (W + i < M) ops.push_back({0, (int)(W + i)});
    ops.push_back({1, (int)i});
  }
  return ops;
}

struct Pipeline {
  uint32_t S, M;
  std::vector<std::vector<Op>> ops;          // [stage][j]
  std::vector<std::vector<int>> fnode, bnode;  // [stage][m] -> node
  Graph g;
  void build(uint64_t tf, uint64_t tb) {
    ops.resize(S);
    fnode.assign(S, std::vector<int>(M, -1));
    bnode.assign(S, std::vector<int>(M, -1));
    for (uint32_t k = 0; k < S; ++k) {
      ops[k] = stage_ops(S, k, M);
      int prev = -1;
      for (const Op& o : ops[k]) {
        const int v = g.add(o.kind == 0 ? tf : tb);
        (o.kind == 0 ? fnode : bnode)[k][o.m] = v;
        g.edge(prev, v);  // resource order
        prev = v;
      }
    }
    for (uint32_t k = 0; k < S; ++k)
      for (uint32_t m = 0; m < M; ++m) {
        if (k > 0) g.edge(fnode[k - 1][m], fnode[k][m]);
        g.edge(k + 1 < S ? bnode[k + 1][m] : fnode[k][m], bnode[k][m]);
      }
  }
};

uint32_t peak(std::vector<std::pair<uint64_t, int>> ev) {
  std::sort(ev.begin(), ev.end());  // (time, -1) sorts before (time, +1)
  int cur = 0, best = 0;
  for (auto& e : ev) best = std::max(best, cur += e.second);
  return (uint32_t)best;
}

void interval(std::vector<std::pair<uint64_t, int>>* ev, uint64_t a, uint64_t b) {
  if (b > a) {
    ev->push_back({a, 1});
    ev->push_back({b, -1});
  }
}

}  // namespace
}  // namespace mpress

using namespace mpress;

extern "C" int mpress_schedule_1f1b(const mpress_1f1b_params* p, mpress_1f1b_slot* slots,
                                    mpress_1f1b_summary* summary) {
  if (!p || !slots) return fail(MPRESS_ERR_ARG, "mpress_schedule_1f1b: null argument");
  const uint32_t S = p->stages, M = p->micro_batches, e = p->stage;
  if (S == 0 || M == 0 || e >= S || S > 4096 || M > 65536)
    return fail(MPRESS_ERR_ARG, "mpress_schedule_1f1b: bad stages/stage/micro_batches");
  try {
    // 1. the no-swap timeline
    Pipeline base{S, M, {}, {}, {}, {}};
    base.build(p->t_fwd_ns, p->t_bwd_ns);
    std::vector<uint64_t> s0, e0;
    if (!base.g.longest(&s0, &e0)) return fail(MPRESS_ERR_ARG, "mpress_schedule_1f1b: cyclic model");
    const std::vector<Op>& ops = base.ops[e];
    std::vector<int> jf(M), jb(M);
    for (size_t j = 0; j < ops.size(); ++j) (ops[j].kind == 0 ? jf : jb)[ops[j].m] = (int)j;
    auto node_of = [&](const Pipeline& P, uint32_t k, size_t j) {
      const Op& o = P.ops[k][j];
      return (o.kind == 0 ? P.fnode : P.bnode)[k][o.m];
    };
    // 2. trigger op of each swap-in: the last op in [F(m), B(m)) whose no-swap
    //    end leaves t_in before B(m)'s no-swap start
    std::vector<int> trig(M);
    for (uint32_t m = 0; m < M; ++m) {
      const uint64_t bs = s0[base.bnode[e][m]];
      int j = jf[m];
      for (int jj = jf[m]; jj < jb[m]; ++jj) {
        const uint64_t end = e0[node_of(base, e, jj)];
        if (end + p->t_in_ns + p->t_slack_ns <= bs) j = jj;  // end <= bs - t_in - slack, no underflow
      }
      trig[m] = j;
    }
    // 3. the timeline with the swap ops of stage e, in executor enqueue order
    Pipeline sw{S, M, {}, {}, {}, {}};
    sw.build(p->t_fwd_ns, p->t_bwd_ns);
    std::vector<int> outn(M, -1), inn(M, -1);
    int last_out = -1, last_in = -1;  // stream order (duplex: two streams)
    for (size_t j = 0; j < ops.size(); ++j) {
      if (ops[j].kind == 0) {
        const int m = ops[j].m;
        const int v = sw.g.add(p->t_out_ns);
        outn[m] = v;
        sw.g.edge(sw.fnode[e][m], v);
        sw.g.edge(last_out, v);
        last_out = v;
        if (!p->duplex) last_in = v;
      }
      for (uint32_t m = 0; m < M; ++m) {
        if (trig[m] != (int)j) continue;
        const int v = sw.g.add(p->t_in_ns);
        inn[m] = v;
        sw.g.edge(outn[m], v);
        sw.g.edge(node_of(sw, e, j), v);
        sw.g.edge(last_in, v);
        last_in = v;
        if (!p->duplex) last_out = v;
        sw.g.edge(v, sw.bnode[e][m]);  // B(m) needs its activations back
      }
    }
    std::vector<uint64_t> s1, e1;
    if (!sw.g.longest(&s1, &e1)) return fail(MPRESS_ERR_ARG, "mpress_schedule_1f1b: cyclic model");
    // 4. per micro-batch results
    std::vector<std::pair<uint64_t, int>> ev0, ev1;
    for (uint32_t m = 0; m < M; ++m) {
      const int f = sw.fnode[e][m], b = sw.bnode[e][m];
      mpress_1f1b_slot& o = slots[m];
      o.fwd_start = s1[f];
      o.fwd_end = e1[f];
      o.bwd_start = s1[b];
      o.bwd_end = e1[b];
      o.live_ns = s0[base.bnode[e][m]] - e0[base.fnode[e][m]];
      o.out_start = s1[outn[m]];
      o.out_end = e1[outn[m]];
      o.in_start = s1[inn[m]];
      o.in_end = e1[inn[m]];
      o.in_trigger = (uint32_t)trig[m];
      // ready without the swap-in: previous op of the stage and the data dependency
      uint64_t ready = e1[node_of(sw, e, jb[m] - 1)];
      const int dep = e + 1 < S ? sw.bnode[e + 1][m] : sw.fnode[e][m];
      ready = std::max(ready, e1[dep]);
      o.hidden = e1[inn[m]] <= ready ? 1u : 0u;
      o.exposed_ns = s1[b] - s0[base.bnode[e][m]];
      interval(&ev0, s0[base.fnode[e][m]], e0[base.bnode[e][m]]);
      interval(&ev1, s1[f], e1[outn[m]]);
      interval(&ev1, s1[inn[m]], e1[b]);
    }
    if (summary) {
      uint64_t mk0 = 0, mk1 = 0;
      for (uint32_t k = 0; k < S; ++k)
        for (uint32_t m = 0; m < M; ++m) {
          mk0 = std::max({mk0, e0[base.fnode[k][m]], e0[base.bnode[k][m]]});
          mk1 = std::max({mk1, e1[sw.fnode[k][m]], e1[sw.bnode[k][m]]});
        }
      summary->makespan_ns = mk1;
      summary->makespan_noswap_ns = mk0;
      summary->peak_resident = peak(ev1);
      summary->peak_resident_noswap = peak(ev0);
      summary->ops = (uint32_t)ops.size();
    }
  } catch (const std::bad_alloc&) {
    return fail(MPRESS_ERR_ARG, "mpress_schedule_1f1b: out of host memory");
  }
  return MPRESS_OK;
}
