// NEXT-4: memory-compaction decision rule (include/mpress.h:
// mpress_compaction_plan; §III-D, Table III, reading R26).
//
// Per tensor, three ways to free its GPU memory for its live interval:
// GPU-CPU swap over PCIe (the pinned host tier, MPRESS_DEVICE_HOST),
// recomputation, or D2D swap into a peer's spare HBM.  A swap is free when the
// live interval covers it and otherwise costs the difference (fn.2,
// P:238); recomputation always costs its forward time.  The initial
// assignment takes the cheaper of GPU-CPU swap and recomputation;
// then the tensors with the largest overhead move to D2D while spare memory
// lasts and D2D is strictly cheaper.  Ties keep the option that
// spends no spare GPU memory.
#include <algorithm>
#include <new>
#include <vector>

#include "common.h"

namespace {
inline uint64_t swap_overhead(uint64_t cost, uint64_t live) { return cost > live ? cost - live : 0; }
}  // namespace

using namespace mpress;

extern "C" int mpress_compaction_plan(uint32_t n, const mpress_tensor_stat* stats, uint64_t d2d_capacity,
                                      uint32_t* choice, uint64_t* overhead_ns, uint64_t* total_overhead_ns,
                                      uint64_t* d2d_bytes) {
  if ((n && (!stats || !choice)) || !total_overhead_ns)
    return fail(MPRESS_ERR_ARG, "mpress_compaction_plan: null argument");
  try {
    std::vector<uint64_t> ovh(n);
    for (uint32_t i = 0; i < n; ++i) {
      const mpress_tensor_stat& t = stats[i];
      const uint64_t c = swap_overhead(t.cpu_swap_ns, t.live_ns);
      if (t.recompute_ns != MPRESS_NOT_RECOMPUTABLE && t.recompute_ns < c) {
        choice[i] = MPRESS_CHOICE_RECOMPUTE;
        ovh[i] = t.recompute_ns;
      } else {
        choice[i] = MPRESS_CHOICE_CPU_SWAP;
        ovh[i] = c;
      }
    }
    std::vector<uint32_t> order(n);
    for (uint32_t i = 0; i < n; ++i) order[i] = i;
    std::stable_sort(order.begin(), order.end(), [&](uint32_t a, uint32_t b) { return ovh[a] > ovh[b]; });
    uint64_t left = d2d_capacity, used = 0;
    for (uint32_t i : order) {
      const uint64_t d = swap_overhead(stats[i].d2d_swap_ns, stats[i].live_ns);
      if (d < ovh[i] && stats[i].bytes <= left) {
        choice[i] = MPRESS_CHOICE_D2D;
        ovh[i] = d;
        left -= stats[i].bytes;
        used += stats[i].bytes;
      }
    }
    uint64_t total = 0;
    for (uint32_t i = 0; i < n; ++i) {
      total += ovh[i];
      if (overhead_ns) overhead_ns[i] = ovh[i];
    }
    *total_overhead_ns = total;
    if (d2d_bytes) *d2d_bytes = used;
  } catch (const std::bad_alloc&) {
    return fail(MPRESS_ERR_ARG, "mpress_compaction_plan: out of host memory");
  }
  return MPRESS_OK;
}
