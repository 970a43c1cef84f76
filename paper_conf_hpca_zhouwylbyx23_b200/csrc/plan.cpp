// Stripe planner (include/mpress.h: mpress_plan, mpress_partition_sequential).
//
// Paper: P:151 equal sub-blocks on symmetric links; P:153 / P:209 sub-block
// sizes proportional to link bandwidth, tensors batched; Fig. 6 line 3
// spare = MEM_CAP - MEM_USE caps every importer; P:213 score = 1 / maximal
// D2D swap time.  Readings R1-R10 fix the discrete rule: K
// units of G bytes, k_p minimising max k_p/B_p under k_p <= cap_p, ties to the
// lower device index.
//
// The unique assignment satisfying that rule is the set of the K smallest
// "unit values" (j/B_p, p), j = 1..cap_p, in lexicographic order.  This
// implementation reaches it by
//   (1) a continuous water-fill: lambda with sum_p min(cap_p, lambda*B_p) = K,
//       solved on the sorted saturation points (double precision), giving
//       k_p = min(cap_p, floor(lambda*B_p));
//   (2) an exact integer fix-up with 128-bit cross-multiplied comparisons:
//       drop the largest taken values / add the smallest untaken ones until
//       sum k = K and max(taken) < min(untaken).
// No floating-point value decides a unit: (1) is only a starting point and
// (2) is exact, so every rank computes the bit-identical plan.
#include <algorithm>
#include <cmath>
#include <new>
#include <vector>

#include "common.h"

struct mpress_plan_s {
  int world = 0;
  int source = 0;
  uint64_t G = 0, V = 0, K = 0;
  std::vector<uint64_t> sizes, offsets, units, peer_bytes;
  std::vector<mpress_stripe> stripes;
};

namespace mpress {
namespace {

using u128 = unsigned __int128;

// Is unit value (j1 / b1, p1) lexicographically smaller than (j2 / b2, p2)?
inline bool unit_less(uint64_t j1, uint64_t b1, int p1, uint64_t j2, uint64_t b2, int p2) {
  u128 l = (u128)j1 * b2, r = (u128)j2 * b1;
  if (l != r) return l < r;
  return p1 < p2;
}

struct Peer {
  int p;
  uint64_t cap, bw, k;
};

// Step (1): continuous water-fill starting point.
void water_fill(std::vector<Peer>& peers, uint64_t K) {
  // Saturation point of peer p: lambda_p = cap_p / B_p.
  std::vector<size_t> order(peers.size());
  for (size_t i = 0; i < order.size(); ++i) order[i] = i;
  std::sort(order.begin(), order.end(), [&](size_t a, size_t b) {
    return (long double)peers[a].cap / peers[a].bw < (long double)peers[b].cap / peers[b].bw;
  });
  long double saturated = 0, free_bw = 0;
  for (auto& q : peers) free_bw += (long double)q.bw;
  long double lambda = 0;
  size_t i = 0;
  for (; i < order.size(); ++i) {
    const Peer& q = peers[order[i]];
    long double t = (long double)q.cap / q.bw;
    long double total_at_t = saturated + t * free_bw;
    if (total_at_t >= (long double)K) break;
    saturated += (long double)q.cap;
    free_bw -= (long double)q.bw;
  }
  if (i == order.size() || free_bw <= 0) {
    lambda = INFINITY;
  } else {
    lambda = ((long double)K - saturated) / free_bw;
  }
  for (auto& q : peers) {
    long double x = lambda * (long double)q.bw;
    if (!(x < (long double)q.cap)) {
      q.k = q.cap;
    } else {
      q.k = x <= 0 ? 0 : (uint64_t)floorl(x);
      if (q.k > q.cap) q.k = q.cap;
    }
  }
}

// Step (2): exact fix-up to the K smallest unit values.
void exact_fixup(std::vector<Peer>& peers, uint64_t K) {
  u128 sum = 0;
  for (auto& q : peers) sum += q.k;
  auto max_taken = [&]() -> int {
    int best = -1;
    for (int i = 0; i < (int)peers.size(); ++i) {
      const Peer& q = peers[i];
      if (q.k == 0) continue;
      if (best < 0 || unit_less(peers[best].k, peers[best].bw, peers[best].p, q.k, q.bw, q.p)) best = i;
    }
    return best;
  };
  auto min_untaken = [&]() -> int {
    int best = -1;
    for (int i = 0; i < (int)peers.size(); ++i) {
      const Peer& q = peers[i];
      if (q.k >= q.cap) continue;
      if (best < 0 || unit_less(q.k + 1, q.bw, q.p, peers[best].k + 1, peers[best].bw, peers[best].p))
        best = i;
    }
    return best;
  };
  while (sum > K) {
    peers[max_taken()].k -= 1;
    sum -= 1;
  }
  while (sum < K) {
    peers[min_untaken()].k += 1;
    sum += 1;
  }
  for (;;) {
    int a = max_taken(), b = min_untaken();
    if (a < 0 || b < 0) break;
    const Peer& x = peers[a];
    const Peer& y = peers[b];
    // stop once every taken value precedes every untaken one
    if (unit_less(x.k, x.bw, x.p, y.k + 1, y.bw, y.p)) break;
    peers[a].k -= 1;
    peers[b].k += 1;
  }
}

int layout_batch(uint32_t n, const uint64_t* sizes, uint64_t G, mpress_plan_s* pl);
void build_layout(mpress_plan_s* pl);

int build_plan(int world, int source, const uint64_t* spare, const uint64_t* bw, uint32_t n,
               const uint64_t* sizes, uint64_t granule, mpress_plan_s* pl) {
  if (world < 1 || source < 0 || source >= world)
    return fail(MPRESS_ERR_ARG, "mpress_plan: source %d out of range [0,%d)", source, world);
  if (!spare || !bw || !sizes)
    return fail(MPRESS_ERR_ARG, "mpress_plan: null spare/link_bw/tensor_bytes");
  if (n == 0) return fail(MPRESS_ERR_ARG, "mpress_plan: empty tensor list");
  const uint64_t G = granule ? granule : MPRESS_DEFAULT_GRANULE;
  if (G % MPRESS_ALIGN != 0)
    return fail(MPRESS_ERR_ARG, "mpress_plan: granule %llu is not a multiple of 256",
                (unsigned long long)G);

  pl->world = world;
  pl->source = source;
  MP_TRY(layout_batch(n, sizes, G, pl));

  std::vector<Peer> peers;
  u128 capsum = 0;
  for (int p = 0; p < world; ++p) {
    if (p == source || bw[p] == 0) continue;
    uint64_t cap = spare[p] / G;
    if (cap == 0) continue;
    peers.push_back({p, cap, bw[p], 0});
    capsum += cap;
  }
  if (capsum < pl->K)
    return fail(MPRESS_ERR_NO_SPACE,
                "mpress_plan: %llu units of %llu B needed, peers hold %llu",
                (unsigned long long)pl->K, (unsigned long long)G, (unsigned long long)capsum);

  water_fill(peers, pl->K);
  exact_fixup(peers, pl->K);

  pl->units.assign(world, 0);
  for (auto& q : peers) pl->units[q.p] = q.k;
  build_layout(pl);
  return MPRESS_OK;
}

// Virtual layout of the batch (offsets, V, K) from the tensor sizes.
int layout_batch(uint32_t n, const uint64_t* sizes, uint64_t G, mpress_plan_s* pl) {
  pl->G = G;
  pl->sizes.assign(sizes, sizes + n);
  pl->offsets.resize(n);
  uint64_t V = 0;
  for (uint32_t i = 0; i < n; ++i) {
    if (sizes[i] == 0) return fail(MPRESS_ERR_ARG, "tensor %u has 0 bytes", i);
    pl->offsets[i] = V;
    uint64_t padded;
    if (sizes[i] > UINT64_MAX - (MPRESS_ALIGN - 1) || !add_ok(V, roundup(sizes[i], MPRESS_ALIGN), &padded))
      return fail(MPRESS_ERR_ARG, "batch size overflows 64 bits");
    V = padded;
  }
  pl->V = V;
  pl->K = V / G + (V % G != 0);
  return MPRESS_OK;
}

// Contiguous ranges per peer (ascending), intersected with the tensors by a
// single forward walk over the batch; pl->units must be set.
void build_layout(mpress_plan_s* pl) {
  const int world = pl->world;
  const uint64_t G = pl->G, V = pl->V;
  const uint32_t n = (uint32_t)pl->sizes.size();
  const uint64_t* sizes = pl->sizes.data();
  pl->stripes.clear();
  pl->peer_bytes.assign(world, 0);
  uint64_t a = 0;
  uint32_t i = 0;
  for (int p = 0; p < world; ++p) {
    const uint64_t k = pl->units[p];
    if (k == 0) continue;
    const uint64_t b = a + k * G;  // this peer's range [a, b) of the virtual batch
    pl->peer_bytes[p] = std::min(b, V) - a;
    while (i < n && pl->offsets[i] < b) {
      const uint64_t t0 = pl->offsets[i], t1 = t0 + sizes[i];
      const uint64_t lo = std::max(t0, a), hi = std::min(t1, b);
      if (hi > lo) pl->stripes.push_back({i, (uint32_t)p, lo - t0, lo - a, hi - lo});
      const uint64_t padded_end = t0 + roundup(sizes[i], MPRESS_ALIGN);
      if (padded_end <= b) ++i;
      else break;  // tensor i continues on the next peer
    }
    a = b;
  }
}

}  // namespace
}  // namespace mpress

using namespace mpress;

extern "C" int mpress_plan(int world, int source, const uint64_t* spare_bytes,
                           const uint64_t* link_bw, uint32_t n_tensors,
                           const uint64_t* tensor_bytes, uint64_t granule,
                           mpress_plan_t** out) {
  if (!out) return fail(MPRESS_ERR_ARG, "mpress_plan: out is null");
  *out = nullptr;
  auto* pl = new (std::nothrow) mpress_plan_s();
  if (!pl) return fail(MPRESS_ERR_ARG, "mpress_plan: out of host memory");
  int rc;
  try {
    rc = build_plan(world, source, spare_bytes, link_bw, n_tensors, tensor_bytes, granule, pl);
  } catch (const std::bad_alloc&) {
    rc = fail(MPRESS_ERR_ARG, "mpress_plan: out of host memory");
  }
  if (rc != MPRESS_OK) {
    delete pl;
    return rc;
  }
  *out = pl;
  return MPRESS_OK;
}

extern "C" int mpress_plan_stripes(const mpress_plan_t* plan, const mpress_stripe** stripes,
                                   uint32_t* n_stripes, const uint64_t** peer_bytes) {
  if (!plan) return fail(MPRESS_ERR_ARG, "mpress_plan_stripes: null plan");
  if (stripes) *stripes = plan->stripes.data();
  if (n_stripes) *n_stripes = (uint32_t)plan->stripes.size();
  if (peer_bytes) *peer_bytes = plan->peer_bytes.data();
  return MPRESS_OK;
}

extern "C" int mpress_plan_units(const mpress_plan_t* plan, const uint64_t** units) {
  if (!plan || !units) return fail(MPRESS_ERR_ARG, "mpress_plan_units: null argument");
  *units = plan->units.data();
  return MPRESS_OK;
}

extern "C" int mpress_plan_get_info(const mpress_plan_t* plan, mpress_plan_info* info) {
  if (!plan || !info) return fail(MPRESS_ERR_ARG, "mpress_plan_get_info: null argument");
  info->world = plan->world;
  info->source = plan->source;
  info->n_tensors = (uint32_t)plan->sizes.size();
  info->n_stripes = (uint32_t)plan->stripes.size();
  info->granule = plan->G;
  info->virtual_bytes = plan->V;
  info->units = plan->K;
  return MPRESS_OK;
}

extern "C" void mpress_plan_free(mpress_plan_t* plan) { delete plan; }

extern "C" int mpress_plan_from_units(int world, int source, const uint64_t* units, uint32_t n_tensors,
                                      const uint64_t* tensor_bytes, uint64_t granule, mpress_plan_t** out) {
  if (!out) return fail(MPRESS_ERR_ARG, "mpress_plan_from_units: out is null");
  *out = nullptr;
  if (world < 1 || source < 0 || source >= world || !units || !tensor_bytes || n_tensors == 0)
    return fail(MPRESS_ERR_ARG, "mpress_plan_from_units: bad argument");
  const uint64_t G = granule ? granule : MPRESS_DEFAULT_GRANULE;
  if (G % MPRESS_ALIGN != 0) return fail(MPRESS_ERR_ARG, "mpress_plan_from_units: granule not a multiple of 256");
  auto* pl = new (std::nothrow) mpress_plan_s();
  if (!pl) return fail(MPRESS_ERR_ARG, "mpress_plan_from_units: out of host memory");
  pl->world = world;
  pl->source = source;
  int rc = layout_batch(n_tensors, tensor_bytes, G, pl);
  u128 sum = 0;
  for (int p = 0; p < world && rc == MPRESS_OK; ++p) sum += units[p];
  if (rc == MPRESS_OK && units[source] != 0)
    rc = fail(MPRESS_ERR_ARG, "mpress_plan_from_units: units on the source itself");
  if (rc == MPRESS_OK && sum != pl->K)
    rc = fail(MPRESS_ERR_ARG, "mpress_plan_from_units: units sum to %llu, the batch has %llu",
              (unsigned long long)sum, (unsigned long long)pl->K);
  if (rc != MPRESS_OK) {
    delete pl;
    return rc;
  }
  pl->units.assign(units, units + world);
  build_layout(pl);
  *out = pl;
  return MPRESS_OK;
}

extern "C" int mpress_partition_sequential(int world, const uint64_t* spare_bytes,
                                           const uint64_t* bw_matrix, uint32_t n_sources,
                                           const int32_t* sources, const uint32_t* n_tensors,
                                           const uint64_t* sizes_flat, const uint32_t* copies,
                                           uint64_t granule, uint64_t* partition) {
  if (world < 1 || !spare_bytes || !bw_matrix || !partition || (n_sources && (!sources || !n_tensors || !sizes_flat || !copies)))
    return fail(MPRESS_ERR_ARG, "mpress_partition_sequential: null argument");
  std::vector<uint64_t> remaining(spare_bytes, spare_bytes + world);
  std::fill(partition, partition + (size_t)world * world, 0);
  // Offsets of each request's sizes inside sizes_flat, then ascending source order.
  std::vector<size_t> first(n_sources + 1, 0);
  for (uint32_t r = 0; r < n_sources; ++r) first[r + 1] = first[r] + n_tensors[r];
  std::vector<uint32_t> order(n_sources);
  for (uint32_t r = 0; r < n_sources; ++r) order[r] = r;
  std::stable_sort(order.begin(), order.end(),
                   [&](uint32_t a, uint32_t b) { return sources[a] < sources[b]; });
  for (uint32_t x = 0; x < n_sources; ++x) {
    if (x > 0 && sources[order[x]] == sources[order[x - 1]])
      return fail(MPRESS_ERR_ARG, "mpress_partition_sequential: source %d listed twice", sources[order[x]]);
  }
  std::vector<uint64_t> per_copy(world);
  for (uint32_t x = 0; x < n_sources; ++x) {
    const uint32_t r = order[x];
    const int s = sources[r];
    if (s < 0 || s >= world || copies[r] == 0)
      return fail(MPRESS_ERR_ARG, "mpress_partition_sequential: bad source %d / copies %u", s, copies[r]);
    for (int p = 0; p < world; ++p) per_copy[p] = remaining[p] / copies[r];
    mpress_plan_s pl;
    MP_TRY(build_plan(world, s, per_copy.data(), bw_matrix + (size_t)s * world, n_tensors[r],
                      sizes_flat + first[r], granule, &pl));
    for (int p = 0; p < world; ++p) {
      const uint64_t take = (uint64_t)copies[r] * pl.units[p] * pl.G;
      remaining[p] -= take;
      partition[(size_t)s * world + p] += take;
    }
  }
  return MPRESS_OK;
}
