// sm_100a swap kernels: the byte movers of swap-out and swap-in
// (P:121).
//
// The D2D swap moves bytes and computes nothing (tensor cores unused), so the
// kernels are shaped by the memory system alone:
//   * one launch per plan (the whole batch, "we also batch tensors"),
//     descriptors passed as a __grid_constant__ parameter (no upload);
//   * the descriptors are grouped by peer (the plan's stripes are sorted by
//     peer) and the chunks of the groups are interleaved by a weighted round
//     robin (round r takes chunk floor(r*n_g/R) of group g, R = the largest
//     group's chunk count rounded up to a power of two, so the division is a
//     shift), so at every moment each peer link carries its proportional
//     share of the swap -- the paper's "transmit them in parallel through
//     disjoint links" with sub-blocks sized to the links.
//     With several sources swapping at once (config 5, or every rank of the
//     N-GPU bench) each peer's NVLink ingress is then shared by all sources
//     all the time instead of every source converging on its first peer;
//   * the CTAs share that interleaved sequence by MPRESS_OPT_SPLIT: a
//     contiguous block each, a grid stride, or blocks claimed from a
//     per-launch counter so all CTAs work on one moving front of it (AUTO:
//     the stride for short launches, the claims for long TMA launches --
//     see Cursor and DynClaim below);
//   * the grid is capped (MPRESS_OPT_MAX_CTAS) so a concurrent GEMM keeps
//     most SMs;
//   * every address is 16-B aligned (tensor pointers are checked; stripe
//     offsets are multiples of 256, R6), so bodies move int4 / bulk pieces and
//     only the last <16 bytes of a tensor take a byte loop.
//
// PATH_DIRECT: THREADS threads, each issuing UNROLL independent 16- or 32-B
//   loads before its UNROLL stores, L1 bypassed on both sides.  Peer addresses
//   route over NVLink by their VA; loads of peer memory bypass the local L2
//   (B300_MICROARCH.md "NVLink"), so the depth of outstanding loads sets
//   swap-in bandwidth (Little's law).
// PATH_BULK: one warp per CTA drives the SM's bulk-async copy engine
//   (cp.async.bulk, SASS UBLKCP): chunk loads land in a ring of shared-memory
//   slots (mbarrier completion), then bulk stores drain them, so one SM keeps
//   STAGES x piece bytes in flight with a single issuing thread.
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstddef>
#include <cstdlib>
#include <type_traits>
#include <mutex>
#include <set>
#include <utility>
#include <vector>

#include "common.h"
#include "hostprof.h"
#include "swap_kernels.h"

namespace mpress {
namespace {

constexpr int kMaxGroups = 64;  // peers per launch (NVSwitch domains up to 64 GPUs)

// Descriptor tables come in five capacities (16, 32, 64, 128, 1024) so a
// small swap does not ship a 28 KB parameter block with its launch: the
// host cost of cudaLaunchKernelEx grows ~0.75 us per KB of parameters
// (16 -> 17 stripes, i.e. a 0.6 KB -> 4.1 KB table: +2.65 us per launch,
// tools/hostcost.py).
template <int CAP>
struct CopyTable {
  // every group holds >= 1 descriptor, so a table needs <= CAP groups
  static constexpr int kGroups = CAP < kMaxGroups ? CAP : kMaxGroups;
  uint32_t n;                        // descriptors
  uint32_t n_groups;                 // runs of descriptors with the same peer
  uint32_t rounds_log2;              // R = 2^rounds_log2 >= chunks of the largest group
  uint32_t pace_ns;                  // 0, or ns between the starts of one CTA's chunks (rate pacing)
  uint32_t split;                    // kSplitBlocked / kSplitStrided: positions -> CTAs (Cursor)
  uint32_t qlim;                     // MPRESS_SPLIT_DYNAMIC: smallest | largest claim << 16 (positions)
  unsigned long long* dyn;           // MPRESS_SPLIT_DYNAMIC: {claimed, CTAs done} (CounterRing slot), else null
  uint32_t g_chunk[kGroups + 1];     // first chunk of each group (prefix)
  uint32_t g_desc[kGroups + 1];      // first descriptor of each group (prefix)
  uint32_t first_chunk[CAP + 1];     // first chunk of each descriptor (prefix)
  CopyDesc d[CAP];
};
static_assert(sizeof(CopyTable<kMaxDescPerLaunch>) <= 32764, "kernel parameter space is 32764 bytes");

// largest i in [0, n) with a[i] <= x  (a[0] == 0 <= x)
__device__ __forceinline__ uint32_t upper_idx(const uint32_t* a, uint32_t n, uint32_t x) {
  uint32_t lo = 0, hi = n;
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (a[mid] <= x) lo = mid; else hi = mid;
  }
  return lo;
}

// The interleaved sequence has R rounds of n_groups positions; position
// (r, g) holds chunk k = floor(r * n_g / R) of group g.  k is non-decreasing
// in r with steps of 0 or 1 and reaches n_g - 1 by r = R - 1, so taking only
// the first round that reaches each k visits every chunk exactly once; the
// other positions are skipped.
//
// Which CTA takes which positions (CopyTable::split):
//   kSplitBlocked (default): CTA b walks the contiguous block of positions
//     [b*P/grid, (b+1)*P/grid), P = R * n_groups.  Every group's valid
//     positions are spread evenly over the sequence, so every block holds
//     total/grid +- n_groups chunks, and inside a block the CTA still visits
//     the peers in proportion.
//   kSplitStrided (round 1): CTA b walks positions b, b + grid, ...  The
//     skip pattern aliases with the stride, so CTAs got up to 1.7x the mean
//     chunk count (cfg2 micro-batch, 128 CTAs of 32 KiB chunks: 0 .. 384
//     chunks, mean 225) -- a tail, and a rate-paced launch ran at mean/max of
//     its rate.
// (r, g) is advanced incrementally (no division per step).
enum : uint32_t { kSplitBlocked = 0, kSplitStrided = 1 };

template <int CAP>
struct Cursor {
  const CopyTable<CAP>& t;
  uint32_t g, gm, gd;
  uint64_t r;
  uint64_t left;  // positions this cursor still visits
  // This CTA's positions under the table's split (one cursor per CTA).
  __device__ explicit Cursor(const CopyTable<CAP>& tt) : t(tt) {
    uint64_t start, stride, end;
    span(tt, 0, 1, &start, &stride, &end);
    init(start, stride, end);
  }
  // Lane `lane` of `lanes` cursors sharing this CTA's positions (the bulk
  // kernel's 32 resolver lanes): every lanes-th position of the CTA's share.
  __device__ Cursor(const CopyTable<CAP>& tt, uint32_t lane, uint32_t lanes) : t(tt) {
    uint64_t start, stride, end;
    span(tt, lane, lanes, &start, &stride, &end);
    init(start, stride, end);
  }
  __device__ static void span(const CopyTable<CAP>& tt, uint32_t lane, uint32_t lanes, uint64_t* start,
                              uint64_t* stride, uint64_t* end) {
    const uint64_t P = (uint64_t)tt.n_groups << tt.rounds_log2;
    if (tt.split == kSplitStrided) {
      *start = blockIdx.x + (uint64_t)lane * gridDim.x;
      *stride = (uint64_t)lanes * gridDim.x;
      *end = P;
    } else {
      const uint64_t b0 = (uint64_t)(((unsigned __int128)P * blockIdx.x) / gridDim.x);
      const uint64_t b1 = (uint64_t)(((unsigned __int128)P * (blockIdx.x + 1)) / gridDim.x);
      *start = b0 + lane;
      *stride = lanes;
      *end = b1;
    }
  }
  __device__ void init(uint64_t start, uint64_t stride, uint64_t end) {
    g = (uint32_t)(start % t.n_groups);
    r = start / t.n_groups;
    gm = (uint32_t)(stride % t.n_groups);
    gd = (uint32_t)(stride / t.n_groups);
    left = start < end ? (end - start + stride - 1) / stride : 0;
  }
  // Next chunk of this cursor: its index *c and its descriptor *s.
  __device__ bool next(uint32_t* c, uint32_t* s) {
    while (left) {
      --left;
      const uint32_t gg = g;
      const uint64_t rr = r;
      g += gm;
      r += gd;
      if (g >= t.n_groups) { g -= t.n_groups; ++r; }
      const uint64_t gc = t.g_chunk[gg + 1] - t.g_chunk[gg];
      const uint64_t k = (rr * gc) >> t.rounds_log2;
      if (rr > 0 && (((rr - 1) * gc) >> t.rounds_log2) == k) continue;
      *c = t.g_chunk[gg] + (uint32_t)k;
      // descriptor: search only inside the group's descriptors
      const uint32_t d0 = t.g_desc[gg];
      *s = d0 + upper_idx(t.first_chunk + d0, t.g_desc[gg + 1] - d0, *c);
      return true;
    }
    return false;
  }
};

// MPRESS_SPLIT_DYNAMIC: a CTA claims blocks [s, s + q) of the launch's
// positions from a counter (atomicAdd), claiming the next block while it
// moves the current one so the atomic's latency hides behind the copies.
// Guided self-scheduling: q = remaining / (2 x grid), clamped to [qmin,
// QMAX], so the last blocks are a few chunks and SMs that run faster take
// more.  Besides removing the tail, this keeps every CTA inside one moving
// window of the sequence (all CTAs claim from the same front) instead of
// 148 separate regions -- fewer pages touched at once.  Every CTA counts
// itself done once its claims ran past the end; the last one resets the
// slot for the next launch that takes it (kernel completion orders that
// reset before any later launch, PDL included: griddepcontrol.wait waits for
// completion and flush).
template <uint32_t QMAX>
struct DynClaim {
  unsigned long long* ctr;
  uint64_t P;
  uint32_t qmin;
  uint64_t next_s = 0;   // the prefetched claim (claiming thread)
  uint32_t next_q = 0;
  uint32_t qmax;
  uint64_t workers;      // claimants in the launch: CTAs, or warps of a two-warp CTA
  __device__ DynClaim(unsigned long long* c, uint64_t p, uint32_t qlim, uint64_t w = 0)
      : ctr(c), P(p), workers(w ? w : gridDim.x) {
    qmax = qlim >> 16;
    qmax = qmax == 0 || qmax > QMAX ? QMAX : qmax;
    qmin = qlim & 0xFFFFu;
    qmin = qmin == 0 ? 1 : qmin > qmax ? qmax : qmin;
  }
  __device__ void claim(uint64_t seen) {
    const uint64_t rem = seen < P ? P - seen : 0;
    const uint64_t q = rem / (2ull * workers);
    next_q = q < qmin ? qmin : q > qmax ? qmax : (uint32_t)q;
    next_s = atomicAdd(ctr, (unsigned long long)next_q);
  }
  __device__ void done() {
    __threadfence();
    if (atomicAdd(ctr + 1, 1ull) == workers - 1ull) {
      atomicExch(ctr, 0ull);
      atomicExch(ctr + 1, 0ull);
    }
  }
};

__device__ __forceinline__ int4 ld_stream(const int4* p) {
  int4 r;
  asm volatile("ld.global.nc.L1::no_allocate.v4.s32 {%0,%1,%2,%3}, [%4];"
               : "=r"(r.x), "=r"(r.y), "=r"(r.z), "=r"(r.w) : "l"(p));
  return r;
}

__device__ __forceinline__ void st_stream(int4* p, const int4& v) {
  asm volatile("st.global.L1::no_allocate.v4.s32 [%0], {%1,%2,%3,%4};"
               :: "l"(p), "r"(v.x), "r"(v.y), "r"(v.z), "r"(v.w) : "memory");
}

// sm_100 moves 32 bytes per thread per instruction (SASS LDG/STG .256), which
// halves the load/store instructions of a chunk; the L2 eviction-priority
// qualifiers exist only at this width.
struct alignas(32) V8 {
  uint32_t v[8];
};

template <bool EVICT_FIRST>
__device__ __forceinline__ V8 ld_stream(const V8* p) {
  V8 r;
  if (EVICT_FIRST)
    asm volatile("ld.global.nc.L1::no_allocate.L2::evict_first.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]),
                   "=r"(r.v[6]), "=r"(r.v[7]) : "l"(p));
  else
    asm volatile("ld.global.nc.L1::no_allocate.v8.b32 {%0,%1,%2,%3,%4,%5,%6,%7}, [%8];"
                 : "=r"(r.v[0]), "=r"(r.v[1]), "=r"(r.v[2]), "=r"(r.v[3]), "=r"(r.v[4]), "=r"(r.v[5]),
                   "=r"(r.v[6]), "=r"(r.v[7]) : "l"(p));
  return r;
}

__device__ __forceinline__ void st_stream(V8* p, const V8& r) {
  asm volatile("st.global.L1::no_allocate.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8};"
               :: "l"(p), "r"(r.v[0]), "r"(r.v[1]), "r"(r.v[2]), "r"(r.v[3]), "r"(r.v[4]), "r"(r.v[5]),
                  "r"(r.v[6]), "r"(r.v[7]) : "memory");
}

// 32-byte store whose L2 lines are marked evict-first (a createpolicy cache
// hint: st has no L2 eviction-priority qualifier), so a swap streaming
// through L2 beside a GEMM does not push the GEMM's tiles out.
__device__ __forceinline__ void st_stream_ef(V8* p, const V8& r, uint64_t pol) {
  asm volatile("st.global.L1::no_allocate.L2::cache_hint.v8.b32 [%0], {%1,%2,%3,%4,%5,%6,%7,%8}, %9;"
               :: "l"(p), "r"(r.v[0]), "r"(r.v[1]), "r"(r.v[2]), "r"(r.v[3]), "r"(r.v[4]), "r"(r.v[5]),
                  "r"(r.v[6]), "r"(r.v[7]), "l"(pol) : "memory");
}

// One vector load / store of width VB (16 or 32 bytes); HINT (32 only) = L2
// evict-first on the loads and on the stores.
template <int VB, bool HINT>
struct Vec;
template <bool HINT>
struct Vec<16, HINT> {
  using T = int4;
  static __device__ __forceinline__ T ld(const T* p) { return ld_stream(p); }
  static __device__ __forceinline__ void st(T* p, const T& v, uint64_t) { st_stream(p, v); }
};
template <bool HINT>
struct Vec<32, HINT> {
  using T = V8;
  static __device__ __forceinline__ T ld(const T* p) { return ld_stream<HINT>(p); }
  static __device__ __forceinline__ void st(T* p, const T& v, uint64_t pol) {
    if (HINT) st_stream_ef(p, v, pol);
    else st_stream(p, v);
  }
};

// Programmatic dependent launch (PDL): a swap kernel is launched with
// programmatic stream serialization, so it may start while the previous
// kernel of its stream is still draining.  It first waits for that grid to
// complete and flush (griddepcontrol.wait: a no-op without a programmatic
// predecessor), then lets its own successor launch early.  Only launch
// latency and CTA ramp-up overlap, never data: ordering stays exact for any
// predecessor (a producing GEMM, the matching swap-out, a user kernel).
__device__ __forceinline__ void pdl_enter() {
  asm volatile("griddepcontrol.wait;" ::: "memory");
  asm volatile("griddepcontrol.launch_dependents;" ::: "memory");
}

// Rate pacing (MPRESS_OPT_PACE_MBPS): chunk i of a CTA may start no earlier
// than t0 + i * pace_ns (%globaltimer, ns), so the launch moves at most the
// requested rate however fast the links are.  A swap only has to finish
// within its tensor's live interval; moving it faster than that only
// takes HBM, L2 and issue slots from the compute it runs beside.  The
// schedule is absolute, so timer granularity and sleep overshoot do not
// accumulate.
struct Pacer {
  uint64_t t0 = 0, next = 0;
  uint32_t step;
  __device__ explicit Pacer(uint32_t pace_ns) : step(pace_ns) {
    if (step) {
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t0));
      next = t0;
    }
  }
  __device__ __forceinline__ void wait() {
    if (!step) return;
    for (;;) {
      uint64_t now;
      asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(now));
      if (now >= next) break;
      const uint64_t d = next - now;
      __nanosleep(d > 100000 ? 100000u : (unsigned)d);
    }
    next += step;
  }
};

// ---------------------------------------------------------------- direct path

struct Span {
  const uint8_t* src;
  uint8_t* dst;
  uint64_t rem;  // bytes of the descriptor from this chunk on
};

template <uint32_t SHIFT, int CAP>
__device__ __forceinline__ Span span_of(const CopyTable<CAP>& t, uint32_t c, uint32_t s) {
  const CopyDesc& d = t.d[s];
  const uint64_t off = (uint64_t)(c - t.first_chunk[s]) << SHIFT;
  return Span{static_cast<const uint8_t*>(d.src) + off, static_cast<uint8_t*>(d.dst) + off, d.len - off};
}
// THREADS threads each keep UNROLL independent VB-byte loads in flight, then
// store them: one chunk = THREADS*UNROLL*VB bytes per CTA iteration.  VB = 32
// needs 32-byte aligned descriptors (checked on the host, else VB = 16).
// DIR only names the instantiation (swap-out vs swap-in in profiles): the
// byte movement is the same, the descriptors say which side is the peer.
template <int DIR, int THREADS, int UNROLL, int VB, bool HINT, bool PF, int CAP>
__device__ __forceinline__ void direct_body(const CopyTable<CAP>& t) {
  using VT = typename Vec<VB, HINT>::T;
  constexpr uint32_t kChunk = THREADS * UNROLL * VB;
  static_assert((kChunk & (kChunk - 1)) == 0, "chunk must be a power of two");
  constexpr uint32_t kShift = __builtin_ctz(kChunk);
  // PF: the next chunk's address is resolved while the current chunk's loads
  // are in flight, so the table lookups (constant-bank reads) stay off the
  // critical path of a latency-bound CTA (<= 1 CTA per SM: +50% at 32 CTAs).
  // With >= 2 CTAs per SM the memory system is saturated anyway and issuing
  // the stores first measured ~6% faster (tools/ab.py), so PF is off there.
  pdl_enter();
  Cursor<CAP> cur(t);
  // MPRESS_SPLIT_DYNAMIC: thread 0 claims blocks of <= 16 positions for the
  // CTA and hands them over through shared memory; every thread's cursor
  // walks the same block, so they all run out -- and refill -- together.
  const bool dyn = t.dyn != nullptr;
  const uint64_t P = (uint64_t)t.n_groups << t.rounds_log2;
  DynClaim<16> dc(t.dyn, P, t.qlim);
  __shared__ uint64_t claim_s;
  __shared__ uint32_t claim_q;
  if (dyn) {
    cur.init(0, 1, 0);
    if (threadIdx.x == 0) dc.claim(0);
  }
  auto next = [&](uint32_t* cc, uint32_t* ss) -> bool {
    while (!cur.next(cc, ss)) {
      if (!dyn) return false;
      __syncthreads();  // every thread has read the previous block
      if (threadIdx.x == 0) {
        claim_s = dc.next_s;
        claim_q = dc.next_q;
        if (dc.next_s < P) dc.claim(dc.next_s + dc.next_q);
      }
      __syncthreads();
      const uint64_t b = claim_s;
      if (b >= P) return false;
      cur.init(b, 1, b + claim_q < P ? b + claim_q : P);
    }
    return true;
  };
  uint32_t c, s;
  if (!next(&c, &s)) {
    if (dyn && threadIdx.x == 0) dc.done();
    return;
  }
  Span sp = span_of<kShift>(t, c, s);
  Pacer pace(t.pace_ns);
  uint64_t pol = 0;
  if (HINT && VB == 32) asm volatile("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(pol));
  for (;;) {
    Span nx{nullptr, nullptr, 0};
    bool more = false;
    pace.wait();
    if (sp.rem >= kChunk) {
      const VT* sv = reinterpret_cast<const VT*>(sp.src) + threadIdx.x;
      VT* dv = reinterpret_cast<VT*>(sp.dst) + threadIdx.x;
      VT r[UNROLL];
#pragma unroll
      for (int j = 0; j < UNROLL; ++j) r[j] = Vec<VB, HINT>::ld(sv + j * THREADS);
      if (PF) {
        more = next(&c, &s);
        if (more) nx = span_of<kShift>(t, c, s);
      }
#pragma unroll
      for (int j = 0; j < UNROLL; ++j) Vec<VB, HINT>::st(dv + j * THREADS, r[j], pol);
      if (!PF) {
        more = next(&c, &s);
        if (more) nx = span_of<kShift>(t, c, s);
      }
    } else {
      // ragged last chunk of a stripe: 16-B body, then the <16-byte tail
      const uint32_t len = (uint32_t)sp.rem;
      const uint32_t n16 = len >> 4;
      const int4* sv = reinterpret_cast<const int4*>(sp.src);
      int4* dv = reinterpret_cast<int4*>(sp.dst);
      for (uint32_t x = threadIdx.x; x < n16; x += THREADS) st_stream(dv + x, ld_stream(sv + x));
      const uint32_t tail = len & 15u;
      if (threadIdx.x < tail) sp.dst[(n16 << 4) + threadIdx.x] = sp.src[(n16 << 4) + threadIdx.x];
      more = next(&c, &s);
      if (more) nx = span_of<kShift>(t, c, s);
    }
    if (!more) break;
    sp = nx;
  }
  if (dyn && threadIdx.x == 0) dc.done();
}

// The table as a kernel parameter (constant bank) ...
template <int DIR, int THREADS, int UNROLL, int VB, bool HINT, bool PF, int CAP>
__global__ void __launch_bounds__(THREADS)
mp_swap_direct(const __grid_constant__ CopyTable<CAP> t) {
  direct_body<DIR, THREADS, UNROLL, VB, HINT, PF, CAP>(t);
}

// ... or device-resident (TableRing, large tables), read through a pointer.
template <int DIR, int THREADS, int UNROLL, int VB, bool HINT, bool PF, int CAP>
__global__ void __launch_bounds__(THREADS)
mp_swap_direct_g(const CopyTable<CAP>* __restrict__ tp) {
  direct_body<DIR, THREADS, UNROLL, VB, HINT, PF, CAP>(*tp);
}

// ---------------------------------------------------------------- bulk path

__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return static_cast<uint32_t>(__cvta_generic_to_shared(p));
}

__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" :: "r"(smem_u32(bar)), "r"(count) : "memory");
}

__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;"
               :: "r"(smem_u32(bar)), "r"(bytes) : "memory");
}

// The wait loop is C++ around a predicate-returning try_wait (no branch
// inside inline asm), so the compiler sees the divergent loop and reconverges
// the warp before the shuffles that follow it.
__device__ __forceinline__ bool mbar_try(uint64_t* bar, uint32_t parity) {
  uint32_t ok;
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
      "selp.u32 %0, 1, 0, p;\n"
      "}\n" : "=r"(ok) : "r"(smem_u32(bar)), "r"(parity) : "memory");
  return ok != 0;
}

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  while (!mbar_try(bar, parity)) {
  }
}

__device__ __forceinline__ void bulk_load(void* smem, const void* gsrc, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];"
      :: "r"(smem_u32(smem)), "l"(gsrc), "r"(bytes), "r"(smem_u32(bar)) : "memory");
}

__device__ __forceinline__ void bulk_store(void* gdst, const void* smem, uint32_t bytes) {
  asm volatile("cp.async.bulk.global.shared::cta.bulk_group [%0], [%1], %2;"
               :: "l"(gdst), "r"(smem_u32(smem)), "r"(bytes) : "memory");
}

__device__ __forceinline__ void bulk_commit() { asm volatile("cp.async.bulk.commit_group;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read1() { asm volatile("cp.async.bulk.wait_group.read 1;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_read0() { asm volatile("cp.async.bulk.wait_group.read 0;" ::: "memory"); }
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

struct Piece {
  const uint8_t* src;
  uint8_t* dst;
  uint32_t bytes;  // multiple of 16
};

template <int SHIFT, int CAP>
__device__ __forceinline__ Piece bulk_piece(const CopyTable<CAP>& t, uint32_t c, uint32_t s) {
  const CopyDesc& d = t.d[s];
  const uint64_t off = (uint64_t)(c - t.first_chunk[s]) << SHIFT;
  const uint64_t rem = d.len - off;
  Piece p;
  p.src = static_cast<const uint8_t*>(d.src) + off;
  p.dst = static_cast<uint8_t*>(d.dst) + off;
  p.bytes = (uint32_t)(rem >= (1ull << SHIFT) ? (1ull << SHIFT) : (rem & ~15ull));
  return p;
}

// 64-bit warp shuffle.
__device__ __forceinline__ uint64_t shfl64(uint64_t v, int lane) {
  const uint32_t lo = __shfl_sync(0xffffffffu, (uint32_t)v, lane);
  const uint32_t hi = __shfl_sync(0xffffffffu, (uint32_t)(v >> 32), lane);
  return ((uint64_t)hi << 32) | lo;
}

// Bulk shape 9 (beside a GEMM): a second warp in the CTA copies pieces
// through registers (LDG/STG, 4 pieces x 2^SHIFT bytes in flight) while the
// first drives the TMA ring, both claiming their own blocks from the
// launch's counter -- twice the bytes in flight per SM inside the shared
// memory a GEMM CTA leaves.  Only with the dynamic claims; under a static
// split (small launches, graph capture) the TMA warp moves everything.
// Registers decide whether it co-resides with the GEMM at all: a cuBLAS
// CTA's 8 warps x 168 registers leave 5632 of each SM sub-partition's 16K,
// so a warp of this kernel must stay at <= 176 registers (it uses 168; a
// build at 180 lost co-residency and cost the GEMM +80%,
// profiles/r02/hybrid/pace_180regs_gemm.jsonl).  Not paced (pacing keeps
// CTAs resident while they sleep, which costs a GEMM more than it saves).
template <int SHIFT, int CAP>
__device__ __forceinline__ void bulk_lsu_warp(const CopyTable<CAP>& t, uint64_t workers) {
  constexpr uint32_t kVec = (1u << SHIFT) / 16u / 32u;  // 16-byte vectors per lane per piece
  constexpr int kPieces = 4;
  const uint32_t lane = threadIdx.x & 31u;
  if (!t.dyn) return;
  const uint64_t P = (uint64_t)t.n_groups << t.rounds_log2;
  DynClaim<32> dc(t.dyn, P, t.qlim, workers);
  if (lane == 0) dc.claim(0);
  Cursor<CAP> cur(t, lane, 32u);
  for (;;) {
    const uint64_t b = shfl64(dc.next_s, 0);
    const uint32_t q = __shfl_sync(0xffffffffu, dc.next_q, 0);
    if (b >= P) break;
    if (lane == 0) dc.claim(b + q);
    cur.init(b + lane, 32u, b + q < P ? b + q : P);   // q <= 32: one position per lane at most
    uint32_t c, sd;
    const bool v = cur.next(&c, &sd);
    Piece mine{nullptr, nullptr, 0};
    if (v) {
      mine = bulk_piece<SHIFT>(t, c, sd);
      if (c + 1 == t.first_chunk[sd + 1]) {  // last chunk of descriptor sd: its tail
        const CopyDesc& d = t.d[sd];
        for (uint64_t x = d.len & ~15ull; x < d.len; ++x)
          static_cast<uint8_t*>(d.dst)[x] = static_cast<const uint8_t*>(d.src)[x];
      }
    }
    __syncwarp();
    uint32_t mask = __ballot_sync(0xffffffffu, mine.bytes != 0);
    while (mask) {
      const int4* src[kPieces];
      int4* dst[kPieces];
      uint32_t nv[kPieces];
#pragma unroll
      for (int p = 0; p < kPieces; ++p) {
        const int j = mask ? __ffs(mask) - 1 : 0;
        const bool has = mask != 0;
        if (has) mask &= mask - 1;
        src[p] = reinterpret_cast<const int4*>(shfl64(reinterpret_cast<uint64_t>(mine.src), j));
        dst[p] = reinterpret_cast<int4*>(shfl64(reinterpret_cast<uint64_t>(mine.dst), j));
        const uint32_t nb = __shfl_sync(0xffffffffu, mine.bytes, j);
        nv[p] = has ? nb >> 4 : 0u;
      }
      int4 r[kPieces][kVec];
#pragma unroll
      for (int p = 0; p < kPieces; ++p)
#pragma unroll
        for (uint32_t k = 0; k < kVec; ++k)
          if (lane + 32u * k < nv[p]) r[p][k] = ld_stream(src[p] + lane + 32u * k);
#pragma unroll
      for (int p = 0; p < kPieces; ++p)
#pragma unroll
        for (uint32_t k = 0; k < kVec; ++k)
          if (lane + 32u * k < nv[p]) st_stream(dst[p] + lane + 32u * k, r[p][k]);
    }
  }
  if (lane == 0) dc.done();
}

// One warp per CTA: lane 0 streams pieces of 2^SHIFT bytes through STAGES
// shared-memory slots with the SM's bulk-copy engine (cp.async.bulk G->S with
// mbarrier completion, then S->G bulk stores).  The 32 lanes resolve the
// chunk sequence in parallel -- lane j walks every 32nd position of the
// CTA's share from the j-th on, with its own cursor -- and hand the pieces to lane 0
// by shuffles, so the descriptor lookups (dependent constant-bank loads) are
// off the issuing thread's critical path (profiles/r01: with one cursor on
// lane 0 they took ~75% of its issue samples).  Each lane also copies the
// <16-byte tail of a descriptor whose last chunk it resolved.  A ring in
// shared memory remembers each slot's destination for its store.  Order:
// piece k's load is issued once the store of piece k - STAGES has been read
// out of its slot.  Small pieces (<= 4 KiB, kEager): issue only that store
// and wait for its read (wait_group.read 0), so STAGES loads are in flight --
// 3 x 4 KiB went from 625 to 1141 GB/s at 148 CTAs.  Larger pieces: also
// store piece k-STAGES+1 and wait for all but the newest store's read
// (read 1), keeping a store in flight -- for 3 x 32 KiB waiting on the
// newest 32 KiB read cost 5% (profiles/r02/bulk_ring_ab.txt).
template <int DIR, int SHIFT, int STAGES, int CAP, int LSU>
__device__ __forceinline__ void bulk_body(const CopyTable<CAP>& t) {
  constexpr uint32_t kSlot = 1u << SHIFT;
  constexpr bool kEager = SHIFT <= 12;
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bars[STAGES];
  __shared__ uint8_t* ring_dst[STAGES];
  __shared__ uint32_t ring_bytes[STAGES];
  const uint32_t lane = threadIdx.x & 31u;
  const uint64_t workers = (uint64_t)gridDim.x * (1 + LSU);

  pdl_enter();
  if (LSU && threadIdx.x >= 32) {
    bulk_lsu_warp<SHIFT, CAP>(t, workers);
    return;
  }
  if (lane == 0) {
    for (int k = 0; k < STAGES; ++k) mbar_init(&bars[k], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
  }
  __syncwarp();

  uint32_t loaded = 0, stored = 0;  // pieces whose load / store was issued (lane 0)
  Pacer pace(lane == 0 ? t.pace_ns : 0u);
  // lane 0: issue the stores of pieces [stored, upto) in order
  auto store_until = [&](uint32_t upto) {
    for (; stored < upto; ++stored) {
      const uint32_t q = stored % STAGES;
      mbar_wait(&bars[q], (stored / STAGES) & 1u);
      if (ring_bytes[q]) bulk_store(ring_dst[q], smem + (size_t)q * kSlot, ring_bytes[q]);
      bulk_commit();
    }
  };

  Cursor<CAP> cur(t, lane, 32u);
  // MPRESS_SPLIT_DYNAMIC: lane 0 claims blocks of <= 32 positions, one per
  // resolver lane; a new block is taken when every lane's cursor is empty.
  const bool dyn = t.dyn != nullptr;
  const uint64_t P = (uint64_t)t.n_groups << t.rounds_log2;
  DynClaim<32> dc(t.dyn, P, t.qlim, workers);
  if (dyn) {
    cur.init(0, 1, 0);
    if (lane == 0) dc.claim(0);
  }
  for (;;) {
    uint32_t c, sd;
    const bool v = cur.next(&c, &sd);
    Piece mine{nullptr, nullptr, 0};
    if (v) {
      mine = bulk_piece<SHIFT>(t, c, sd);
      if (c + 1 == t.first_chunk[sd + 1]) {  // last chunk of descriptor sd: its tail
        const CopyDesc& d = t.d[sd];
        for (uint64_t b = d.len & ~15ull; b < d.len; ++b)
          static_cast<uint8_t*>(d.dst)[b] = static_cast<const uint8_t*>(d.src)[b];
      }
    }
    // Lanes leave their cursor loops after different trip counts: reconverge
    // explicitly before the ballot and the shuffles (without it the ballot was
    // compiled without a warp sync and saw only the lanes already done).
    __syncwarp();
    uint32_t mask = __ballot_sync(0xffffffffu, v);
    if (!mask) {
      if (!dyn) break;
      const uint64_t b = shfl64(dc.next_s, 0);
      const uint32_t q = __shfl_sync(0xffffffffu, dc.next_q, 0);
      if (b >= P) break;
      if (lane == 0) dc.claim(b + q);
      cur.init(b + lane, 32u, b + q < P ? b + q : P);
      continue;
    }
    while (mask) {
      const int j = __ffs(mask) - 1;
      mask &= mask - 1;
      const uint8_t* src = reinterpret_cast<const uint8_t*>(shfl64(reinterpret_cast<uint64_t>(mine.src), j));
      uint8_t* dst = reinterpret_cast<uint8_t*>(shfl64(reinterpret_cast<uint64_t>(mine.dst), j));
      const uint32_t bytes = __shfl_sync(0xffffffffu, mine.bytes, j);
      if (lane == 0) {
        const uint32_t k = loaded;
        if (k >= STAGES) {
          if (kEager) {
            // only the store of piece k-STAGES (the slot's previous piece),
            // then its smem read: STAGES loads stay in flight
            store_until(k - STAGES + 1);
            bulk_wait_read0();
          } else {
            // also store piece k-STAGES+1 and wait only for all but the
            // newest store's read: one store stays in flight behind it
            store_until(k - STAGES + 2 <= k ? k - STAGES + 2 : k);  // stores through piece k-STAGES+1
            bulk_wait_read1();  // all but the newest store have left smem: slot of k-STAGES is free
          }
        }
        pace.wait();
        const uint32_t q = k % STAGES;
        ring_dst[q] = dst;
        ring_bytes[q] = bytes;
        mbar_expect_tx(&bars[q], bytes);
        if (bytes) bulk_load(smem + (size_t)q * kSlot, src, bytes, &bars[q]);
        ++loaded;
      }
      __syncwarp();
    }
  }
  if (lane == 0) {
    store_until(loaded);
    bulk_wait_all();
    if (dyn) dc.done();
  }
}

// (LSU: at least 6 CTAs' worth of registers per SM = <= 168 registers per
// thread, the co-residency bound with a GEMM CTA -- see bulk_lsu_warp)
template <int DIR, int SHIFT, int STAGES, int CAP, int LSU>
__global__ void __launch_bounds__(32 * (1 + LSU), LSU ? 6 : 1)
mp_swap_bulk(const __grid_constant__ CopyTable<CAP> t) {
  bulk_body<DIR, SHIFT, STAGES, CAP, LSU>(t);
}

template <int DIR, int SHIFT, int STAGES, int CAP, int LSU>
__global__ void __launch_bounds__(32 * (1 + LSU), LSU ? 6 : 1)
mp_swap_bulk_g(const CopyTable<CAP>* __restrict__ tp) {
  bulk_body<DIR, SHIFT, STAGES, CAP, LSU>(*tp);
}

// ---------------------------------------------------------------- variants

struct Shape {
  int threads;
  uint32_t shift;   // log2 bytes per chunk / bulk piece
  size_t smem;      // dynamic shared memory
  int per_sm;       // default CTAs per SM when MPRESS_OPT_MAX_CTAS = 0
  int vb;           // vector bytes per thread access (direct path)
  int fallback;     // variant used when a 32-byte variant meets 16-byte-aligned data
};

// direct (threads, unroll, vector bytes): 0 (256,8,16) 1 (512,8,16)
// 2 (256,16,16) 3 (1024,4,16) 4 (128,8,16) 5 (256,4,32) 6 (256,8,32)
// 7 (128,4,32) 8 (256,4,32 + L2 evict-first loads) 9 (128,8,32)
// 10 (128,16,32) 11 (64,16,32) -- 32 / 64 KiB in flight per CTA with few
// warps, for a capped grid beside a GEMM (its CTA leaves ~22.5K registers)
// 12 (128,8,32 + L2 evict-first loads and stores) 13 (32,16,32: one warp,
// 16 KiB in flight -- the direct twin of the one-warp bulk shapes)
// bulk (piece, stages, CTAs/SM): 0 (32K,6,1) 1 (16K,12,1) 2 (64K,3,1) 3 (32K,3,1)
// 4 (16K,4,3) 5 (8K,2,1) 6 (4K,3,1) 7 (4K,4,1) 8 (2K,8,1) 9 (4K,4,1 plus an
// LSU warp with 4 x 4 KiB in registers, dynamic claims only) -- 5-9 use 16 /
// 12 / 16 / 16 / 16 KB of shared memory, small enough to sit beside a cuBLAS
// GEMM CTA (214 KB of the SM's 233.5 KB)
constexpr Shape kDirect[kDirectVariants] = {
    {256, 15, 0, 2, 16, 0}, {512, 16, 0, 1, 16, 1}, {256, 16, 0, 2, 16, 2}, {1024, 16, 0, 1, 16, 3},
    {128, 14, 0, 4, 16, 4}, {256, 15, 0, 2, 32, 0}, {256, 16, 0, 2, 32, 2}, {128, 14, 0, 4, 32, 4},
    {256, 15, 0, 2, 32, 0}, {128, 15, 0, 4, 32, 4}, {128, 16, 0, 4, 32, 4}, {64, 15, 0, 8, 32, 4},
    {128, 15, 0, 4, 32, 4}, {32, 14, 0, 8, 32, 4}};
constexpr Shape kBulk[kBulkVariants] = {
    {32, 15, 6u << 15, 1, 16, 0}, {32, 14, 12u << 14, 1, 16, 1}, {32, 16, 3u << 16, 1, 16, 2},
    {32, 15, 3u << 15, 1, 16, 3}, {32, 14, 4u << 14, 3, 16, 4}, {32, 13, 2u << 13, 1, 16, 5},
    {32, 12, 3u << 12, 1, 16, 6}, {32, 12, 4u << 12, 1, 16, 7}, {32, 11, 8u << 11, 1, 16, 8},
    {64, 12, 4u << 12, 1, 16, 9}};

template <int CAP>
using KernelFn = void (*)(CopyTable<CAP>);
template <int CAP>
using KernelFnG = void (*)(const CopyTable<CAP>*);

// Entry point of one instantiation; `if constexpr` keeps the pointer-table
// (G) kernels from being instantiated for the capacities that never use them.
template <int CAP, bool G, int D, int SH, int ST, int LSU = 0>
void* bulk_ptr() {
  if constexpr (G) return reinterpret_cast<void*>(mp_swap_bulk_g<D, SH, ST, CAP, LSU>);
  else return reinterpret_cast<void*>(mp_swap_bulk<D, SH, ST, CAP, LSU>);
}
template <int CAP, bool G, int D, int T, int U, int VB, bool H, bool PF>
void* direct_ptr() {
  if constexpr (G) return reinterpret_cast<void*>(mp_swap_direct_g<D, T, U, VB, H, PF, CAP>);
  else return reinterpret_cast<void*>(mp_swap_direct<D, T, U, VB, H, PF, CAP>);
}

// G = false: the table is a __grid_constant__ parameter; G = true: a pointer
// to a device-resident table (TableRing).
template <int CAP, bool G>
std::conditional_t<G, KernelFnG<CAP>, KernelFn<CAP>> kernel_for(int path, int variant, int dir, bool pf) {
  const bool o = dir == kDirOut;
#define MP_BULK(SH, ST) (o ? bulk_ptr<CAP, G, kDirOut, SH, ST>() : bulk_ptr<CAP, G, kDirIn, SH, ST>())
#define MP_DIRECT1(D, T, U, VB, H) \
  (pf ? direct_ptr<CAP, G, D, T, U, VB, H, true>() : direct_ptr<CAP, G, D, T, U, VB, H, false>())
#define MP_DIRECT(T, U, VB, H) (o ? MP_DIRECT1(kDirOut, T, U, VB, H) : MP_DIRECT1(kDirIn, T, U, VB, H))
  void* k;
  if (path == MPRESS_PATH_BULK) {
    switch (variant) {
      case 1: k = MP_BULK(14, 12); break;
      case 2: k = MP_BULK(16, 3); break;
      case 3: k = MP_BULK(15, 3); break;
      case 4: k = MP_BULK(14, 4); break;
      case 5: k = MP_BULK(13, 2); break;
      case 6: k = MP_BULK(12, 3); break;
      case 7: k = MP_BULK(12, 4); break;
      case 8: k = MP_BULK(11, 8); break;
      case 9: k = o ? bulk_ptr<CAP, G, kDirOut, 12, 4, 1>() : bulk_ptr<CAP, G, kDirIn, 12, 4, 1>(); break;
      default: k = MP_BULK(15, 6); break;
    }
  } else {
    switch (variant) {
      case 1: k = MP_DIRECT(512, 8, 16, false); break;
      case 2: k = MP_DIRECT(256, 16, 16, false); break;
      case 3: k = MP_DIRECT(1024, 4, 16, false); break;
      case 4: k = MP_DIRECT(128, 8, 16, false); break;
      case 5: k = MP_DIRECT(256, 4, 32, false); break;
      case 6: k = MP_DIRECT(256, 8, 32, false); break;
      case 7: k = MP_DIRECT(128, 4, 32, false); break;
      case 8: k = MP_DIRECT(256, 4, 32, true); break;
      case 9: k = MP_DIRECT(128, 8, 32, false); break;
      case 10: k = MP_DIRECT(128, 16, 32, false); break;
      case 11: k = MP_DIRECT(64, 16, 32, false); break;
      case 12: k = MP_DIRECT(128, 8, 32, true); break;
      case 13: k = MP_DIRECT(32, 16, 32, false); break;
      default: k = MP_DIRECT(256, 8, 16, false); break;
    }
  }
#undef MP_DIRECT
#undef MP_DIRECT1
#undef MP_BULK
  return reinterpret_cast<std::conditional_t<G, KernelFnG<CAP>, KernelFn<CAP>>>(k);
}

const Shape& shape_of(int path, int variant) {
  return path == MPRESS_PATH_BULK ? kBulk[variant] : kDirect[variant];
}

// Per-device cache of the default grid.
struct DevCache {
  std::mutex mu;
  int wave[2][16][64] = {};
};
DevCache g_cache;

// Opt a kernel into > 48 KB of dynamic shared memory, once per device.
template <typename K>
int prepare(K k, const Shape& sh) {
  if (sh.smem <= 48 * 1024) return MPRESS_OK;
  static std::mutex mu;
  static std::set<std::pair<int, const void*>> done;
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return fail(MPRESS_ERR_CUDA, "cudaGetDevice failed");
  std::lock_guard<std::mutex> lk(mu);
  if (done.count({dev, (const void*)k})) return MPRESS_OK;
  cudaError_t e = cudaFuncSetAttribute((const void*)k, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sh.smem);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "cudaFuncSetAttribute(smem): %s", cudaGetErrorString(e));
  done.insert({dev, (const void*)k});
  return MPRESS_OK;
}

// Fill the table for descriptors d[0..n) (group ids gid[]); *chunks = the
// launch's chunk count (0: nothing to move).
template <int CAP>
int build_table(CopyTable<CAP>& t, const CopyDesc* d, const int* gid, uint32_t n, uint32_t shift,
                uint64_t* chunks_out) {
  t.n = n;
  t.pace_ns = 0;
  t.split = 0;
  t.qlim = 0;
  t.dyn = nullptr;
  uint64_t chunks = 0;
  uint32_t ng = 0;
  for (uint32_t i = 0; i < n; ++i) {
    if (i == 0 || (gid && gid[i] != gid[i - 1])) {
      if (ng == (uint32_t)CopyTable<CAP>::kGroups) return fail(MPRESS_ERR_ARG, "more than %d peers in one swap", CopyTable<CAP>::kGroups);
      t.g_desc[ng] = i;
      t.g_chunk[ng++] = (uint32_t)chunks;
    }
    t.d[i] = d[i];
    t.first_chunk[i] = (uint32_t)chunks;
    chunks += (d[i].len + (1ull << shift) - 1) >> shift;
    if (chunks > 0xFFFFFFFFull) return fail(MPRESS_ERR_ARG, "swap batch exceeds 2^32 chunks");
  }
  t.first_chunk[n] = (uint32_t)chunks;
  t.g_chunk[ng] = (uint32_t)chunks;
  t.g_desc[ng] = n;
  t.n_groups = ng;
  uint32_t largest = 0;
  for (uint32_t g = 0; g < ng; ++g) largest = std::max(largest, t.g_chunk[g + 1] - t.g_chunk[g]);
  t.rounds_log2 = 0;
  while ((1ull << t.rounds_log2) < largest) ++t.rounds_log2;
  *chunks_out = chunks;
  return MPRESS_OK;
}

// ns between one CTA's chunks so that `grid` CTAs move 2^shift-byte chunks
// at pace_mbps MB/s in total (0 = unpaced).
uint32_t pace_ns_of(uint64_t pace_mbps, uint32_t shift, unsigned grid) {
  if (!pace_mbps) return 0;
  const uint64_t ns = ((uint64_t)grid << shift) * 1000ull / pace_mbps;
  return (uint32_t)std::min<uint64_t>(std::max<uint64_t>(ns, 1), 0xFFFFFFFFull);
}

template <typename K, typename Arg>
int launch_kernel(K k, const Shape& sh, unsigned grid, bool pdl, cudaStream_t stream, Arg arg) {
  MP_TRY(prepare(k, sh));
  cudaLaunchConfig_t cfg = {};
  cfg.gridDim = dim3(grid);
  cfg.blockDim = dim3(sh.threads);
  cfg.dynamicSmemBytes = sh.smem;
  cfg.stream = stream;
  cudaLaunchAttribute attr[1];
  attr[0].id = cudaLaunchAttributeProgrammaticStreamSerialization;
  attr[0].val.programmaticStreamSerializationAllowed = 1;
  cfg.attrs = attr;
  cfg.numAttrs = pdl ? 1 : 0;
  HP_START();
  cudaError_t e = cudaLaunchKernelEx(&cfg, k, arg);
  HP_LAP(11, "launch: cudaLaunchKernelEx");
  if (e == cudaSuccess) e = cudaGetLastError();
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "swap kernel launch: %s", cudaGetErrorString(e));
  return MPRESS_OK;
}

// One launch with the table as a kernel parameter.
// MPRESS_SPLIT_DYNAMIC: the claim-counter slot of a launch of `chunks`
// chunks over `grid` CTAs (*slot = -1 and a static split otherwise).
// Tuning knobs of the dynamic split for A/B runs (tools/split_ab.py):
// MPRESS_DYN_QMIN / _QMAX (smallest / largest claim, positions; 0 = the
// default) and MPRESS_DYN_MIN (chunks per CTA below which a launch stays
// blocked; 0 = the default).
uint32_t env_u32(const char* name, uint32_t dflt) {
  const char* v = getenv(name);
  return v && *v ? (uint32_t)strtoul(v, nullptr, 10) : dflt;
}

int take_counter(CounterRing* r, int path, int split, uint32_t shift, uint64_t chunks, unsigned grid,
                 bool full_grid, unsigned long long** dyn, int* slot, uint32_t* split_out, uint32_t* qlim) {
  static const uint32_t kQmin = env_u32("MPRESS_DYN_QMIN", 1);
  static const uint32_t kQmax = env_u32("MPRESS_DYN_QMAX", 0);
  static const uint32_t kMinPerCta = env_u32("MPRESS_DYN_MIN", 0);
  *dyn = nullptr;
  *slot = -1;
  // largest claim ~128 KiB of pieces (4 x 32 KiB ... 32 x 4 KiB): a tight
  // front, few enough atomics (tools/split_ab.py, profiles/r02/split_ab)
  const uint32_t qmax = kQmax ? kQmax : std::min(32u, std::max(4u, (1u << 17) >> shift));
  *qlim = (kQmin & 0xFFFFu) | (qmax << 16);
  // AUTO: launches of < kDynAutoChunksPerCta chunks per CTA take the grid
  // stride (every CTA inside one window of the sequence: +4-7% at 64 MiB,
  // +1-2% at 256 MiB over blocked on B200 loopback), larger TMA launches the
  // dynamic claims, larger direct launches the blocked split (there the
  // claims and the stride cost 2-12%: profiles/r02/split_ab/);
  // DYNAMIC: claims for any launch of >= kDynMinChunksPerCta chunks per CTA
  // (the stride only on a full grid: on a capped one the skipped positions
  // of a multi-peer sequence alias with it, 8-12% slower at 32-64 CTAs)
  const bool small = chunks < (uint64_t)kDynAutoChunksPerCta * grid;
  const bool stride = split == MPRESS_SPLIT_STRIDED || (split == MPRESS_SPLIT_AUTO && small && full_grid);
  *split_out = (uint32_t)(stride ? kSplitStrided : kSplitBlocked);
  const bool dynamic =
      r && ((split == MPRESS_SPLIT_DYNAMIC &&
             chunks >= (uint64_t)(kMinPerCta ? kMinPerCta : kDynMinChunksPerCta) * grid) ||
            (split == MPRESS_SPLIT_AUTO && path == MPRESS_PATH_BULK &&
             chunks >= (uint64_t)(kMinPerCta ? kMinPerCta : kDynAutoChunksPerCta) * grid));
  if (!dynamic) return MPRESS_OK;
  const int k = r->next;
  if (r->armed[k]) {
    const cudaError_t e = cudaEventSynchronize(r->ev[k]);   // blocks only if the ring wrapped
    if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "claim-counter ring: %s", cudaGetErrorString(e));
    r->armed[k] = false;
  }
  r->next = (k + 1) % r->nslots;
  *dyn = r->dev + (size_t)k * 16;
  *slot = k;
  return MPRESS_OK;
}

int arm_counter(CounterRing* r, int slot, cudaStream_t stream) {
  if (slot < 0) return MPRESS_OK;
  const cudaError_t e = cudaEventRecord(r->ev[slot], stream);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "claim-counter event: %s", cudaGetErrorString(e));
  r->armed[slot] = true;
  return MPRESS_OK;
}

template <int CAP>
int launch_batch(int path, int variant, int dir, const CopyDesc* d, const int* gid, uint32_t n,
                 uint32_t shift, int cap, int sms, bool pdl, uint64_t pace_mbps, int split, CounterRing* cr,
                 cudaStream_t stream, bool* launched) {
  CopyTable<CAP> t;
  uint64_t chunks = 0;
  *launched = false;
  MP_TRY(build_table(t, d, gid, n, shift, &chunks));
  if (chunks == 0) return MPRESS_OK;
  const unsigned grid = (unsigned)std::min<uint64_t>(chunks, (uint64_t)cap);
  t.pace_ns = pace_ns_of(pace_mbps, shift, grid);
  int slot;
  MP_TRY(take_counter(cr, path, split, shift, chunks, grid, (int)grid >= sms, &t.dyn, &slot, &t.split, &t.qlim));
  const Shape& sh = shape_of(path, variant);
  MP_TRY(launch_kernel(kernel_for<CAP, false>(path, variant, dir, (int)grid <= sms), sh, grid, pdl, stream, t));
  *launched = true;
  return arm_counter(cr, slot, stream);
}

// One launch with the table device-resident (TableRing): built in a pinned
// staging slot, copied to the device slot on `stream` (only the used prefix),
// read by the kernel through a pointer; the slot's event, recorded after the
// kernel, guards both slots' reuse.
int launch_batch_ring(TableRing* r, int path, int variant, int dir, const CopyDesc* d, const int* gid, uint32_t n,
                      uint32_t shift, int cap, int sms, bool pdl, uint64_t pace_mbps, int split, CounterRing* cr,
                      cudaStream_t stream, bool* launched) {
  using T = CopyTable<kMaxDescPerLaunch>;
  *launched = false;
  const int slot = r->next;
  if (r->armed[slot]) {
    const cudaError_t e = cudaEventSynchronize(r->ev[slot]);   // blocks only if the ring wrapped
    if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "descriptor ring: %s", cudaGetErrorString(e));
    r->armed[slot] = false;
  }
  T* ht = reinterpret_cast<T*>(r->host + (size_t)slot * r->slot_bytes);
  T* dt = reinterpret_cast<T*>(r->dev + (size_t)slot * r->slot_bytes);
  uint64_t chunks = 0;
  MP_TRY(build_table(*ht, d, gid, n, shift, &chunks));
  if (chunks == 0) return MPRESS_OK;
  r->next = (slot + 1) % r->nslots;
  const unsigned grid = (unsigned)std::min<uint64_t>(chunks, (uint64_t)cap);
  ht->pace_ns = pace_ns_of(pace_mbps, shift, grid);
  int cslot;
  MP_TRY(take_counter(cr, path, split, shift, chunks, grid, (int)grid >= sms, &ht->dyn, &cslot, &ht->split, &ht->qlim));
  const size_t bytes = offsetof(T, d) + (size_t)n * sizeof(CopyDesc);
  cudaError_t e = cudaMemcpyAsync(dt, ht, bytes, cudaMemcpyHostToDevice, stream);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "descriptor upload: %s", cudaGetErrorString(e));
  const Shape& sh = shape_of(path, variant);
  MP_TRY(launch_kernel(kernel_for<kMaxDescPerLaunch, true>(path, variant, dir, (int)grid <= sms), sh, grid, pdl,
                       stream, static_cast<const T*>(dt)));
  e = cudaEventRecord(r->ev[slot], stream);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "descriptor ring event: %s", cudaGetErrorString(e));
  r->armed[slot] = true;
  *launched = true;
  return arm_counter(cr, cslot, stream);
}

}  // namespace

int sm_count(int* dev_out) {
  // per device, queried once (every swap call needs it: grid caps, PDL and
  // the AUTO path depend on "capped to <= one CTA per SM")
  static std::atomic<int> cache[64];
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  if (dev_out) *dev_out = dev;
  if (dev < 0 || dev >= 64) {
    int sms = 0;
    return cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) == cudaSuccess ? sms : 0;
  }
  int sms = cache[dev].load(std::memory_order_relaxed);
  if (sms == 0) {
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
    cache[dev].store(sms, std::memory_order_relaxed);
  }
  return sms;
}

int copy_wave_ctas(int path, int variant) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
  const int pi = path == MPRESS_PATH_BULK ? 1 : 0;
  std::lock_guard<std::mutex> lk(g_cache.mu);
  int& w = g_cache.wave[pi][variant][dev];
  if (w == 0) {
    const Shape& sh = shape_of(path, variant);
    KernelFn<kMaxDescPerLaunch> k = kernel_for<kMaxDescPerLaunch, false>(path, variant, kDirOut, false);
    if (prepare(k, sh) != MPRESS_OK) return 0;
    int sms = 0, per_sm = 0;
    if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
    if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, (const void*)k, sh.threads, sh.smem) != cudaSuccess)
      return 0;
    w = sms * std::max(1, std::min(per_sm, sh.per_sm));
  }
  return w;
}

namespace {
template <int CAP, bool G>
int preload_cap() {
  for (int path : {MPRESS_PATH_DIRECT, MPRESS_PATH_BULK}) {
    const int nvar = path == MPRESS_PATH_BULK ? kBulkVariants : kDirectVariants;
    for (int v = 0; v < nvar; ++v)
      for (int dir : {kDirOut, kDirIn})
        for (bool pf : {false, true}) {
          cudaFuncAttributes a;
          auto k = kernel_for<CAP, G>(path, v, dir, pf);
          if (cudaFuncGetAttributes(&a, (const void*)k) != cudaSuccess)
            return fail(MPRESS_ERR_CUDA, "cannot load the swap kernels");
          MP_TRY(prepare(k, shape_of(path, v)));
        }
  }
  return MPRESS_OK;
}
}  // namespace

// With lazy module loading (the CUDA 12 default) a kernel's first launch may
// wait for the whole device; loading every swap kernel at context creation
// keeps that stall out of the training step.
int preload_kernels() {
  MP_TRY((preload_cap<16, false>()));
  MP_TRY((preload_cap<32, false>()));
  MP_TRY((preload_cap<64, false>()));
  MP_TRY((preload_cap<128, false>()));
  MP_TRY((preload_cap<kMaxDescPerLaunch, false>()));
  return preload_cap<kMaxDescPerLaunch, true>();
}

int table_ring_create(int device, TableRing** out) {
  *out = nullptr;
  auto* r = new TableRing();
  r->device = device;
  r->slot_bytes = (sizeof(CopyTable<kMaxDescPerLaunch>) + 255) / 256 * 256;
  r->nslots = 256;   // 7.4 MB device + 7.4 MB pinned: 256 large launches in flight before the host waits
  r->ev = new cudaEvent_t[r->nslots]();
  r->armed = new bool[r->nslots]();
  const size_t bytes = r->slot_bytes * r->nslots;
  cudaError_t e = cudaMalloc(&r->dev, bytes);
  if (e == cudaSuccess) e = cudaHostAlloc(&r->host, bytes, cudaHostAllocDefault);
  for (int i = 0; i < r->nslots && e == cudaSuccess; ++i) e = cudaEventCreateWithFlags(&r->ev[i], cudaEventDisableTiming);
  if (e != cudaSuccess) {
    table_ring_destroy(r);
    return fail(MPRESS_ERR_CUDA, "descriptor ring (%zu B): %s", bytes, cudaGetErrorString(e));
  }
  *out = r;
  return MPRESS_OK;
}

void table_ring_destroy(TableRing* r) {
  if (!r) return;
  for (int i = 0; i < r->nslots; ++i) {
    if (r->armed[i]) cudaEventSynchronize(r->ev[i]);
    if (r->ev[i]) cudaEventDestroy(r->ev[i]);
  }
  if (r->dev) cudaFree(r->dev);
  if (r->host) cudaFreeHost(r->host);
  delete[] r->ev;
  delete[] r->armed;
  delete r;
}

int counter_ring_create(int device, CounterRing** out) {
  *out = nullptr;
  auto* r = new CounterRing();
  r->device = device;
  r->nslots = 256;
  r->ev = new cudaEvent_t[r->nslots]();
  r->armed = new bool[r->nslots]();
  const size_t bytes = (size_t)r->nslots * 16 * sizeof(unsigned long long);
  cudaError_t e = cudaMalloc(&r->dev, bytes);
  if (e == cudaSuccess) e = cudaMemset(r->dev, 0, bytes);
  if (e == cudaSuccess) e = cudaDeviceSynchronize();
  for (int i = 0; i < r->nslots && e == cudaSuccess; ++i) e = cudaEventCreateWithFlags(&r->ev[i], cudaEventDisableTiming);
  if (e != cudaSuccess) {
    counter_ring_destroy(r);
    return fail(MPRESS_ERR_CUDA, "claim-counter ring: %s", cudaGetErrorString(e));
  }
  *out = r;
  return MPRESS_OK;
}

void counter_ring_destroy(CounterRing* r) {
  if (!r) return;
  for (int i = 0; i < r->nslots; ++i) {
    if (r->armed[i]) cudaEventSynchronize(r->ev[i]);
    if (r->ev[i]) cudaEventDestroy(r->ev[i]);
  }
  if (r->dev) cudaFree(r->dev);
  delete[] r->ev;
  delete[] r->armed;
  delete r;
}

int launch_copy(int path, int variant, int dir, const CopyDesc* d, const int* group, size_t n,
                int max_ctas, int pdl_mode, cudaStream_t stream, int* launches, TableRing* ring,
                uint64_t pace_mbps, int split, CounterRing* counters) {
  const int sms = sm_count(nullptr);
  if (sms <= 0) return fail(MPRESS_ERR_CUDA, "cannot query the SM count");
  // PDL (MPRESS_OPT_PDL): mode 1 only for an uncapped grid.  A capped swap
  // runs beside a GEMM, and there a PDL chain of swap kernels (the next one
  // launched early, parked in griddepcontrol.wait) cost the concurrent cuBLAS
  // GEMM +60% instead of +6-9% (profiles/r01/pdl_gemm_ab.txt).
  const bool capped = max_ctas > 0 && max_ctas <= sms;
  const bool pdl = pdl_mode == 2 || (pdl_mode == 1 && !capped);
  if (variant == MPRESS_VARIANT_AUTO) {
    // direct, capped grid (<= one CTA per SM, i.e. beside a GEMM): 128-thread
    // CTAs fit in the registers and shared memory a cuBLAS GEMM CTA leaves
    // free (168 regs x 256 threads + 214 KB smem, profiles/r01), so they
    // co-reside instead of taking SMs away from it; full grid: 2 x 256-thread
    // CTAs per SM saturate HBM (profiles/r01 sweeps).  Both use 32-byte
    // vectors (LDG/STG .256, +1% over 16-byte ones; 16-byte fallback when the
    // data is only 16-byte aligned).  bulk: 3 x 32 KiB, one CTA per SM
    // (profiles/r01/sweep_bulk_variants.jsonl).
    // Capped: 128 x 8 x 32 B (shape 9), 32 KiB of loads in flight per CTA --
    // twice shape 7's, which left a 64-CTA swap latency-bound at 1.2 TB/s on
    // loopback (2x that latency over NVLink); 1.8 TB/s now, ~96 registers x
    // 128 threads, still beside a GEMM CTA (profiles/r02/capped_*).
    if (path == MPRESS_PATH_DIRECT)
      variant = (max_ctas > 0 && max_ctas <= sms) ? 9 : 5;
    else
      variant = 3;
    // Few chunks per SM on a full grid (< 16: a launch of < ~74 MiB): the
    // whole launch is ramp and tail, and a deeper ring per SM wins -- bulk
    // 6 x 32 KiB (shape 0) instead of 3 x 32 KiB, direct 512 x 8 x 16 B
    // (shape 1, 64 KiB of loads per CTA) instead of 2 x 256 x 4 x 32 B: e.g.
    // 32 MiB over 3 peers 2428 -> 3069 GB/s out (bulk), 2333 -> 2997
    // (direct); 16 MiB 1827 -> 2232 in.  At 128 MiB (28 chunks per CTA) the
    // default shapes are faster again (bulk 3005 vs 2746, direct 2918 vs 2842).
    // (profiles/r02/small_shapes*.jsonl).
    if (!capped) {
      const uint32_t sh = shape_of(path, variant).shift;
      uint64_t chunks = 0;
      for (size_t i = 0; i < n; ++i) chunks += (d[i].len + (1ull << sh) - 1) >> sh;
      if (chunks < (uint64_t)kDeepChunksPerCta * (uint64_t)sms)
        variant = path == MPRESS_PATH_DIRECT ? 1 : 0;
    }
  }
  const int nvar = path == MPRESS_PATH_BULK ? kBulkVariants : kDirectVariants;
  if (variant < 0 || variant >= nvar) return fail(MPRESS_ERR_ARG, "kernel variant %d out of range", variant);
  if (shape_of(path, variant).vb == 32) {  // 32-byte vectors need 32-byte aligned addresses
    for (size_t i = 0; i < n; ++i)
      if ((reinterpret_cast<uintptr_t>(d[i].src) | reinterpret_cast<uintptr_t>(d[i].dst)) & 31) {
        variant = shape_of(path, variant).fallback;
        break;
      }
  }
  const int wave = copy_wave_ctas(path, variant);
  if (wave <= 0) return fail(MPRESS_ERR_CUDA, "occupancy query failed");
  const int cap = max_ctas > 0 ? max_ctas : wave;
  const uint32_t shift = shape_of(path, variant).shift;
  for (size_t base = 0; base < n; base += kMaxDescPerLaunch) {
    const uint32_t m = (uint32_t)std::min<size_t>(kMaxDescPerLaunch, n - base);
    const int* g = group ? group + base : nullptr;
    bool launched = false;
    if (ring && m > (uint32_t)kParamDescMax)
      MP_TRY(launch_batch_ring(ring, path, variant, dir, d + base, g, m, shift, cap, sms, pdl, pace_mbps, split, counters, stream, &launched));
    else if (m <= 16)
      MP_TRY(launch_batch<16>(path, variant, dir, d + base, g, m, shift, cap, sms, pdl, pace_mbps, split, counters, stream, &launched));
    else if (m <= 32)
      MP_TRY(launch_batch<32>(path, variant, dir, d + base, g, m, shift, cap, sms, pdl, pace_mbps, split, counters, stream, &launched));
    else if (m <= 64)
      MP_TRY(launch_batch<64>(path, variant, dir, d + base, g, m, shift, cap, sms, pdl, pace_mbps, split, counters, stream, &launched));
    else if (m <= 128)
      MP_TRY(launch_batch<128>(path, variant, dir, d + base, g, m, shift, cap, sms, pdl, pace_mbps, split, counters, stream, &launched));
    else
      MP_TRY(launch_batch<kMaxDescPerLaunch>(path, variant, dir, d + base, g, m, shift, cap, sms, pdl, pace_mbps, split, counters, stream, &launched));
    if (launched && launches) ++*launches;
  }
  return MPRESS_OK;
}

}  // namespace mpress
