// sm_100a swap kernels: the byte movers of swap-out and swap-in
// (P:121).
//
// The D2D swap moves bytes and computes nothing (tensor cores unused), so the
// kernels are shaped by the memory system alone:
//   * one launch per plan (the whole batch, "we also batch tensors"),
//     descriptors passed as a __grid_constant__ parameter (no upload);
//   * the batch is cut into fixed-size chunks that a grid of CTAs walks with a
//     grid stride, so adjacent chunks are in flight on different SMs at once;
//   * the grid is capped (MPRESS_OPT_MAX_CTAS) so a concurrent GEMM keeps
//     most SMs;
//   * every address is 16-B aligned (tensor pointers are checked; stripe
//     offsets are multiples of 256, R6), so bodies move int4 / bulk pieces and
//     only the last <16 bytes of a tensor take a byte loop.
//
// PATH_DIRECT: 256 threads, each issuing 8 independent 16-B loads before its
//   8 stores (32 KiB per CTA in flight per chunk), L1 bypassed on both sides.
//   Peer addresses route over NVLink by their VA; loads of peer memory bypass
//   the local L2 (B300_MICROARCH.md "NVLink"), so depth of outstanding loads
//   sets swap-in bandwidth (Little's law).
// PATH_BULK: one warp per CTA drives the bulk-async copy engine of the SM
//   (cp.async.bulk, SASS UBLKCP): chunk loads land in a ring of shared-memory
//   slots (mbarrier completion), then bulk stores drain them, so one SM keeps
//   kStages*32 KiB in flight with a single issuing thread.
#include <cuda_runtime.h>

#include <algorithm>
#include <mutex>

#include "common.h"
#include "swap_kernels.h"

namespace mpress {
namespace {

constexpr int kThreads = 256;                 // direct path CTA size
constexpr int kUnroll = 8;                    // 16-B vectors in flight per thread
constexpr uint32_t kChunk = kThreads * kUnroll * 16;  // 32 KiB per chunk
constexpr uint32_t kChunkShift = 15;
static_assert((1u << kChunkShift) == kChunk, "chunk must be a power of two");

constexpr int kBulkThreads = 32;
constexpr uint32_t kSlot = 32768;             // bytes per bulk piece / smem slot
constexpr int kStages = 6;                    // 192 KiB of shared memory per CTA
constexpr uint32_t kSlotShift = 15;
static_assert((1u << kSlotShift) == kSlot, "slot must be a power of two");

struct CopyTable {
  uint32_t n;                                  // descriptors
  uint32_t total_chunks;                       // chunks over all descriptors
  uint32_t first_chunk[kMaxDescPerLaunch + 1]; // prefix sum of chunks
  CopyDesc d[kMaxDescPerLaunch];
};
static_assert(sizeof(CopyTable) <= 32764, "kernel parameter space is 32764 bytes");

__device__ __forceinline__ uint32_t find_desc(const CopyTable& t, uint32_t c) {
  // largest s with first_chunk[s] <= c (first_chunk[0] == 0)
  uint32_t lo = 0, hi = t.n;
  while (hi - lo > 1) {
    uint32_t mid = (lo + hi) >> 1;
    if (t.first_chunk[mid] <= c) lo = mid; else hi = mid;
  }
  return lo;
}

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

// Bytes [off, off+len) of one descriptor, len <= kChunk, by all kThreads threads.
__device__ __forceinline__ void copy_partial(const uint8_t* src, uint8_t* dst, uint32_t len) {
  const uint32_t n16 = len >> 4;
  const int4* s = reinterpret_cast<const int4*>(src);
  int4* o = reinterpret_cast<int4*>(dst);
  for (uint32_t v = threadIdx.x; v < n16; v += kThreads) st_stream(o + v, ld_stream(s + v));
  const uint32_t tail = len & 15u;
  if (threadIdx.x < tail) dst[(n16 << 4) + threadIdx.x] = src[(n16 << 4) + threadIdx.x];
}

template <int DIR>
__global__ void __launch_bounds__(kThreads)
mp_swap_direct(const __grid_constant__ CopyTable t) {
  for (uint32_t c = blockIdx.x; c < t.total_chunks; c += gridDim.x) {
    const uint32_t s = find_desc(t, c);
    const CopyDesc& d = t.d[s];
    const uint64_t off = (uint64_t)(c - t.first_chunk[s]) << kChunkShift;
    const uint8_t* src = static_cast<const uint8_t*>(d.src) + off;
    uint8_t* dst = static_cast<uint8_t*>(d.dst) + off;
    const uint64_t rem = d.len - off;
    if (rem >= kChunk) {
      const int4* sv = reinterpret_cast<const int4*>(src) + threadIdx.x;
      int4* dv = reinterpret_cast<int4*>(dst) + threadIdx.x;
      int4 v[kUnroll];
#pragma unroll
      for (int j = 0; j < kUnroll; ++j) v[j] = ld_stream(sv + j * kThreads);
#pragma unroll
      for (int j = 0; j < kUnroll; ++j) st_stream(dv + j * kThreads, v[j]);
    } else {
      copy_partial(src, dst, (uint32_t)rem);
    }
  }
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

__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  asm volatile(
      "{\n"
      ".reg .pred p;\n"
      "WAIT_%=:\n"
      "mbarrier.try_wait.parity.shared::cta.b64 p, [%0], %1;\n"
      "@!p bra WAIT_%=;\n"
      "}\n" :: "r"(smem_u32(bar)), "r"(parity) : "memory");
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
template <int N>
__device__ __forceinline__ void bulk_wait_read() {
  asm volatile("cp.async.bulk.wait_group.read %0;" :: "n"(N) : "memory");
}
__device__ __forceinline__ void bulk_wait_all() { asm volatile("cp.async.bulk.wait_group 0;" ::: "memory"); }

struct Piece {
  const uint8_t* src;
  uint8_t* dst;
  uint32_t bytes;  // multiple of 16
};

__device__ __forceinline__ Piece bulk_piece(const CopyTable& t, uint32_t c) {
  const uint32_t s = find_desc(t, c);
  const CopyDesc& d = t.d[s];
  const uint64_t off = (uint64_t)(c - t.first_chunk[s]) << kSlotShift;
  const uint64_t rem = d.len - off;
  Piece p;
  p.src = static_cast<const uint8_t*>(d.src) + off;
  p.dst = static_cast<uint8_t*>(d.dst) + off;
  p.bytes = (uint32_t)(rem >= kSlot ? kSlot : (rem & ~15ull));
  return p;
}

template <int DIR>
__global__ void __launch_bounds__(kBulkThreads)
mp_swap_bulk(const __grid_constant__ CopyTable t) {
  extern __shared__ __align__(128) uint8_t smem[];
  __shared__ __align__(8) uint64_t bars[kStages];

  const uint32_t first = blockIdx.x;
  const uint32_t mine = first < t.total_chunks ? (t.total_chunks - first + gridDim.x - 1) / gridDim.x : 0;

  // Sub-16-byte tails (last chunk of a descriptor whose length % 16 != 0):
  // plain byte copies by the warp, disjoint from every bulk piece.
  for (uint32_t i = 0; i < mine; ++i) {
    const uint32_t c = first + i * gridDim.x;
    const uint32_t s = find_desc(t, c);
    if (c + 1 != t.first_chunk[s + 1]) continue;  // not the last chunk of desc s
    const CopyDesc& d = t.d[s];
    const uint32_t tail = (uint32_t)(d.len & 15u);
    if (threadIdx.x < tail) {
      const uint64_t b = (d.len & ~15ull) + threadIdx.x;
      static_cast<uint8_t*>(d.dst)[b] = static_cast<const uint8_t*>(d.src)[b];
    }
  }
  if (threadIdx.x != 0 || mine == 0) return;

  for (int k = 0; k < kStages; ++k) mbar_init(&bars[k], 1);
  asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");

  auto issue_load = [&](uint32_t i) {
    const Piece p = bulk_piece(t, first + i * gridDim.x);
    uint64_t* bar = &bars[i % kStages];
    mbar_expect_tx(bar, p.bytes);
    if (p.bytes) bulk_load(smem + (size_t)(i % kStages) * kSlot, p.src, p.bytes, bar);
  };

  const uint32_t prologue = mine < (uint32_t)kStages ? mine : (uint32_t)kStages;
  for (uint32_t i = 0; i < prologue; ++i) issue_load(i);
  for (uint32_t i = 0; i < mine; ++i) {
    mbar_wait(&bars[i % kStages], (i / kStages) & 1u);
    const Piece p = bulk_piece(t, first + i * gridDim.x);
    if (p.bytes) bulk_store(p.dst, smem + (size_t)(i % kStages) * kSlot, p.bytes);
    bulk_commit();
    // Refill the slot of piece i-1 once its store has finished reading smem
    // (at most the newest group, piece i's store, may still be reading).
    if (i >= 1) {
      const uint32_t nxt = i - 1 + kStages;
      if (nxt < mine) {
        bulk_wait_read<1>();
        issue_load(nxt);
      }
    }
  }
  bulk_wait_all();
}

struct WaveCache {
  std::mutex mu;
  int ctas[2][64] = {};
};
WaveCache g_wave;

template <typename K>
int wave_of(K kernel, int threads, size_t smem) {
  int dev = 0, sms = 0, per_sm = 0;
  if (cudaGetDevice(&dev) != cudaSuccess) return 0;
  if (cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev) != cudaSuccess) return 0;
  if (cudaOccupancyMaxActiveBlocksPerMultiprocessor(&per_sm, kernel, threads, smem) != cudaSuccess) return 0;
  return sms * std::max(per_sm, 1);
}

constexpr size_t kBulkSmem = (size_t)kStages * kSlot;

int configure_bulk_once() {
  // The dynamic-smem opt-in is a per-device function attribute.
  static std::mutex mu;
  static bool done[64] = {};
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64)
    return fail(MPRESS_ERR_CUDA, "cudaGetDevice failed");
  std::lock_guard<std::mutex> lk(mu);
  if (done[dev]) return MPRESS_OK;
  cudaError_t err = cudaFuncSetAttribute(mp_swap_bulk<kDirOut>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBulkSmem);
  if (err == cudaSuccess)
    err = cudaFuncSetAttribute(mp_swap_bulk<kDirIn>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)kBulkSmem);
  if (err != cudaSuccess)
    return fail(MPRESS_ERR_CUDA, "cudaFuncSetAttribute(bulk smem): %s", cudaGetErrorString(err));
  done[dev] = true;
  return MPRESS_OK;
}

}  // namespace

int copy_wave_ctas(int path) {
  int dev = 0;
  if (cudaGetDevice(&dev) != cudaSuccess || dev < 0 || dev >= 64) return 0;
  const int slot = path == MPRESS_PATH_BULK ? 1 : 0;
  std::lock_guard<std::mutex> lk(g_wave.mu);
  if (g_wave.ctas[slot][dev] == 0) {
    if (slot == 1) {
      if (configure_bulk_once() != MPRESS_OK) return 0;
      g_wave.ctas[slot][dev] = wave_of(mp_swap_bulk<kDirOut>, kBulkThreads, kBulkSmem);
    } else {
      g_wave.ctas[slot][dev] = wave_of(mp_swap_direct<kDirOut>, kThreads, 0);
    }
  }
  return g_wave.ctas[slot][dev];
}

int launch_copy(int path, int dir, const CopyDesc* d, size_t n, int max_ctas,
                cudaStream_t stream, int* launches) {
  const bool bulk = path == MPRESS_PATH_BULK;
  if (bulk) MP_TRY(configure_bulk_once());
  const int wave = copy_wave_ctas(path);
  if (wave <= 0) return fail(MPRESS_ERR_CUDA, "occupancy query failed");
  const int cap = max_ctas > 0 ? std::min(max_ctas, wave) : wave;
  const uint32_t shift = bulk ? kSlotShift : kChunkShift;
  for (size_t base = 0; base < n; base += kMaxDescPerLaunch) {
    CopyTable t;
    t.n = (uint32_t)std::min<size_t>(kMaxDescPerLaunch, n - base);
    uint64_t chunks = 0;
    for (uint32_t i = 0; i < t.n; ++i) {
      t.d[i] = d[base + i];
      t.first_chunk[i] = (uint32_t)chunks;
      chunks += (d[base + i].len + (1ull << shift) - 1) >> shift;
      if (chunks > 0xFFFFFFFFull) return fail(MPRESS_ERR_ARG, "swap batch exceeds 2^32 chunks");
    }
    t.first_chunk[t.n] = (uint32_t)chunks;
    t.total_chunks = (uint32_t)chunks;
    if (chunks == 0) continue;
    const unsigned grid = (unsigned)std::min<uint64_t>(chunks, (uint64_t)cap);
    if (bulk) {
      if (dir == kDirOut) mp_swap_bulk<kDirOut><<<grid, kBulkThreads, kBulkSmem, stream>>>(t);
      else mp_swap_bulk<kDirIn><<<grid, kBulkThreads, kBulkSmem, stream>>>(t);
    } else {
      if (dir == kDirOut) mp_swap_direct<kDirOut><<<grid, kThreads, 0, stream>>>(t);
      else mp_swap_direct<kDirIn><<<grid, kThreads, 0, stream>>>(t);
    }
    cudaError_t e = cudaGetLastError();
    if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "swap kernel launch: %s", cudaGetErrorString(e));
    if (launches) ++*launches;
  }
  return MPRESS_OK;
}

}  // namespace mpress
