// Internal interface of the swap copy kernels (swap_kernels.cu).
#pragma once

#include <cuda_runtime.h>

#include <cstddef>
#include <cstdint>

namespace mpress {

// One contiguous byte move, already resolved to device addresses:
// swap-out: src = tensor + src_off (local), dst = peer slice + dst_off (peer VA);
// swap-in : src = peer slice + dst_off,      dst = destination + src_off.
struct CopyDesc {
  const void* src;
  void* dst;
  uint64_t len;
};

constexpr int kMaxDescPerLaunch = 1024;  // fits the 32 KB kernel-parameter space
constexpr int kDirectVariants = 14;      // MPRESS_OPT_VARIANT range, direct path
constexpr int kBulkVariants = 10;        // MPRESS_OPT_VARIANT range, bulk path
constexpr int kCeVariants = 1;           // copy engines: 0 = cudaMemcpyAsync per stripe, per-peer streams

enum CopyDir { kDirOut = 0, kDirIn = 1 };

// Device-resident descriptor tables for launches with more than
// kParamDescMax descriptors: a 28 KB __grid_constant__ table costs ~20 us of
// host time per launch and fills the driver's launch queue after ~60 queued
// launches (tools/hostcost.py), so large tables are written into a pinned
// staging slot, copied to a device slot on the launch's stream, and the
// kernel reads them through a pointer.  A slot is reused once the event
// recorded after its kernel has completed.  Not used under graph capture (a
// replay would re-read a staging slot that later launches overwrote).
struct TableRing {
  int device = -1;
  size_t slot_bytes = 0;
  int nslots = 0;
  uint8_t* dev = nullptr;     // nslots x slot_bytes, device memory
  uint8_t* host = nullptr;    // nslots x slot_bytes, pinned staging
  cudaEvent_t* ev = nullptr;  // per slot: recorded after the kernel reading it
  bool* armed = nullptr;      // per slot: ev was recorded
  int next = 0;
};
constexpr int kParamDescMax = 128;
int table_ring_create(int device, TableRing** out);
void table_ring_destroy(TableRing* r);

// Claim counters of MPRESS_SPLIT_DYNAMIC launches: one slot {claimed, CTAs
// done} per launch (one 128-byte line each, so concurrent launches do not
// share a line), zeroed at creation and reset by each launch's last CTA.  A
// slot is reused once the event recorded after its launch has completed.
struct CounterRing {
  int device = -1;
  int nslots = 0;
  unsigned long long* dev = nullptr;  // nslots x 16 u64
  cudaEvent_t* ev = nullptr;
  bool* armed = nullptr;
  int next = 0;
};
int counter_ring_create(int device, CounterRing** out);
void counter_ring_destroy(CounterRing* r);

// Enqueue kernels moving every descriptor on `stream`; `path` is
// MPRESS_PATH_DIRECT or MPRESS_PATH_BULK, `variant` its kernel shape;
// `max_ctas` caps the grid (0 = the variant's default grid); `pdl_mode`
// (MPRESS_OPT_PDL: 0 never, 1 uncapped grids only, 2 always) launches with
// programmatic stream serialization.  Adds the number
// of kernel launches to *launches.  Returns MPRESS_OK or MPRESS_ERR_*.
// `ring` (may be null): device-resident tables for launches of more than
// kParamDescMax descriptors.
// `pace_mbps` (MPRESS_OPT_PACE_MBPS, 0 = off): the launch's CTAs space their
// chunks so the whole launch moves at most pace_mbps MB/s.  `split`
// (MPRESS_OPT_SPLIT): 0 = each CTA takes a contiguous block of the
// interleaved chunk sequence, 1 = a grid stride over it (round 1), 2 =
// blocks claimed from a counter in `counters` (null: as 0); a launch with
// fewer than kDynMinChunksPerCta chunks per CTA runs as 0; 3 (AUTO) = 2 for
// bulk-kernel launches of >= kDynAutoChunksPerCta chunks per CTA, else 0.
constexpr int kDynMinChunksPerCta = 4;
constexpr int kDynAutoChunksPerCta = 32;
// MPRESS_VARIANT_AUTO on a full grid: launches of fewer chunks per SM (of
// the default shape) than this take the deeper-ring shape (bulk 0, direct 1).
constexpr int kDeepChunksPerCta = 16;
int launch_copy(int path, int variant, int dir, const CopyDesc* d, const int* group, size_t n,
                int max_ctas, int pdl_mode,
                cudaStream_t stream, int* launches, TableRing* ring = nullptr, uint64_t pace_mbps = 0,
                int split = 0, CounterRing* counters = nullptr);

// SM count of the current device (cached per device; 0 on error); *dev = the
// device ordinal if dev is not null.
int sm_count(int* dev);

// Default grid of a path/variant on the current device (SMs x CTAs per SM).
int copy_wave_ctas(int path, int variant);

// Load every swap kernel on the current device (no lazy-loading stall later).
int preload_kernels();

}  // namespace mpress
