// Internal state of a libmpress context and its handles (not part of the ABI).
#pragma once

#include <cuda.h>
#include <cuda_runtime.h>

#include <deque>
#include <map>
#include <memory>
#include <mutex>
#include <set>
#include <vector>

#include "common.h"
#include "swap_kernels.h"

namespace mpress {

// CUDA driver entry points, fetched through cudart (cudaGetDriverEntryPoint)
// so libmpress.so has no link-time dependency on libcuda.so: it loads and
// plans on a host without a GPU driver.
struct Driver {
  CUresult (*mem_create)(CUmemGenericAllocationHandle*, size_t, const CUmemAllocationProp*, unsigned long long);
  CUresult (*mem_release)(CUmemGenericAllocationHandle);
  CUresult (*mem_address_reserve)(CUdeviceptr*, size_t, size_t, CUdeviceptr, unsigned long long);
  CUresult (*mem_address_free)(CUdeviceptr, size_t);
  CUresult (*mem_map)(CUdeviceptr, size_t, size_t, CUmemGenericAllocationHandle, unsigned long long);
  CUresult (*mem_unmap)(CUdeviceptr, size_t);
  CUresult (*mem_set_access)(CUdeviceptr, size_t, const CUmemAccessDesc*, size_t);
  CUresult (*mem_export)(void*, CUmemGenericAllocationHandle, CUmemAllocationHandleType, unsigned long long);
  CUresult (*mem_import)(CUmemGenericAllocationHandle*, void*, CUmemAllocationHandleType);
  CUresult (*mem_granularity)(size_t*, const CUmemAllocationProp*, CUmemAllocationGranularity_flags);
  CUresult (*get_error_string)(CUresult, const char**);
};
int driver(const Driver** out);
int cu_fail(const Driver* d, CUresult r, const char* what);

// RAII: make `dev` current, restore the caller's device afterwards.
struct DeviceGuard {
  int prev = -1;
  explicit DeviceGuard(int dev) {
    cudaGetDevice(&prev);
    if (prev != dev) cudaSetDevice(dev);
  }
  ~DeviceGuard() {
    int cur = -1;
    cudaGetDevice(&cur);
    if (prev >= 0 && cur != prev) cudaSetDevice(prev);
  }
};

// A VMM mapping: physical allocation (created or imported) mapped at `va`.
struct Mapping {
  CUmemGenericAllocationHandle handle = 0;
  CUdeviceptr va = 0;
  size_t size = 0;
  bool reserved = false, mapped = false, has_handle = false;
  void* host = nullptr;  // NEXT-4: pinned host pool (cudaHostAlloc, mapped)
  void* ipc_owned = nullptr;   // legacy-IPC transport: this rank's cudaMalloc pool
  void* ipc_opened = nullptr;  // legacy-IPC transport: a peer's pool, opened here
};

// A CUDA event shared by a handle and the fences its swap-in leaves behind;
// it returns to the context's pool when the last owner releases it.
using EvRef = std::shared_ptr<CUevent_st>;
using EvPool = std::shared_ptr<std::vector<cudaEvent_t>>;

// A released slice whose bytes a pending swap-in may still be reading.
struct Fence {
  uint64_t off, len;
  EvRef ev;
  cudaStream_t stream;   // where `ev` was recorded; no_stream() if unknown / a graph
};
// Fence::stream of a fence that must always be waited on.
inline cudaStream_t no_stream() { return reinterpret_cast<cudaStream_t>(~uintptr_t(0)); }

// This source's partition of one peer's stash pool (R21).
struct Partition {
  uint8_t* base = nullptr;            // local VA of the partition start
  uint64_t size = 0;
  std::map<uint64_t, uint64_t> free;  // first-fit free list: offset -> length
  std::deque<Fence> fences;           // in release order (oldest first)
};

// The options a swap launch runs with (mpress_set_option's swap keys): the
// context's, or an executor's own copy (mpress_executor_set_option).
struct SwapOpts {
  int path = MPRESS_PATH_AUTO;
  int max_ctas = 0;
  int variant = MPRESS_VARIANT_AUTO;
  int order = MPRESS_ORDER_INTERLEAVE;
  int pdl = 1;                        // MPRESS_OPT_PDL
  uint64_t pace_mbps = 0;             // MPRESS_OPT_PACE_MBPS (0 = unpaced)
  int split = MPRESS_SPLIT_AUTO;      // MPRESS_OPT_SPLIT
};
// Set one swap option (validated); kNotSwapOption if `key` is not one.
constexpr int kNotSwapOption = 1;
int set_swap_option(SwapOpts* o, int key, int64_t value);
int get_swap_option(const SwapOpts& o, int key, int64_t* value);  // kNotSwapOption if not one

}  // namespace mpress

struct mpress_handle_s;

struct mpress_ctx_s {
  int device = -1;
  int world = 0;
  int source = 0;                     // this context's rank = the exporter it serves
  bool local = false;                 // mpress_init_local
  mpress_exchange_fn exchange = nullptr;
  void* exchange_user = nullptr;
  std::vector<uint64_t> partition;    // [world*world]
  mpress::Mapping own;                // multi-process: this rank's exported pool
  std::vector<mpress::Mapping> maps;  // [world] pool mappings used by this source
  std::vector<mpress::Partition> parts;  // [world]
  mpress::SwapOpts opt;               // the swap options (mpress_set_option)
  int last_path = -1;                 // path the last swap call ran (MPRESS_OPT_LAST_PATH)
  bool host_peer = false;             // a peer pool is pinned host memory (NEXT-4)
  // SM path MPRESS_PATH_AUTO takes for an uncapped grid, per direction
  // (kDirOut, kDirIn) and size class (a launch moving < MPRESS_AUTO_SMALL_BYTES,
  // or more); until mpress_autotune measures otherwise: direct for small
  // launches, bulk for large ones (profiles/r01/sweep_sizes_v2.jsonl)
  int auto_path[2][2] = {{MPRESS_PATH_DIRECT, MPRESS_PATH_BULK}, {MPRESS_PATH_DIRECT, MPRESS_PATH_BULK}};
  int transport = MPRESS_TRANSPORT_LOCAL;
  int last_launches = 0;
  std::vector<cudaStream_t> ce_streams;  // copy-engine comparator, one per peer
  mpress::TableRing* ring = nullptr;  // device-resident tables of large launches (lazy)
  mpress::CounterRing* counters = nullptr;  // MPRESS_SPLIT_DYNAMIC claim counters (lazy)
  mpress::EvPool ev_pool = std::make_shared<std::vector<cudaEvent_t>>();
  std::set<mpress_handle_s*> handles;
  std::vector<mpress::CopyDesc> scratch_desc;  // per-call buffers, reused
  std::vector<int> scratch_peer;
  std::mutex mu;
};

struct mpress_handle_s {
  mpress_ctx_s* ctx = nullptr;
  int state = 0;
  std::vector<mpress_stripe> stripes;
  uint32_t n_tensors = 0;
  std::vector<uint64_t> slice_off;    // [world], UINT64_MAX if unused
  std::vector<uint64_t> slice_len;    // [world]
  mpress::EvRef out_done;
  mpress::EvRef in_done;
  cudaStream_t out_stream = nullptr;  // the swap-out's stream (a swap-in there needs no wait)
  bool slices_held = false;
  // Graph handle: the swap-out was enqueued while its stream was being
  // captured into a CUDA graph.  Every replay re-runs the captured kernels
  // into the same slices, so the slices stay held until mpress_handle_free.
  // out_done / in_done are capture-internal (joins inside the capture);
  // out_ext / in_ext are external event-record nodes, re-recorded by every
  // replay, which queries, eager waits and slice fences use.
  bool graph = false;
  mpress::EvRef out_ext;
  mpress::EvRef in_ext;
};

namespace mpress {
// A pooled CUDA event (disable-timing) owned by reference; sched.cpp.
EvRef take_event(mpress_ctx_s* c);
// mpress_swap_out / mpress_swap_in with explicit options (the executor's);
// sched.cpp.  The public calls pass the context's options.
int swap_out_with(mpress_ctx_s* c, const SwapOpts& o, const mpress_plan_t* plan, void* const* tensors,
                  void* stream, void* after, mpress_handle_t** out);
int swap_in_with(mpress_ctx_s* c, const SwapOpts& o, mpress_handle_t* h, void* const* dst, void* stream);
}  // namespace mpress
