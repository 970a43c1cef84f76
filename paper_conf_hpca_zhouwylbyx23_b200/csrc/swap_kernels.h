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
constexpr int kDirectVariants = 10;      // MPRESS_OPT_VARIANT range, direct path
constexpr int kBulkVariants = 7;         // MPRESS_OPT_VARIANT range, bulk path
constexpr int kCeVariants = 2;           // copy engines: 0 per-peer streams, 1 one batch call

enum CopyDir { kDirOut = 0, kDirIn = 1 };

// Enqueue kernels moving every descriptor on `stream`; `path` is
// MPRESS_PATH_DIRECT or MPRESS_PATH_BULK, `variant` its kernel shape;
// `max_ctas` caps the grid (0 = the variant's default grid); `pdl_mode`
// (MPRESS_OPT_PDL: 0 never, 1 uncapped grids only, 2 always) launches with
// programmatic stream serialization.  Adds the number
// of kernel launches to *launches.  Returns MPRESS_OK or MPRESS_ERR_*.
int launch_copy(int path, int variant, int dir, const CopyDesc* d, const int* group, size_t n,
                int max_ctas, int pdl_mode,
                cudaStream_t stream, int* launches);

// Default grid of a path/variant on the current device (SMs x CTAs per SM).
int copy_wave_ctas(int path, int variant);

// Load every swap kernel on the current device (no lazy-loading stall later).
int preload_kernels();

}  // namespace mpress
