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

enum CopyDir { kDirOut = 0, kDirIn = 1 };

// Enqueue kernels moving every descriptor on `stream`; `path` is
// MPRESS_PATH_DIRECT or MPRESS_PATH_BULK; `max_ctas` caps the grid (0 = one
// full wave).  Adds the number of kernel launches to *launches.
// Returns MPRESS_OK or MPRESS_ERR_CUDA (message set).
int launch_copy(int path, int dir, const CopyDesc* d, size_t n, int max_ctas,
                cudaStream_t stream, int* launches);

// CTAs of the given path that fit on one wave of the current device.
int copy_wave_ctas(int path);

}  // namespace mpress
