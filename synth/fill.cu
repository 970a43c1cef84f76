// GPU twin of synth/gen.py: the counter-based input generator (no method
// arithmetic).  Byte b of tensor t under seed s is byte (b % 8) of
// splitmix64(s ^ (t << 40) ^ (b / 8)), little-endian.  Used to fill GB-scale
// inputs on the device and to check round trips against the generator
// without host copies.  Built separately into synth/libsynth.so; shares no
// code with libmpress.
#include <cuda_runtime.h>
#include <stdint.h>

namespace {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

// Bytes [start, start+n) of tensor `key` into dst (dst[0] = byte `start`).
__global__ void fill_kernel(uint8_t* dst, uint64_t n, uint64_t key, uint64_t start) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  const uint64_t w_first = start >> 3;
  const uint64_t w_last = (start + n + 7) >> 3;
  for (uint64_t w = w_first + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < w_last; w += stride) {
    const uint64_t v = splitmix64(key ^ w);
    const uint64_t b0 = w << 3;
    if (b0 >= start && b0 + 8 <= start + n && (((uintptr_t)(dst + (b0 - start))) & 7) == 0) {
      *reinterpret_cast<uint64_t*>(dst + (b0 - start)) = v;
    } else {
      for (int k = 0; k < 8; ++k) {
        const uint64_t b = b0 + k;
        if (b >= start && b < start + n) dst[b - start] = (uint8_t)(v >> (8 * k));
      }
    }
  }
}

// Count bytes of buf (bytes [start, start+n) of tensor `key`) that differ.
__global__ void check_kernel(const uint8_t* buf, uint64_t n, uint64_t key, uint64_t start,
                             unsigned long long* bad) {
  const uint64_t stride = (uint64_t)gridDim.x * blockDim.x;
  unsigned long long local = 0;
  const uint64_t w_first = start >> 3;
  const uint64_t w_last = (start + n + 7) >> 3;
  for (uint64_t w = w_first + blockIdx.x * (uint64_t)blockDim.x + threadIdx.x; w < w_last; w += stride) {
    const uint64_t v = splitmix64(key ^ w);
    for (int k = 0; k < 8; ++k) {
      const uint64_t b = (w << 3) + k;
      if (b >= start && b < start + n) local += buf[b - start] != (uint8_t)(v >> (8 * k));
    }
  }
  if (local) atomicAdd(bad, local);
}

uint64_t key_of(uint64_t seed, uint64_t tensor_id) { return seed ^ (tensor_id << 40); }

}  // namespace

extern "C" int synth_fill(void* dst, uint64_t n, uint64_t seed, uint64_t tensor_id,
                          uint64_t start, void* stream) {
  if (n == 0) return 0;
  fill_kernel<<<1184, 256, 0, (cudaStream_t)stream>>>((uint8_t*)dst, n, key_of(seed, tensor_id), start);
  return (int)cudaGetLastError();
}

// Returns the number of mismatching bytes (synchronous), or -1 on error.
extern "C" long long synth_check(const void* buf, uint64_t n, uint64_t seed, uint64_t tensor_id,
                                 uint64_t start, void* stream) {
  if (n == 0) return 0;
  unsigned long long* d_bad = nullptr;
  unsigned long long h_bad = 0;
  if (cudaMalloc(&d_bad, sizeof *d_bad) != cudaSuccess) return -1;
  cudaMemsetAsync(d_bad, 0, sizeof *d_bad, (cudaStream_t)stream);
  check_kernel<<<1184, 256, 0, (cudaStream_t)stream>>>((const uint8_t*)buf, n, key_of(seed, tensor_id), start, d_bad);
  cudaMemcpyAsync(&h_bad, d_bad, sizeof h_bad, cudaMemcpyDeviceToHost, (cudaStream_t)stream);
  cudaError_t e = cudaStreamSynchronize((cudaStream_t)stream);
  cudaFree(d_bad);
  return e == cudaSuccess ? (long long)h_bad : -1;
}

// ---- pipeline-replay helpers (tools/replay_1f1b.py) -------------------------
// A replayed stage must wait for the other (absent) pipeline stages: stamp a
// base time on the device, then gate each op until %globaltimer reaches
// base + offset.  No method arithmetic.
namespace {
__device__ __forceinline__ unsigned long long gtimer() {
  unsigned long long t;
  asm volatile("mov.u64 %0, %%globaltimer;" : "=l"(t));
  return t;
}
__global__ void stamp_kernel(unsigned long long* base) { *base = gtimer(); }
__global__ void gate_kernel(const unsigned long long* base, unsigned long long offset) {
  const unsigned long long until = *base + offset;
  while (gtimer() < until) __nanosleep(500);
}
}  // namespace

extern "C" int synth_stamp(void* base, void* stream) {
  stamp_kernel<<<1, 1, 0, (cudaStream_t)stream>>>((unsigned long long*)base);
  return (int)cudaGetLastError();
}

extern "C" int synth_gate(const void* base, uint64_t offset_ns, void* stream) {
  gate_kernel<<<1, 1, 0, (cudaStream_t)stream>>>((const unsigned long long*)base, offset_ns);
  return (int)cudaGetLastError();
}
