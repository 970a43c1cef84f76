// The swap executor of the paper's runtime ("the executor executes the
// memory saving operators (i.e., swap-out ...) ... and state recovering ones
// (i.e., swap-in ...)"), for the exporter stage of a 1F1B pipeline.
//
// The caller runs its own compute ops in 1F1B order on its compute stream and
// brackets each op j with mpress_executor_before / _after; the executor
//   * after F(m): enqueues the swap-out of m's activations on the swap-out
//     stream, ordered after F(m) by an event on the compute stream;
//   * after the trigger op of a swap-in (mpress_schedule_1f1b: the last op
//     that still leaves the swap-in time before B(m)): enqueues the swap-in of
//     m on the swap-in stream into the buffers registered for m;
//   * before B(m): makes the compute stream wait for that swap-in.
// Everything is enqueue-only (no blocking of the main thread).
#include <initializer_list>
#include <new>
#include <vector>

#include "ctx.h"

struct mpress_executor_s {
  mpress_ctx_s* ctx = nullptr;
  const mpress_plan_t* plan = nullptr;
  cudaStream_t out_stream = nullptr, in_stream = nullptr;
  uint32_t n_tensors = 0;
  std::vector<int> kind, mb;                 // per op: 0 = F, 1 = B; its micro-batch
  std::vector<std::vector<uint32_t>> trig;   // per op: micro-batches whose swap-in it triggers
  std::vector<mpress_handle_t*> handle;      // per micro-batch
  std::vector<std::vector<void*>> restore;   // per micro-batch: destination pointers
  std::vector<mpress_1f1b_slot> slots;
  // the options of this executor's swaps: the context's at creation, then
  // mpress_executor_set_option (a stage picks its transfer path: the NEXT-2
  // replay found no one path best for every stage)
  mpress::SwapOpts opt;
};

using namespace mpress;

extern "C" int mpress_executor_create(mpress_ctx_t* ctx, const mpress_plan_t* plan,
                                      const mpress_1f1b_params* params, void* out_stream, void* in_stream,
                                      mpress_executor_t** out) {
  if (!ctx || !plan || !params || !out) return fail(MPRESS_ERR_ARG, "mpress_executor_create: null argument");
  *out = nullptr;
  mpress_plan_info info;
  MP_TRY(mpress_plan_get_info(plan, &info));
  if (info.source != ctx->source || info.world != ctx->world)
    return fail(MPRESS_ERR_PEER, "mpress_executor_create: plan is not for this context's source");
  const uint32_t M = params->micro_batches;
  auto* x = new (std::nothrow) mpress_executor_s();
  if (!x) return fail(MPRESS_ERR_ARG, "mpress_executor_create: out of host memory");
  try {
    x->slots.resize(M ? M : 1);
    int rc = mpress_schedule_1f1b(params, x->slots.data(), nullptr);
    if (rc != MPRESS_OK) {
      delete x;
      return rc;
    }
    x->ctx = ctx;
    {
      std::lock_guard<std::mutex> lk(ctx->mu);
      x->opt = ctx->opt;
    }
    x->plan = plan;
    x->out_stream = static_cast<cudaStream_t>(out_stream);
    x->in_stream = static_cast<cudaStream_t>(in_stream);
    x->n_tensors = info.n_tensors;
    // the exporter stage's ops in 1F1B order (same rule as the scheduler)
    const uint32_t S = params->stages, e = params->stage;
    const uint32_t W = (S - 1 - e) < M ? (S - 1 - e) : M;
    for (uint32_t m = 0; m < W; ++m) { x->kind.push_back(0); x->mb.push_back((int)m); }
    for (uint32_t i = 0; i < M; ++i) {
      if (W + i < M) { x->kind.push_back(0); x->mb.push_back((int)(W + i)); }
      x->kind.push_back(1);
      x->mb.push_back((int)i);
    }
    x->trig.assign(x->kind.size(), {});
    for (uint32_t m = 0; m < M; ++m) x->trig[x->slots[m].in_trigger].push_back(m);
    x->handle.assign(M, nullptr);
    x->restore.assign(M, {});
  } catch (const std::bad_alloc&) {
    delete x;
    return fail(MPRESS_ERR_ARG, "mpress_executor_create: out of host memory");
  }
  *out = x;
  return MPRESS_OK;
}

extern "C" int mpress_executor_restore_to(mpress_executor_t* x, uint32_t micro_batch, void* const* dst) {
  if (!x || !dst || micro_batch >= x->handle.size())
    return fail(MPRESS_ERR_ARG, "mpress_executor_restore_to: bad argument");
  x->restore[micro_batch].assign(dst, dst + x->n_tensors);
  return MPRESS_OK;
}

namespace {
// The executor frees each micro-batch's handle at its backward and reuses the
// slices for later micro-batches; under graph capture those slices would be
// handed back to eager swaps while the graph still replays into them, so an
// executor step is not capturable (capture individual swap pairs instead).
bool any_capturing(std::initializer_list<cudaStream_t> ss) {
  for (cudaStream_t s : ss) {
    cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
    if (cudaStreamIsCapturing(s, &st) != cudaSuccess) {
      cudaGetLastError();
      continue;
    }
    if (st != cudaStreamCaptureStatusNone) return true;
  }
  return false;
}
}  // namespace

extern "C" int mpress_executor_before(mpress_executor_t* x, uint32_t op, void* compute_stream, uint32_t* kind,
                                      uint32_t* micro_batch) {
  if (!x || op >= x->kind.size()) return fail(MPRESS_ERR_ARG, "mpress_executor_before: bad op");
  if (any_capturing({static_cast<cudaStream_t>(compute_stream), x->out_stream, x->in_stream}))
    return fail(MPRESS_ERR_STATE, "mpress_executor_before: executor steps cannot be captured into a CUDA graph");
  const int m = x->mb[op];
  if (kind) *kind = (uint32_t)x->kind[op];
  if (micro_batch) *micro_batch = (uint32_t)m;
  if (x->kind[op] == 1) {  // B(m): its activations must be back
    mpress_handle_t* h = x->handle[m];
    if (!h) return fail(MPRESS_ERR_STATE, "mpress_executor_before: micro-batch %d was never swapped out", m);
    MP_TRY(mpress_wait(x->ctx, h, compute_stream));
    // the wait is enqueued; the handle's events live on in the fences
    MP_TRY(mpress_handle_free(x->ctx, h, 0));
    x->handle[m] = nullptr;
  }
  return MPRESS_OK;
}

extern "C" int mpress_executor_after(mpress_executor_t* x, uint32_t op, void* compute_stream,
                                     void* const* activations) {
  if (!x || op >= x->kind.size()) return fail(MPRESS_ERR_ARG, "mpress_executor_after: bad op");
  if (any_capturing({static_cast<cudaStream_t>(compute_stream), x->out_stream, x->in_stream}))
    return fail(MPRESS_ERR_STATE, "mpress_executor_after: executor steps cannot be captured into a CUDA graph");
  mpress_ctx_s* c = x->ctx;
  DeviceGuard g(c->device);
  EvRef done = take_event(c);
  if (!done) return fail(MPRESS_ERR_CUDA, "cudaEventCreate failed");
  cudaError_t e = cudaEventRecord(done.get(), static_cast<cudaStream_t>(compute_stream));
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "cudaEventRecord: %s", cudaGetErrorString(e));
  // `done` may go back to the pool when this call returns: the swap-out's
  // and swap-in stream's waits below captured its record already
  const int m = x->mb[op];
  if (x->kind[op] == 0) {  // F(m) produced the activations: swap them out
    if (!activations) return fail(MPRESS_ERR_ARG, "mpress_executor_after: F(%d) needs its activations", m);
    if (x->handle[m]) return fail(MPRESS_ERR_STATE, "mpress_executor_after: micro-batch %d already out", m);
    MP_TRY(swap_out_with(c, x->opt, x->plan, activations, x->out_stream, done.get(), &x->handle[m]));
  }
  for (uint32_t mm : x->trig[op]) {  // swap-ins issued as late as still hidden
    if (!x->handle[mm]) return fail(MPRESS_ERR_STATE, "mpress_executor_after: micro-batch %u not swapped out", mm);
    if (x->restore[mm].size() != x->n_tensors)
      return fail(MPRESS_ERR_STATE, "mpress_executor_after: no restore buffers for micro-batch %u", mm);
    e = cudaStreamWaitEvent(x->in_stream, done.get(), 0);
    if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "cudaStreamWaitEvent: %s", cudaGetErrorString(e));
    MP_TRY(swap_in_with(c, x->opt, x->handle[mm], x->restore[mm].data(), x->in_stream));
  }
  return MPRESS_OK;
}

extern "C" int mpress_executor_release(mpress_executor_t* x, uint32_t micro_batch, void* stream) {
  if (!x || micro_batch >= x->handle.size()) return fail(MPRESS_ERR_ARG, "mpress_executor_release: bad argument");
  mpress_handle_t* h = x->handle[micro_batch];
  if (!h || !h->out_done)
    return fail(MPRESS_ERR_STATE, "mpress_executor_release: micro-batch %u is not swapped out", micro_batch);
  DeviceGuard g(x->ctx->device);
  const cudaError_t e = cudaStreamWaitEvent(static_cast<cudaStream_t>(stream), h->out_done.get(), 0);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "mpress_executor_release: %s", cudaGetErrorString(e));
  return MPRESS_OK;
}

extern "C" int mpress_executor_set_option(mpress_executor_t* x, int key, int64_t value) {
  if (!x) return fail(MPRESS_ERR_ARG, "mpress_executor_set_option: null executor");
  const int rc = set_swap_option(&x->opt, key, value);
  return rc == kNotSwapOption ? fail(MPRESS_ERR_ARG, "option %d is not a swap option", key) : rc;
}

extern "C" int mpress_executor_get_option(const mpress_executor_t* x, int key, int64_t* value) {
  if (!x || !value) return fail(MPRESS_ERR_ARG, "mpress_executor_get_option: null argument");
  const int rc = get_swap_option(x->opt, key, value);
  return rc == kNotSwapOption ? fail(MPRESS_ERR_ARG, "option %d is not a swap option", key) : rc;
}

extern "C" int mpress_executor_slot(const mpress_executor_t* x, uint32_t micro_batch, mpress_1f1b_slot* slot) {
  if (!x || !slot || micro_batch >= x->slots.size())
    return fail(MPRESS_ERR_ARG, "mpress_executor_slot: bad argument");
  *slot = x->slots[micro_batch];
  return MPRESS_OK;
}

extern "C" int mpress_executor_ops(const mpress_executor_t* x) {
  return x ? (int)x->kind.size() : fail(MPRESS_ERR_ARG, "mpress_executor_ops: null");
}

extern "C" int mpress_executor_free(mpress_executor_t* x) {
  if (!x) return MPRESS_OK;
  for (auto* h : x->handle)
    if (h) mpress_handle_free(x->ctx, h, 1);
  delete x;
  return MPRESS_OK;
}
