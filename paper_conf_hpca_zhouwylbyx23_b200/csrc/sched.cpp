// Event-driven swap scheduler: handles = the
// paper's D2D metadata table ("number of sub-blocks, the sizes of each
// sub-block, and the indices of target GPU devices ... recorded before the
// execution of the swap-out operator ... used to guide the execution of the
// latter swap-in operator and updated when it completes"), stash-slice
// allocation inside the source's partition (R21), and completion events.
//
// The paper runs swap-out and swap-in on two executor threads with their own
// CUDA streams so launches and status checks never block the main thread
// (P:236).  Here the caller's side streams carry the kernels and CUDA
// events carry completion: every call only enqueues work, and
// mpress_wait / mpress_query are enqueue-only / non-blocking, so no helper
// thread is needed.
//
// Host cost per call is kept small (a swap of a few KiB is latency-bound by
// the host): events are pooled and shared by reference between a handle and
// the fences of its slices, fences are reaped oldest-first, and descriptor
// buffers are reused.
#include <algorithm>

#include "ctx.h"
#include "hostprof.h"
#include "swap_kernels.h"

namespace mpress {

EvRef take_event(mpress_ctx_s* c) {
  cudaEvent_t e = nullptr;
  EvPool pool = c->ev_pool;
  if (!pool->empty()) {
    e = pool->back();
    pool->pop_back();
  } else if (cudaEventCreateWithFlags(&e, cudaEventDisableTiming) != cudaSuccess) {
    return EvRef();
  }
  return EvRef(e, [pool](CUevent_st* ev) { pool->push_back(ev); });
}

namespace {

// Fence lists are reaped only past this length: a fence recorded on the
// stream of the next swap-out costs nothing (stream order covers it), so the
// event queries of a reap are spent only when the list grows.
constexpr size_t kReapAt = 32;

// Can work enqueued on `s` rely on plain stream order after work enqueued on
// `prev`?  Not for the per-thread default stream (one handle value, one stream
// per thread) or unknown streams.
bool same_stream(cudaStream_t prev, cudaStream_t s) {
  return prev == s && s != cudaStreamPerThread && s != no_stream();
}

// Drop the fences whose swap-in has completed (oldest first; stops at the
// first one still pending, so the cost is O(1) amortised).
void reap_fences(Partition* part) {
  auto& f = part->fences;
  while (!f.empty()) {
    const cudaError_t r = cudaEventQuery(f.front().ev.get());
    if (r != cudaSuccess) {
      if (r == cudaErrorNotReady) cudaGetLastError();  // not sticky; clear it
      break;
    }
    f.pop_front();
  }
}

// First fit, lowest address.
bool alloc_slice(Partition* part, uint64_t len, uint64_t* off) {
  for (auto it = part->free.begin(); it != part->free.end(); ++it) {
    if (it->second >= len) {
      *off = it->first;
      const uint64_t rest = it->second - len, roff = it->first + len;
      part->free.erase(it);
      if (rest) part->free[roff] = rest;
      return true;
    }
  }
  return false;
}

void free_slice(Partition* part, uint64_t off, uint64_t len) {
  auto next = part->free.lower_bound(off);
  if (next != part->free.end() && off + len == next->first) {  // merge right
    len += next->second;
    next = part->free.erase(next);
  }
  if (next != part->free.begin()) {  // merge left
    auto prev = std::prev(next);
    if (prev->first + prev->second == off) {
      prev->second += len;
      return;
    }
  }
  part->free[off] = len;
}

int check_ptrs(void* const* p, size_t n, const char* what) {
  if (!p) return fail(MPRESS_ERR_ARG, "%s: null pointer array", what);
  for (size_t i = 0; i < n; ++i) {
    if (!p[i]) return fail(MPRESS_ERR_ARG, "%s: pointer %zu is null", what, i);
    if (reinterpret_cast<uintptr_t>(p[i]) & 15)
      return fail(MPRESS_ERR_ALIGN, "%s: pointer %zu (%p) is not 16-byte aligned", what, i, p[i]);
  }
  return MPRESS_OK;
}

int cuda_fail(cudaError_t e, const char* what) {
  return fail(MPRESS_ERR_CUDA, "%s: %s", what, cudaGetErrorString(e));
}

// Is `s` being captured into a CUDA graph (cudaStreamBeginCapture /
// torch.cuda.graph)?  Capture changes what an enqueue-only call may do: no
// event queries (they are not allowed while a global-mode capture runs), and
// events from outside the capture are waited on as external nodes.
bool capturing(cudaStream_t s) {
  cudaStreamCaptureStatus st = cudaStreamCaptureStatusNone;
  if (cudaStreamIsCapturing(s, &st) != cudaSuccess) {
    cudaGetLastError();
    return false;
  }
  return st == cudaStreamCaptureStatusActive;
}

// Record `ev` on `s`; under capture first record `ext` as an external
// event-record node (re-recorded by every replay of the graph).  The
// external node goes first so that a join on `ev` also joins it: a node after
// the last join would be work the capture never rejoins.
int record_done(mpress_ctx_s* c, cudaStream_t s, bool graph, EvRef* ev, EvRef* ext, const char* what) {
  if (graph) {
    *ext = take_event(c);
    if (!*ext) return fail(MPRESS_ERR_CUDA, "cudaEventCreate failed");
    const cudaError_t e = cudaEventRecordWithFlags(ext->get(), s, cudaEventRecordExternal);
    if (e != cudaSuccess) return cuda_fail(e, what);
  }
  *ev = take_event(c);
  if (!*ev) return fail(MPRESS_ERR_CUDA, "cudaEventCreate failed");
  const cudaError_t e = cudaEventRecord(ev->get(), s);
  return e == cudaSuccess ? MPRESS_OK : cuda_fail(e, what);
}

// Move every descriptor on `stream` with the context's path.
int run_copy(mpress_ctx_s* c, const SwapOpts& o, int dir, const std::vector<CopyDesc>& d,
             const std::vector<int>& desc_peer, cudaStream_t stream, bool graph) {
  c->last_launches = 0;
  int path = o.path;
  if (path == MPRESS_PATH_AUTO) {
    // full grid: per direction and size class, the kernel mpress_autotune
    // measured faster on this context's links (before it runs: direct below
    // MPRESS_AUTO_SMALL_BYTES, bulk above -- TMA, +0.8% on B200 loopback);
    // direct when the grid is capped to <= one CTA per SM (small CTAs that
    // co-reside with a GEMM) or the launch mixes device peers and pinned
    // host pools; the copy engines when every stripe goes to a host pool
    // (over PCIe every SM kernel shape stops at ~52.6 GB/s, the engines at
    // ~56.9: profiles/r02/sweep_host_paths.jsonl)
    const int sms = sm_count(nullptr);
    const bool capped = o.max_ctas > 0 && o.max_ctas <= sms;
    uint64_t total = 0;
    for (const CopyDesc& x : d) total += x.len;
    int host = 0;
    if (c->host_peer)
      for (int p : desc_peer) host += c->maps[p].host != nullptr;
    if (host && host == (int)desc_peer.size())
      path = MPRESS_PATH_CE;
    else
      path = (capped || host) ? MPRESS_PATH_DIRECT : c->auto_path[dir][total >= MPRESS_AUTO_SMALL_BYTES];
  }
  c->last_path = path;
  if (path != MPRESS_PATH_CE) {
    // Large tables live in device memory (TableRing), except under graph
    // capture: a replay would re-read a staging slot later launches reused.
    if (!graph && d.size() > (size_t)kParamDescMax && !c->ring) MP_TRY(table_ring_create(c->device, &c->ring));
    // Claim counters likewise: a replayed launch would reuse a slot that
    // later eager launches take (dynamic falls back to blocked there).
    if (!graph && o.split >= MPRESS_SPLIT_DYNAMIC && !c->counters)
      MP_TRY(counter_ring_create(c->device, &c->counters));
    return launch_copy(path, o.variant, dir, d.data(),
                       o.order == MPRESS_ORDER_INTERLEAVE ? desc_peer.data() : nullptr, d.size(), o.max_ctas,
                       o.pdl, stream, &c->last_launches, graph ? nullptr : c->ring, o.pace_mbps, o.split,
                       graph ? nullptr : c->counters);
  }

  // Copy-engine comparator (the prior-art mechanism):
  // one cudaMemcpyAsync per stripe, one side stream per peer so the engines of
  // different peers overlap; fork/join by events.
  if (c->ce_streams.empty()) {
    c->ce_streams.assign(c->world, nullptr);
    for (int p = 0; p < c->world; ++p) {
      cudaError_t e = cudaStreamCreateWithFlags(&c->ce_streams[p], cudaStreamNonBlocking);
      if (e != cudaSuccess) return cuda_fail(e, "cudaStreamCreate (copy-engine path)");
    }
  }
  EvRef fork = take_event(c);
  if (!fork) return fail(MPRESS_ERR_CUDA, "cudaEventCreate failed");
  cudaEventRecord(fork.get(), stream);
  std::vector<char> used(c->world, 0);
  for (int p : desc_peer) used[p] = 1;
  for (int p = 0; p < c->world; ++p) {
    if (!used[p]) continue;
    cudaStream_t s = c->ce_streams[p];
    cudaStreamWaitEvent(s, fork.get(), 0);
    for (size_t i = 0; i < d.size(); ++i) {
      if (desc_peer[i] != p) continue;
      cudaError_t e = cudaMemcpyAsync(d[i].dst, d[i].src, d[i].len, cudaMemcpyDefault, s);
      if (e != cudaSuccess) return cuda_fail(e, "cudaMemcpyAsync (copy-engine path)");
    }
    EvRef join = take_event(c);
    if (!join) return fail(MPRESS_ERR_CUDA, "cudaEventCreate failed");
    cudaEventRecord(join.get(), s);
    cudaStreamWaitEvent(stream, join.get(), 0);
  }  // the events may be re-recorded once the waits above are enqueued
  return MPRESS_OK;
}

}  // namespace
}  // namespace mpress

using namespace mpress;

namespace {
int swap_out_locked(mpress_ctx_s* c, const SwapOpts& o, const mpress_plan_t* plan_, void* const* tensors,
                    void* stream_, void* after, mpress_handle_t** out);
}  // namespace

extern "C" int mpress_swap_out(mpress_ctx_t* c, const mpress_plan_t* plan_, void* const* tensors,
                               void* stream_, void* after, mpress_handle_t** out) {
  if (!c || !plan_ || !out) return fail(MPRESS_ERR_ARG, "mpress_swap_out: null argument");
  std::lock_guard<std::mutex> lk(c->mu);
  return swap_out_locked(c, c->opt, plan_, tensors, stream_, after, out);
}

namespace mpress {
int swap_out_with(mpress_ctx_s* c, const SwapOpts& o, const mpress_plan_t* plan_, void* const* tensors,
                  void* stream_, void* after, mpress_handle_t** out) {
  if (!c || !plan_ || !out) return fail(MPRESS_ERR_ARG, "mpress_swap_out: null argument");
  std::lock_guard<std::mutex> lk(c->mu);
  return swap_out_locked(c, o, plan_, tensors, stream_, after, out);
}
}  // namespace mpress

namespace {
int swap_out_locked(mpress_ctx_s* c, const SwapOpts& o, const mpress_plan_t* plan_, void* const* tensors,
                    void* stream_, void* after, mpress_handle_t** out) {
  HP_START();
  *out = nullptr;
  const uint64_t *units, *peer_bytes;
  const mpress_stripe* st;
  uint32_t n_st;
  mpress_plan_info info;
  MP_TRY(mpress_plan_get_info(plan_, &info));
  MP_TRY(mpress_plan_units(plan_, &units));
  MP_TRY(mpress_plan_stripes(plan_, &st, &n_st, &peer_bytes));
  if (info.world != c->world || info.source != c->source)
    return fail(MPRESS_ERR_PEER, "mpress_swap_out: plan is for source %d of %d, context serves %d of %d",
                info.source, info.world, c->source, c->world);
  MP_TRY(check_ptrs(tensors, info.n_tensors, "mpress_swap_out(tensors)"));
  DeviceGuard g(c->device);
  cudaStream_t stream = static_cast<cudaStream_t>(stream_);
  const bool graph = capturing(stream);
  HP_LAP(0, "out: plan/ptrs/capture query");

  auto* h = new mpress_handle_s();
  h->ctx = c;
  h->graph = graph;
  h->slice_off.assign(c->world, UINT64_MAX);
  h->slice_len.assign(c->world, 0);
  int rc = MPRESS_OK;
  for (int p = 0; p < c->world && rc == MPRESS_OK; ++p) {
    if (units[p] == 0) continue;
    Partition& part = c->parts[p];
    if (!part.base) {
      rc = fail(MPRESS_ERR_PEER, "mpress_swap_out: peer %d is not mapped (partition 0)", p);
      break;
    }
    if (!graph && part.fences.size() > kReapAt) reap_fences(&part);
    const uint64_t len = units[p] * info.granule;
    uint64_t off;
    if (!alloc_slice(&part, len, &off)) {
      rc = fail(MPRESS_ERR_NO_SPACE, "mpress_swap_out: no %llu-byte slice left in the partition on peer %d",
                (unsigned long long)len, p);
      break;
    }
    h->slice_off[p] = off;
    h->slice_len[p] = len;
    // earlier swap-ins still reading these bytes: order this swap-out after
    // them -- free when they ran on this stream; under capture the waits
    // become external wait nodes (every replay waits for the fence's latest
    // record)
    for (const Fence& f : part.fences)
      if (f.off < off + len && off < f.off + f.len && (graph || !same_stream(f.stream, stream)))
        cudaStreamWaitEvent(stream, f.ev.get(), graph ? cudaEventWaitExternal : 0);
  }
  if (rc != MPRESS_OK) {
    for (int p = 0; p < c->world; ++p)
      if (h->slice_off[p] != UINT64_MAX) free_slice(&c->parts[p], h->slice_off[p], h->slice_len[p]);
    delete h;
    return rc;
  }
  HP_LAP(1, "out: handle + slices + fences");
  h->slices_held = true;
  h->stripes.assign(st, st + n_st);
  h->n_tensors = info.n_tensors;

  std::vector<CopyDesc>& d = c->scratch_desc;
  std::vector<int>& dp = c->scratch_peer;
  d.resize(n_st);
  dp.resize(n_st);
  for (uint32_t i = 0; i < n_st; ++i) {
    const mpress_stripe& s = st[i];
    d[i].src = static_cast<const uint8_t*>(tensors[s.tensor]) + s.src_off;
    d[i].dst = c->parts[s.peer].base + h->slice_off[s.peer] + s.dst_off;
    d[i].len = s.len;
    dp[i] = (int)s.peer;
  }
  if (after) cudaStreamWaitEvent(stream, static_cast<cudaEvent_t>(after), 0);
  HP_LAP(2, "out: descriptors");
  rc = run_copy(c, o, kDirOut, d, dp, stream, graph);
  HP_LAP(3, "out: run_copy (launch)");
  if (rc == MPRESS_OK) rc = record_done(c, stream, graph, &h->out_done, &h->out_ext, "cudaEventRecord(out_done)");
  HP_LAP(4, "out: event record");
  if (rc != MPRESS_OK) {
    // Kernels may already be queued: keep the slices fenced by a sync (a
    // failed capture is invalidated anyway: nothing was enqueued for real).
    if (!graph) cudaStreamSynchronize(stream);
    for (int p = 0; p < c->world; ++p)
      if (h->slice_off[p] != UINT64_MAX) free_slice(&c->parts[p], h->slice_off[p], h->slice_len[p]);
    delete h;
    return rc;
  }
  h->state = MPRESS_STATE_OUT_PENDING;
  h->out_stream = graph ? no_stream() : stream;
  c->handles.insert(h);
  *out = h;
  return MPRESS_OK;
}

int swap_in_locked(mpress_ctx_s* c, const SwapOpts& o, mpress_handle_t* h, void* const* dst, void* stream_);
}  // namespace

extern "C" int mpress_swap_in(mpress_ctx_t* c, mpress_handle_t* h, void* const* dst, void* stream_) {
  if (!c || !h) return fail(MPRESS_ERR_ARG, "mpress_swap_in: null argument");
  std::lock_guard<std::mutex> lk(c->mu);
  return swap_in_locked(c, c->opt, h, dst, stream_);
}

namespace mpress {
int swap_in_with(mpress_ctx_s* c, const SwapOpts& o, mpress_handle_t* h, void* const* dst, void* stream_) {
  if (!c || !h) return fail(MPRESS_ERR_ARG, "mpress_swap_in: null argument");
  std::lock_guard<std::mutex> lk(c->mu);
  return swap_in_locked(c, o, h, dst, stream_);
}
}  // namespace mpress

namespace {
int swap_in_locked(mpress_ctx_s* c, const SwapOpts& o, mpress_handle_t* h, void* const* dst, void* stream_) {
  HP_START();
  if (h->ctx != c || !c->handles.count(h)) return fail(MPRESS_ERR_ARG, "mpress_swap_in: handle not of this context");
  if (h->state != MPRESS_STATE_OUT_PENDING && h->state != MPRESS_STATE_OUT)
    return fail(MPRESS_ERR_STATE, "mpress_swap_in: handle is in state %d, not swapped out", h->state);
  if (h->graph && h->in_done)
    return fail(MPRESS_ERR_STATE, "mpress_swap_in: the graph handle's swap-in was already captured");
  MP_TRY(check_ptrs(dst, h->n_tensors, "mpress_swap_in(dst)"));
  DeviceGuard g(c->device);
  cudaStream_t stream = static_cast<cudaStream_t>(stream_);
  if (capturing(stream) != h->graph)
    return fail(MPRESS_ERR_STATE, h->graph ? "mpress_swap_in: the swap-out was captured into a graph; capture the "
                                             "swap-in into the same capture"
                                           : "mpress_swap_in: the swap-out ran eagerly; it cannot be swapped in "
                                             "under graph capture");

  std::vector<CopyDesc>& d = c->scratch_desc;
  std::vector<int>& dp = c->scratch_peer;
  d.resize(h->stripes.size());
  dp.resize(h->stripes.size());
  for (size_t i = 0; i < h->stripes.size(); ++i) {
    const mpress_stripe& s = h->stripes[i];
    d[i].src = c->parts[s.peer].base + h->slice_off[s.peer] + s.dst_off;
    d[i].dst = static_cast<uint8_t*>(dst[s.tensor]) + s.src_off;
    d[i].len = s.len;
    dp[i] = (int)s.peer;
  }
  if (h->graph || !same_stream(h->out_stream, stream)) cudaStreamWaitEvent(stream, h->out_done.get(), 0);
  HP_LAP(5, "in: checks + capture query + desc");
  int rc = run_copy(c, o, kDirIn, d, dp, stream, h->graph);
  HP_LAP(6, "in: run_copy (launch)");
  if (rc != MPRESS_OK) return rc;
  EvRef in_done, in_ext;
  MP_TRY(record_done(c, stream, h->graph, &in_done, &in_ext, "cudaEventRecord(in_done)"));
  HP_LAP(7, "in: event record");
  h->in_done = in_done;
  h->in_ext = in_ext;
  h->state = MPRESS_STATE_IN_PENDING;
  // A graph handle keeps its slices: every replay writes and reads them again.
  if (h->graph) return MPRESS_OK;

  // Release the slices now; their bytes stay fenced by the swap-in's event
  // until it completes (the table entry is "updated when it completes").
  for (int p = 0; p < c->world; ++p) {
    if (h->slice_off[p] == UINT64_MAX) continue;
    // Older fences inside this slice are dominated: this handle's swap-out
    // waited on every fence overlapping the slice (none can appear while the
    // slice is held), so the new event completes after them.
    auto& fs = c->parts[p].fences;
    const uint64_t a = h->slice_off[p], b = a + h->slice_len[p];
    for (auto it = fs.begin(); it != fs.end();) {
      if (it->off >= a && it->off + it->len <= b) it = fs.erase(it);
      else ++it;
    }
    fs.push_back({h->slice_off[p], h->slice_len[p], in_done, stream});
    free_slice(&c->parts[p], h->slice_off[p], h->slice_len[p]);
  }
  h->slices_held = false;
  HP_LAP(8, "in: fences + slice release");
  return MPRESS_OK;
}
}  // namespace

extern "C" int mpress_wait(mpress_ctx_t* c, mpress_handle_t* h, void* consumer) {
  if (!c || !h || h->ctx != c) return fail(MPRESS_ERR_ARG, "mpress_wait: bad argument");
  std::lock_guard<std::mutex> lk(c->mu);
  DeviceGuard g(c->device);
  const bool in = h->state == MPRESS_STATE_IN_PENDING || h->state == MPRESS_STATE_IN;
  // A graph handle: inside the capture, join on the capture's own event;
  // outside it, wait for the latest replay (the external record).
  const bool ext = h->graph && !capturing(static_cast<cudaStream_t>(consumer));
  const EvRef& e = ext ? (in ? h->in_ext : h->out_ext) : (in ? h->in_done : h->out_done);
  if (!e) return fail(MPRESS_ERR_STATE, "mpress_wait: nothing enqueued");
  cudaError_t r = cudaStreamWaitEvent(static_cast<cudaStream_t>(consumer), e.get(), 0);
  if (r != cudaSuccess) return cuda_fail(r, "mpress_wait: cudaStreamWaitEvent");
  return MPRESS_OK;
}

extern "C" int mpress_query(mpress_ctx_t* c, mpress_handle_t* h) {
  if (!c || !h || h->ctx != c) return fail(MPRESS_ERR_ARG, "mpress_query: bad argument");
  std::lock_guard<std::mutex> lk(c->mu);
  DeviceGuard g(c->device);
  if (h->graph) {  // the latest replay's completion; the state does not move
    const EvRef& x = h->in_ext ? h->in_ext : h->out_ext;
    const cudaError_t r = cudaEventQuery(x.get());
    if (r == cudaSuccess) return 1;
    if (r == cudaErrorNotReady) { cudaGetLastError(); return 0; }
    return cuda_fail(r, "mpress_query: cudaEventQuery");
  }
  cudaEvent_t e;
  int next;
  switch (h->state) {
    case MPRESS_STATE_OUT: case MPRESS_STATE_IN: return 1;
    case MPRESS_STATE_OUT_PENDING: e = h->out_done.get(); next = MPRESS_STATE_OUT; break;
    case MPRESS_STATE_IN_PENDING: e = h->in_done.get(); next = MPRESS_STATE_IN; break;
    default: return fail(MPRESS_ERR_STATE, "mpress_query: bad state %d", h->state);
  }
  cudaError_t r = cudaEventQuery(e);
  if (r == cudaSuccess) { h->state = next; return 1; }
  if (r == cudaErrorNotReady) { cudaGetLastError(); return 0; }
  return cuda_fail(r, "mpress_query: cudaEventQuery");
}

extern "C" int mpress_handle_state(const mpress_handle_t* h) { return h ? h->state : MPRESS_ERR_ARG; }

extern "C" int mpress_handle_is_graph(const mpress_handle_t* h) {
  if (!h) return fail(MPRESS_ERR_ARG, "mpress_handle_is_graph: null handle");
  return h->graph ? 1 : 0;
}

extern "C" int mpress_handle_slices(const mpress_handle_t* h, uint64_t* slice_off) {
  if (!h || !slice_off) return fail(MPRESS_ERR_ARG, "mpress_handle_slices: null argument");
  std::copy(h->slice_off.begin(), h->slice_off.end(), slice_off);
  return MPRESS_OK;
}

extern "C" int mpress_handle_free(mpress_ctx_t* c, mpress_handle_t* h, int force) {
  if (!c || !h) return fail(MPRESS_ERR_ARG, "mpress_handle_free: null argument");
  HP_START();
  std::lock_guard<std::mutex> lk(c->mu);
  if (h->ctx != c || !c->handles.count(h)) return fail(MPRESS_ERR_ARG, "mpress_handle_free: handle not of this context");
  DeviceGuard g(c->device);
  if (h->graph) {
    // The caller no longer replays the graph.  Release the slices fenced by
    // the latest replay's swap-in (or swap-out, if no swap-in was captured).
    if (!h->in_ext && !force)
      return fail(MPRESS_ERR_STATE, "mpress_handle_free: graph handle without a captured swap-in; force to drop "
                                    "the stashed data");
    const EvRef& fence = h->in_ext ? h->in_ext : h->out_ext;
    for (int p = 0; p < c->world; ++p) {
      if (h->slice_off[p] == UINT64_MAX) continue;
      c->parts[p].fences.push_back({h->slice_off[p], h->slice_len[p], fence, no_stream()});
      free_slice(&c->parts[p], h->slice_off[p], h->slice_len[p]);
    }
    h->slices_held = false;
  }
  if (h->slices_held) {
    if (!force)
      return fail(MPRESS_ERR_STATE, "mpress_handle_free: data still only in the stash (state %d); swap in or force", h->state);
    cudaEventSynchronize(h->out_done.get());  // swap-out kernels may still write the slices
    for (int p = 0; p < c->world; ++p)
      if (h->slice_off[p] != UINT64_MAX) free_slice(&c->parts[p], h->slice_off[p], h->slice_len[p]);
  }
  // An IN_PENDING handle's slices stay fenced: the fences share its event.
  c->handles.erase(h);
  delete h;
  HP_LAP(9, "handle_free");
  return MPRESS_OK;
}

namespace mpress {
namespace {

// Collective step of mpress_autotune: all ranks learn whether every rank is
// still fine (and start the next probe together).  Local contexts: no-op.
int autotune_barrier(mpress_ctx_t* c, int rc) {
  if (c->local) return rc;
  int32_t ok = rc == MPRESS_OK;
  std::vector<int32_t> all(c->world);
  if (c->exchange(c->exchange_user, &ok, sizeof ok, all.data()) != 0)
    return rc != MPRESS_OK ? rc : fail(MPRESS_ERR_SYS, "mpress_autotune: exchange failed");
  for (int r = 0; r < c->world; ++r)
    if (!all[r]) return rc != MPRESS_OK ? rc : fail(MPRESS_ERR_PEER, "mpress_autotune: rank %d failed", r);
  return rc;
}

float median(std::vector<float> v) {
  if (v.empty()) return 0.f;
  std::sort(v.begin(), v.end());
  return v[v.size() / 2];
}

}  // namespace
}  // namespace mpress

// Runtime choice of the SM path MPRESS_PATH_AUTO takes for an uncapped grid:
// time both SM kernels on this context's own peers, for a small and a large
// launch, and keep the faster per direction and size class
// (include/mpress.h).  The stash partitions serve as the probe's scratch, so
// no handle may be live.
extern "C" int mpress_autotune(mpress_ctx_t* c, uint64_t probe_bytes, int trials, void* stream_, float* ms_out) {
  if (!c || trials < 1 || trials > 64 || probe_bytes == 0)
    return fail(MPRESS_ERR_ARG, "mpress_autotune: bad argument");
  std::lock_guard<std::mutex> lk(c->mu);
  DeviceGuard g(c->device);
  cudaStream_t stream = static_cast<cudaStream_t>(stream_);
  int rc = c->handles.empty() ? MPRESS_OK
                              : fail(MPRESS_ERR_STATE, "mpress_autotune: %zu live handle(s); the probe uses the "
                                                       "stash as scratch", c->handles.size());
  // probe layout: an equal share of probe_bytes on every mapped device peer
  std::vector<int> peers;
  if (rc == MPRESS_OK)
    for (int p = 0; p < c->world; ++p)
      if (p != c->source && c->parts[p].base && !(c->host_peer && c->maps[p].host)) peers.push_back(p);
  std::vector<uint64_t> off(c->world, UINT64_MAX), len(c->world, 0);
  uint64_t total = 0;
  if (rc == MPRESS_OK && !peers.empty()) {
    const uint64_t share = probe_bytes / peers.size() / MPRESS_ALIGN * MPRESS_ALIGN;
    for (int p : peers) {
      uint64_t best = 0;
      for (auto& kv : c->parts[p].free) best = std::max(best, kv.second);
      len[p] = std::min(share, best / MPRESS_ALIGN * MPRESS_ALIGN);
      if (len[p] == 0 || !alloc_slice(&c->parts[p], len[p], &off[p])) { len[p] = 0; continue; }
      // A freed IN_PENDING handle leaves fences whose swap-in may still read
      // these bytes: the probe writes them only after those swap-ins.
      for (const Fence& f : c->parts[p].fences)
        if (f.off < off[p] + len[p] && off[p] < f.off + f.len) cudaStreamWaitEvent(stream, f.ev.get(), 0);
      total += len[p];
    }
  }
  uint8_t *src = nullptr, *dst = nullptr;
  cudaEvent_t ev[3] = {nullptr, nullptr, nullptr};
  if (rc == MPRESS_OK && total) {
    cudaError_t e = cudaMalloc(&src, total);
    if (e == cudaSuccess) e = cudaMalloc(&dst, total);
    if (e == cudaSuccess) e = cudaMemsetAsync(src, 0, total, stream);
    for (int i = 0; i < 3 && e == cudaSuccess; ++i) e = cudaEventCreate(&ev[i]);
    if (e != cudaSuccess) rc = cuda_fail(e, "mpress_autotune: probe buffers");
  }
  // Two probes per path, each a run of back-to-back launches over successive
  // windows of the probe buffers, as a pipeline streams fresh tensors: the
  // working set is the whole probe (beyond L2 for >= 256 MiB, so HBM / NVLink
  // is timed, not L2) and launch ramps overlap their predecessors (PDL) as in
  // steady state -- one isolated launch per trial overstated the bulk
  // kernel's ramp and flipped a 1% decision against it.
  // Class 1 ("large"): kLargeReps launches of probe/kLargeReps.  Class 0
  // ("small"): kSmallReps launches of kSmallProbe (both split over the peers).
  constexpr uint64_t kSmallProbe = 16ull << 20;
  constexpr int kSmallReps = 16, kLargeReps = 4;
  std::vector<CopyDesc> dout[2][kSmallReps], din[2][kSmallReps];
  std::vector<int> grp;
  uint64_t at = 0;
  const uint64_t small_share =
      peers.empty() ? 0 : std::max<uint64_t>(MPRESS_ALIGN, kSmallProbe / peers.size() / MPRESS_ALIGN * MPRESS_ALIGN);
  for (int p : peers) {
    if (!len[p]) continue;
    grp.push_back(p);
    for (int cls = 0; cls < 2; ++cls) {
      const int reps = cls ? kLargeReps : kSmallReps;
      const uint64_t n = cls ? std::max<uint64_t>(MPRESS_ALIGN, len[p] / kLargeReps / MPRESS_ALIGN * MPRESS_ALIGN)
                             : std::min(len[p], small_share);
      const uint64_t windows = std::max<uint64_t>(1, len[p] / n);
      for (int w = 0; w < reps; ++w) {
        const uint64_t o = (w % windows) * n;
        const uint64_t m = std::min(n, len[p] - o);
        dout[cls][w].push_back({src + at + o, c->parts[p].base + off[p] + o, m});
        din[cls][w].push_back({c->parts[p].base + off[p] + o, dst + at + o, m});
      }
    }
    at += len[p];
  }
  // warm-up round (-1), then `trials` rounds alternating which path goes first
  const int paths[2] = {MPRESS_PATH_DIRECT, MPRESS_PATH_BULK};
  if (rc == MPRESS_OK && c->opt.split >= MPRESS_SPLIT_DYNAMIC && !c->counters)
    rc = counter_ring_create(c->device, &c->counters);  // the probes run the context's split
  std::vector<float> t[2][2][2];  // [class][path][dir], ms per launch
  for (int r = -1; r < trials; ++r) {
    for (int cls = 0; cls < 2; ++cls) {
      const int reps = cls ? kLargeReps : kSmallReps;
      for (int k = 0; k < 2; ++k) {
        const int pi = (r & 1) ? 1 - k : k;
        rc = autotune_barrier(c, rc);
        if (rc != MPRESS_OK || grp.empty()) continue;
        int launches = 0;
        cudaEventRecord(ev[0], stream);
        for (int i = 0; i < reps && rc == MPRESS_OK; ++i)
          rc = launch_copy(paths[pi], MPRESS_VARIANT_AUTO, kDirOut, dout[cls][i].data(), grp.data(),
                           dout[cls][i].size(), 0, c->opt.pdl, stream, &launches, nullptr, 0, c->opt.split,
                           c->counters);
        cudaEventRecord(ev[1], stream);
        for (int i = 0; i < reps && rc == MPRESS_OK; ++i)
          rc = launch_copy(paths[pi], MPRESS_VARIANT_AUTO, kDirIn, din[cls][i].data(), grp.data(),
                           din[cls][i].size(), 0, c->opt.pdl, stream, &launches, nullptr, 0, c->opt.split,
                           c->counters);
        cudaEventRecord(ev[2], stream);
        cudaError_t e = cudaEventSynchronize(ev[2]);
        float a = 0, b = 0;
        if (e == cudaSuccess) e = cudaEventElapsedTime(&a, ev[0], ev[1]);
        if (e == cudaSuccess) e = cudaEventElapsedTime(&b, ev[1], ev[2]);
        if (e != cudaSuccess && rc == MPRESS_OK) rc = cuda_fail(e, "mpress_autotune: probe timing");
        if (r >= 0) {
          t[cls][pi][kDirOut].push_back(a / reps);
          t[cls][pi][kDirIn].push_back(b / reps);
        }
      }
    }
  }
  rc = autotune_barrier(c, rc);
  for (int p : peers)
    if (len[p]) free_slice(&c->parts[p], off[p], len[p]);
  cudaFree(src);
  cudaFree(dst);
  for (auto e : ev) if (e) cudaEventDestroy(e);
  if (rc != MPRESS_OK) return rc;
  for (int cls = 0; cls < 2; ++cls) {
    float m[2][2];
    for (int pi = 0; pi < 2; ++pi)
      for (int d = 0; d < 2; ++d) m[pi][d] = median(t[cls][pi][d]);
    if (!grp.empty())
      for (int d = 0; d < 2; ++d) {  // the class's choice stays unless the other kernel is >= 2% faster
        const int def = c->auto_path[d][cls];
        const int other = def == MPRESS_PATH_DIRECT ? MPRESS_PATH_BULK : MPRESS_PATH_DIRECT;
        const float t_def = m[def == MPRESS_PATH_BULK][d], t_other = m[other == MPRESS_PATH_BULK][d];
        c->auto_path[d][cls] = t_other < 0.98f * t_def ? other : def;
      }
    if (ms_out)
      for (int pi = 0; pi < 2; ++pi)
        for (int d = 0; d < 2; ++d) ms_out[cls * 4 + pi * 2 + d] = m[pi][d];
  }
  return MPRESS_OK;
}
