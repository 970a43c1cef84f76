/*
 * mpress.h -- C ABI of libmpress: MPress's device-to-device (D2D) stripe swap
 * (Zhou et al., "MPress", HPCA 2023), built B200-native.
 *
 * Citations: P:<n> = line n of the paper text (§III-C "D2D Swap"
 * unless stated), R<n> = a reading of the paper recorded in DESIGN.md §3.
 *
 * What the library does:
 *   A GPU with high memory pressure (an early pipeline stage, the "source" or
 *   "exporter") moves a batch of tensors into the spare HBM of light-load
 *   peers ("importers") over NVLink, striping each batch into sub-blocks whose
 *   sizes follow the per-link bandwidth and never exceed a peer's spare
 *   memory, then streams them back before the next use.
 *
 *   mpress_plan      -- the stripe planner (P:151, P:153, P:209, P:213,
 *                       Fig. 6 lines 2-8 P:156-170).  Host only, integers only.
 *   mpress_init*     -- the peer-memory layer: each importer reserves a stash
 *                       pool out of its spare HBM (cuMemCreate), exports it,
 *                       and every source maps the pools it uses (cuMemMap +
 *                       cuMemSetAccess over NVLink / NVSwitch).
 *   mpress_swap_out  -- hand-written sm_100a copy kernel: local tensor bytes
 *                       -> peer stash ("swap-out" operator).
 *   mpress_swap_in   -- peer stash -> caller's destination buffers (P:145
 *                       "swap-in" operator), guided by the handle = the
 *                       metadata-table entry of P:211.
 *   mpress_wait / mpress_query -- completion is signalled with CUDA events,
 *                       so the compute stream overlaps the swap and the host
 *                       never blocks.
 *   mpress_autotune  -- times the two SM kernels on the context's own links
 *                       and sets the default path per direction and size.
 *   mpress_set_option -- path, grid cap, kernel shape, chunk order, CTA
 *                       split, PDL, and rate pacing (a swap hidden in
 *                       its tensor's live interval needs no more bandwidth).
 *   Beyond the hot path: the multi-source and
 *   global planners, the device-stage mapping search, the 1F1B schedule and
 *   executor, the compaction decision rule, and a pinned host pool as a peer.
 *
 * Conventions
 *   - Every entry point returns int: MPRESS_OK (0) or a negative MPRESS_ERR_*;
 *     mpress_last_error() then returns a thread-local message.  No C++
 *     exception crosses this boundary.
 *   - Sizes and offsets are bytes (uint64_t).  "Device pointer" = a CUDA
 *     device address valid on the context's device.
 *   - CUDA handles are passed as void*: a `cudaStream_t` / `cudaEvent_t`
 *     (NULL stream = the legacy default stream).
 *   - Ownership: the caller owns tensors, destination buffers, streams and
 *     events it passes in.  The library owns plans, contexts, handles, the
 *     events inside handles, the stash pools and the peer mappings.
 *   - A context is single-threaded: calls on one context must not race.
 *     Different contexts are independent.
 */
#ifndef MPRESS_H_
#define MPRESS_H_

#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

#define MPRESS_VERSION 1

#if defined(__GNUC__)
#define MPRESS_API __attribute__((visibility("default")))
#else
#define MPRESS_API
#endif

/* ---- status codes --------------------------------------------------------- */
#define MPRESS_OK             0
#define MPRESS_ERR_ARG       -1  /* null pointer, granule % 256 != 0, source out
                                    of range, n_tensors == 0, size overflow     */
#define MPRESS_ERR_NO_SPACE  -2  /* peers' spare cannot hold the batch (P:295,
                                    R9) or the stash partition is full (R21)   */
#define MPRESS_ERR_ALIGN     -3  /* tensor / destination not 16-byte aligned    */
#define MPRESS_ERR_STATE     -4  /* illegal handle transition (R13)             */
#define MPRESS_ERR_PEER      -5  /* peer not mapped / no peer access            */
#define MPRESS_ERR_CUDA      -6  /* a CUDA runtime or driver call failed        */
#define MPRESS_ERR_SYS       -7  /* socket / fd-passing failure at init         */

#define MPRESS_ALIGN            256u    /* virtual tensor alignment (R6)        */
#define MPRESS_DEFAULT_GRANULE  65536u  /* planning unit G (R3)                 */

/* ---- the plan (metadata table) ------------------------------------- */

/* One sub-block: bytes [src_off, src_off+len) of tensor `tensor` live at
 * [dst_off, dst_off+len) of the source's slice on peer `peer`.
 * src_off and dst_off are multiples of 256 (R6).                           */
typedef struct mpress_stripe {
  uint32_t tensor;
  uint32_t peer;
  uint64_t src_off;
  uint64_t dst_off;
  uint64_t len;
} mpress_stripe;

typedef struct mpress_plan_info {
  int32_t  world;          /* number of devices the plan spans               */
  int32_t  source;         /* the exporter                                   */
  uint32_t n_tensors;
  uint32_t n_stripes;
  uint64_t granule;        /* G                                              */
  uint64_t virtual_bytes;  /* V = sum_i roundup(S_i, 256)                    */
  uint64_t units;          /* K = ceil(V / G)                                */
} mpress_plan_info;

typedef struct mpress_plan_s   mpress_plan_t;    /* opaque, library-owned */
typedef struct mpress_ctx_s    mpress_ctx_t;     /* opaque, library-owned */
typedef struct mpress_handle_s mpress_handle_t;  /* opaque, library-owned */

/*
 * mpress_plan -- stripe assignment of one source's tensor batch over its
 * peers (P:151 equal sub-blocks on symmetric links; P:153/P:209 sub-block
 * sizes proportional to link bandwidth, tensors batched; Fig. 6 line 3 P:160
 * spare = MEM_CAP - MEM_USE bounds each peer; P:213 best score = minimum of the
 * maximal swap time).
 *
 *   world         number of devices, >= 1
 *   source        exporter index in [0, world)
 *   spare_bytes   [world] spare HBM of each device; the source's entry is ignored.
 *                 Usable = floor(spare/G)*G (R8).
 *   link_bw       [world] integer bandwidth weight of link source->p; 0 = not an
 *                 NVLink neighbour (R10).  Only ratios matter.
 *   n_tensors     >= 1;  tensor_bytes [n_tensors], each >= 1
 *   granule       G; 0 -> MPRESS_DEFAULT_GRANULE; must be a multiple of 256
 *   out           receives a new plan; free with mpress_plan_free
 *
 * Result (R1-R7): the batch is laid out virtually (tensor i at a 256-aligned
 * offset, list order), cut into K units of G bytes, and peer p receives k_p
 * units minimising max_p k_p/B_p subject to k_p*G <= spare_p, ties to the lower
 * device index; peer p stores one contiguous range of the virtual batch
 * (peers ascending).  Integer arithmetic only: the result is bit-identical on
 * every rank and every call.
 * Errors: MPRESS_ERR_ARG, MPRESS_ERR_NO_SPACE (no partial plans, R9).
 */
MPRESS_API int mpress_plan(int world, int source, const uint64_t* spare_bytes,
                const uint64_t* link_bw, uint32_t n_tensors,
                const uint64_t* tensor_bytes, uint64_t granule,
                mpress_plan_t** out);

/* Borrow the plan's stripe list (sorted by peer, then tensor) and the
 * per-peer byte counts [world].  Pointers stay valid until mpress_plan_free. */
MPRESS_API int mpress_plan_stripes(const mpress_plan_t* plan, const mpress_stripe** stripes,
                        uint32_t* n_stripes, const uint64_t** peer_bytes);
/* Borrow the per-peer unit counts k_p [world]. */
MPRESS_API int mpress_plan_units(const mpress_plan_t* plan, const uint64_t** units);
MPRESS_API int mpress_plan_get_info(const mpress_plan_t* plan, mpress_plan_info* info);
MPRESS_API void mpress_plan_free(mpress_plan_t* plan);

/*
 * mpress_partition_sequential -- the stash partition of several sources
 * (Fig. 6 lines 2-8 P:156-170, reading R12): sources are planned in ascending
 * index, each against floor(remaining_p / copies_s) per peer, and reserve
 * copies_s * k_p * G bytes of peer p.
 *   bw_matrix     [world*world] row s = link_bw of source s
 *   n_sources     entries in sources / n_tensors / copies
 *   sizes_flat    concatenated tensor_bytes of the sources, in the order given
 *   partition     [world*world] out: partition[s*world+p] = bytes of p's pool
 *                 owned by source s (0 for non-sources)
 * Errors: as mpress_plan for any source.
 */
MPRESS_API int mpress_partition_sequential(int world, const uint64_t* spare_bytes,
                                const uint64_t* bw_matrix, uint32_t n_sources,
                                const int32_t* sources, const uint32_t* n_tensors,
                                const uint64_t* sizes_flat, const uint32_t* copies,
                                uint64_t granule, uint64_t* partition);

/*
 * mpress_plan_global -- NEXT-1: joint assignment of several exporters'
 * batches to the importers' spare memory (Fig. 6: every way to
 * distribute each importer's spare among its overflowed neighbours, combined
 * and scored by the reciprocal of the maximal D2D swap time; reading
 * R23).  All sources swap at once; with x_sp units of source s on importer p
 *   T = max( x_sp / B_sp  (every used link),
 *            sum_p x_sp / E_s  (egress port, if egress && egress[s] > 0),
 *            sum_s x_sp / I_p  (ingress port, if ingress && ingress[p] > 0) )
 * is minimised exactly over integer units subject to sum_p x_sp = K_s and
 * sum_s x_sp <= floor(spare_p / G).
 *   sources [n_sources] distinct exporters; n_tensors [n_sources];
 *   sizes_flat the exporters' tensor sizes, concatenated in that order;
 *   bw_matrix [world*world] row s = link weights of s (0 = no link);
 *   egress / ingress [world] port weights or NULL (no port limit);
 *   units_out [n_sources*world] out: x (row i = sources[i]);
 *   makespan_num / makespan_den out (may be NULL): T* = num / den units per
 *   weight unit.
 * T* is unique; the assignment is one optimal x, identical on every rank.
 * Turn a row into a plan with mpress_plan_from_units.
 * Errors: MPRESS_ERR_ARG, MPRESS_ERR_NO_SPACE.
 */
MPRESS_API int mpress_plan_global(int world, uint32_t n_sources, const int32_t* sources,
                                  const uint32_t* n_tensors, const uint64_t* sizes_flat,
                                  const uint64_t* spare_bytes, const uint64_t* bw_matrix,
                                  const uint64_t* egress, const uint64_t* ingress, uint64_t granule,
                                  uint64_t* units_out, uint64_t* makespan_num,
                                  uint64_t* makespan_den);

/* mpress_plan_from_units -- the plan (layout and stripes, R6/R7) of one batch
 * for a given unit split units[world] (e.g. a row of mpress_plan_global).
 * Errors: MPRESS_ERR_ARG if units[source] != 0 or sum(units) != K. */
MPRESS_API int mpress_plan_from_units(int world, int source, const uint64_t* units,
                                      uint32_t n_tensors, const uint64_t* tensor_bytes,
                                      uint64_t granule, mpress_plan_t** out);

/*
 * mpress_map_search -- NEXT-3: device-stage mapping search (Fig. 6 lines
 * 10-26; reading R25).  Every mapping of the n
 * pipeline stages onto the n GPUs is enumerated in lexicographic order of
 * (gpu of stage 0, gpu of stage 1, ...); each is scored by the joint optimum
 * of mpress_plan_global (the overflowed stages' demands on the light stages'
 * spare, over the GPUs' links); the first mapping with the smallest swap
 * time wins.  n! mappings: n <= 10.  On symmetric links every mapping scores
 * the same and the paper skips the search.
 *   demand [n] bytes each stage must swap out (0 = light stage)
 *   spare  [n] spare bytes of each light stage (ignored for overflowed ones)
 *   link   [n*n] link weights between GPUs (0 = not an NVLink neighbour)
 *   egress / ingress [n] per-GPU port weights or NULL
 *   stage_to_gpu [n] out; makespan_num / makespan_den / evaluated may be NULL.
 * Errors: MPRESS_ERR_ARG, MPRESS_ERR_NO_SPACE (no mapping fits).
 */
MPRESS_API int mpress_map_search(int n, const uint64_t* demand, const uint64_t* spare,
                                 const uint64_t* link, const uint64_t* egress,
                                 const uint64_t* ingress, uint64_t granule, int32_t* stage_to_gpu,
                                 uint64_t* makespan_num, uint64_t* makespan_den,
                                 uint64_t* evaluated);

/* ---- NEXT-4: memory-compaction decision rule (§III-D) ---------------------------- */

/* Cost statistics of one tensor (Table III; all times ns). */
typedef struct mpress_tensor_stat {
  uint64_t bytes;
  uint64_t live_ns;       /* live interval (P:226 fn.1)                        */
  uint64_t recompute_ns;  /* extra forward time; MPRESS_NOT_RECOMPUTABLE for
                             non-activations (optimizer states, gradients)     */
  uint64_t cpu_swap_ns;   /* GPU-CPU swap out + in over PCIe                   */
  uint64_t d2d_swap_ns;   /* D2D swap out + in over NVLink                     */
} mpress_tensor_stat;

#define MPRESS_NOT_RECOMPUTABLE  UINT64_MAX
#define MPRESS_CHOICE_CPU_SWAP   1u
#define MPRESS_CHOICE_RECOMPUTE  2u
#define MPRESS_CHOICE_D2D        3u

/*
 * mpress_compaction_plan -- NEXT-4: which optimization frees each tensor
 * (§III-D; reading R26).  A swap costs max(0, cost - live
 * interval) (fn.2 P:238), recomputation its forward time; the initial
 * assignment is the cheaper of GPU-CPU swap and recomputation (ties -> swap,
 * P:224-228); then tensors in order of decreasing overhead move to D2D swap
 * when it is strictly cheaper and they fit in the remaining d2d_capacity bytes
 * (P:229-232); ties keep the option that spends no spare GPU memory
 * (Table III discussion).
 *   choice [n] out (MPRESS_CHOICE_*); overhead_ns [n] out or NULL;
 *   total_overhead_ns out; d2d_bytes out or NULL.
 * Errors: MPRESS_ERR_ARG.
 */
MPRESS_API int mpress_compaction_plan(uint32_t n, const mpress_tensor_stat* stats,
                                      uint64_t d2d_capacity, uint32_t* choice,
                                      uint64_t* overhead_ns, uint64_t* total_overhead_ns,
                                      uint64_t* d2d_bytes);

/* ---- NEXT-2: 1F1B swap schedule with the live-interval check ------------------ */

/* Inputs (all times in ns, integers).  Computation-balanced stages:
 * every stage takes t_fwd_ns / t_bwd_ns per micro-batch. */
typedef struct mpress_1f1b_params {
  uint32_t stages;         /* S >= 1 pipeline stages (Fig. 1)            */
  uint32_t stage;          /* the exporter stage e in [0, S) that swaps            */
  uint32_t micro_batches;  /* M >= 1 per mini-batch                                */
  uint32_t duplex;         /* 1: swap-outs and swap-ins on two streams     */
  uint64_t t_fwd_ns;
  uint64_t t_bwd_ns;
  uint64_t t_out_ns;       /* swap-out of one micro-batch's activations            */
  uint64_t t_in_ns;        /* swap-in of them (from the measured GB/s)             */
  uint64_t t_slack_ns;     /* extra lead the swap-in keeps before the backward     */
} mpress_1f1b_params;

typedef struct mpress_1f1b_slot {  /* one micro-batch at the exporter stage */
  uint64_t fwd_start, fwd_end, bwd_start, bwd_end;  /* with swapping          */
  uint64_t live_ns;        /* live interval without swapping: backward start -
                              forward end (P:226 fn.1)                         */
  uint64_t out_start, out_end, in_start, in_end;
  uint32_t in_trigger;     /* the swap-in is enqueued when op #in_trigger of the
                              stage (1F1B order, 0-based) has ended: the last op
                              that still leaves t_in before the backward       */
  uint32_t hidden;         /* 1 if the swap-in ended before the backward could
                              otherwise start (no extra delay)          */
  uint64_t exposed_ns;     /* backward start with swapping - without           */
} mpress_1f1b_slot;

typedef struct mpress_1f1b_summary {
  uint64_t makespan_ns;            /* whole pipeline, with the exporter swapping */
  uint64_t makespan_noswap_ns;
  uint32_t peak_resident;          /* max micro-batch activation sets resident on
                                      the exporter at once, with swapping       */
  uint32_t peak_resident_noswap;
  uint32_t ops;                    /* compute ops of the exporter stage (2M)    */
  uint32_t pad;
} mpress_1f1b_summary;

/*
 * mpress_schedule_1f1b -- the swap schedule of the exporter stage in a 1F1B
 * pipeline (PipeDream / DAPPLE): every micro-batch's
 * activations are swapped out after its forward and swapped back in
 * on the swap-in stream as late as the no-swap timeline allows them to
 * still arrive before the backward; per micro-batch it reports the live
 * interval (P:226 fn.1), the swap times, whether the swap is hidden
 * and the exposed delay (fn.2), plus peak resident activation sets
 * with and without swapping (the memory the D2D swap saves).  Model: reading
 * R24.  slots [micro_batches] out; summary may be NULL.
 * Errors: MPRESS_ERR_ARG.
 */
MPRESS_API int mpress_schedule_1f1b(const mpress_1f1b_params* params, mpress_1f1b_slot* slots,
                                    mpress_1f1b_summary* summary);

/*
 * The swap executor (the runtime "executor executes the memory saving
 * operators ... swap-out ... and state recovering ones ... swap-in") of the
 * exporter stage in a 1F1B pipeline, driven by mpress_schedule_1f1b.  The
 * caller runs its compute ops in 1F1B order (mpress_executor_ops() of them)
 * on its compute stream and brackets each op j:
 *   mpress_executor_before(x, j, compute, &kind, &m)  -- kind 0 = F(m),
 *       1 = B(m); for B(m) the compute stream waits for m's swap-in;
 *   <enqueue the op on `compute`>
 *   mpress_executor_after(x, j, compute, activations) -- for F(m), swaps out
 *       `activations` ([n_tensors] device pointers of the plan's batch) on the
 *       swap-out stream after the op; then enqueues every swap-in this op
 *       triggers on the swap-in stream, into the buffers given by
 *       mpress_executor_restore_to(x, m, dst) beforehand.
 * mpress_executor_release(x, m, stream) -- makes `stream` wait until m's
 *       swap-out has read its activations (between after(F(m)) and
 *       before(B(m))).  Freeing the activations is the point of the swap
 *       (memory saving operators); a caching allocator on `stream`
 *       may hand their memory to the next op only after this call.
 * Enqueue-only.  One executor serves any number of steps.
 * An executor step cannot be captured into a CUDA graph (MPRESS_ERR_STATE
 * while any of its streams is capturing): it recycles stash slices between
 * micro-batches, which a replayed graph would share with eager swaps.
 * Free executors before mpress_finalize of their context.
 * Errors: MPRESS_ERR_ARG, MPRESS_ERR_STATE (op order violated, no restore
 * buffers), plus those of swap_out / swap_in.
 */
typedef struct mpress_executor_s mpress_executor_t;
MPRESS_API int mpress_executor_create(mpress_ctx_t* ctx, const mpress_plan_t* plan,
                                      const mpress_1f1b_params* params, void* out_stream,
                                      void* in_stream, mpress_executor_t** out);
MPRESS_API int mpress_executor_ops(const mpress_executor_t* x);
MPRESS_API int mpress_executor_slot(const mpress_executor_t* x, uint32_t micro_batch,
                                    mpress_1f1b_slot* slot);
MPRESS_API int mpress_executor_restore_to(mpress_executor_t* x, uint32_t micro_batch,
                                          void* const* dst);
MPRESS_API int mpress_executor_before(mpress_executor_t* x, uint32_t op, void* compute_stream,
                                      uint32_t* kind, uint32_t* micro_batch);
MPRESS_API int mpress_executor_after(mpress_executor_t* x, uint32_t op, void* compute_stream,
                                     void* const* activations);
MPRESS_API int mpress_executor_release(mpress_executor_t* x, uint32_t micro_batch, void* stream);
/* The executor's own swap options (MPRESS_OPT_PATH, _MAX_CTAS, _VARIANT,
 * _ORDER, _PDL, _PACE_MBPS, _SPLIT; same values and validation as
 * mpress_set_option): a copy of the context's taken at mpress_executor_create,
 * so one pipeline stage can run its swaps on another transfer path or grid
 * than the rest of the process -- the NEXT-2 replay measured no single path
 * best for every stage (copy engines beside short GEMMs, the TMA kernel
 * beside long ones).  A B200 addition (§9).
 * Errors: MPRESS_ERR_ARG (not a swap option, bad value). */
MPRESS_API int mpress_executor_set_option(mpress_executor_t* x, int option, int64_t value);
MPRESS_API int mpress_executor_get_option(const mpress_executor_t* x, int option, int64_t* value);
MPRESS_API int mpress_executor_free(mpress_executor_t* x);

/* ---- peer-memory layer ----------------------------------------------------- */

/* All-gather callback, implemented by the caller over its process group:
 * every rank passes `len` bytes in `mine`; on return `all` holds world*len
 * bytes, rank r's at all + r*len.  Must act as a barrier.  Return 0 on success. */
typedef int (*mpress_exchange_fn)(void* user, const void* mine, size_t len, void* all);

/*
 * mpress_init -- the memory manager's allocation side for the D2D tier
 * ("the memory manager takes over the memory allocation/deallocation";
 * it "is responsible for allocating and releasing the GPU/CPU memory
 * space"): each light-load GPU reserves the spare HBM the plan stripes into
 * and every source maps its partitions on those peers.
 * Collective over `world` processes, one per GPU (torchrun).
 *   device     CUDA ordinal this rank runs on
 *   partition  [world*world], identical on all ranks (see
 *              mpress_partition_sequential).  Rank p creates a stash pool of
 *              sum_s partition[s*world+p] bytes (rounded up to the VMM
 *              granularity) in its own HBM; source s's partition starts at
 *              sum_{s'<s} partition[s'*world+p].
 *   exchange   all-gather used to swap process ids and to synchronise; the
 *              pool handles themselves travel as POSIX file descriptors over
 *              Unix-domain sockets (SCM_RIGHTS).
 * Every rank maps each peer pool it owns a partition in, with read/write
 * access for `device` (peer access over NVLink).
 * Errors: MPRESS_ERR_ARG, MPRESS_ERR_CUDA, MPRESS_ERR_PEER, MPRESS_ERR_SYS.
 */
MPRESS_API int mpress_init(int device, int world, int rank, const uint64_t* partition,
                mpress_exchange_fn exchange, void* exchange_user,
                mpress_ctx_t** out);

/*
 * mpress_init_local -- single-process variant of mpress_init (same passages,
 * P:145 / P:236 / P:151): peer p's pool lives on
 * devices[p] and holds only this source's partition (partition[source*world+p]
 * bytes).  With every devices[p] equal it is the 1-GPU "loopback" mode: the
 * peers are disjoint VMM pools of the same GPU, so the whole data path
 * (planner, mapping, kernels, scheduler) runs with HBM standing in for NVLink.
 * devices[p] == MPRESS_DEVICE_HOST makes peer p a pinned host pool (NEXT-4,
 * the GPU-CPU swap tier of P:105/P:145/P:236): the same plan, kernels and
 * events move the bytes over PCIe; give it a link weight in proportion to
 * PCIe bandwidth and the planner stripes between NVLink peers and the host
 * (P:153).  devices[source] must be a GPU.
 */
#define MPRESS_DEVICE_HOST (-1)
MPRESS_API int mpress_init_local(int world, int source, const int* devices,
                      const uint64_t* partition, mpress_ctx_t** out);

/* mpress_finalize -- the memory manager's release side ("the memory
 * manager takes over the memory allocation/deallocation"; it is
 * "responsible for allocating and releasing the GPU/CPU memory space"):
 * collective for contexts made by mpress_init (barrier, unmap, release of
 * the pools); a local context releases at once.  Outstanding handles are
 * freed (their stashed data is dropped).  NULL is a no-op.
 * Errors: MPRESS_ERR_SYS (the closing barrier failed), MPRESS_ERR_CUDA. */
MPRESS_API int mpress_finalize(mpress_ctx_t* ctx);

/* mpress_stash_free -- the memory manager "monitoring the per-device memory
 * usage" for the D2D tier: largest contiguous free extent of this
 * source's partition on each peer, written to free_bytes [world, caller
 * owned] -> the spare_bytes argument of mpress_plan for the next batch
 * (reading R21).  Errors: MPRESS_ERR_ARG (NULL argument). */
MPRESS_API int mpress_stash_free(const mpress_ctx_t* ctx, uint64_t* free_bytes);

/* Tunables.  MPRESS_OPT_PATH: 0 = SM kernel, direct 16/32-B loads/stores;
 * 1 = SM kernel, bulk-async copies (the SM's TMA engine, cp.async.bulk)
 * staged through shared memory; 2 = copy engines (cudaMemcpyAsync per stripe
 * on per-peer streams, the measured comparator); 3 = MPRESS_PATH_AUTO
 * (default): per launch, at a full grid (max_ctas 0 or above the SM count)
 * the kernel mpress_autotune measured faster on this context's links for
 * that direction and size class (until then direct below
 * MPRESS_AUTO_SMALL_BYTES per launch, bulk above), direct when the grid is
 * capped to <= one CTA per SM (its
 * 128-thread CTAs co-reside with a GEMM, bulk CTAs' shared memory does not)
 * or when the launch mixes device peers and host pools, and the copy
 * engines when every stripe of the launch goes to a host pool (over PCIe
 * they beat every SM kernel shape, 56.9 vs 52.6 GB/s).
 * MPRESS_OPT_LAST_PATH (read-only) reports the path the last swap call ran.
 * Setting the path resets the variant to MPRESS_VARIANT_AUTO; under
 * MPRESS_PATH_AUTO only MPRESS_VARIANT_AUTO is accepted.
 * MPRESS_OPT_MAX_CTAS: cap on the kernel grid (0 = the variant's default
 * grid, a multiple of the SM count); CTAs spread one per SM first, so this is
 * the SM-count cap that protects a concurrent GEMM.
 * MPRESS_OPT_VARIANT: kernel shape within the path -- direct: 0 = 256
 * threads x 8 vectors (2 CTAs/SM by default), 1 = 512x8, 2 = 256x16,
 * 3 = 1024x4, 4 = 128x8 (16-byte vectors), 5 = 256x4, 6 = 256x8, 7 = 128x4,
 * 8 = 256x4 with L2 evict-first loads and stores, 9 = 128x8, 10 = 128x16, 11 = 64x16,
 * 12 = 128x8 with L2 evict-first loads and stores, 13 = 32x16 (one warp)
 * (32-byte vectors, used
 * only when every address is 32-byte aligned, else the 16-byte shape);
 * (beside a long bf16 GEMM under the power cap, MPRESS_PATH_BULK shape 5 on
 * one CTA per SM cost the GEMM ~10% where the direct shapes cost ~17-21% at
 * the same rate)
 * bulk: 0 = 6 slots x 32 KiB, 1 = 12 x 16 KiB, 2 = 3 x 64 KiB (one CTA per
 * SM), 3 = 3 x 32 KiB (one per SM; twice as many fit), 4 = 4 x 16 KiB (three
 * per SM),
 * 5 = 2 x 8 KiB, 6 = 3 x 4 KiB, 7 = 4 x 4 KiB, 8 = 8 x 2 KiB, 9 = 4 x 4 KiB
 * plus a second warp copying 4 x 4 KiB through registers, both claiming
 * work under the dynamic split (one per SM; small enough to share an SM
 * with a GEMM CTA);
 * copy engines: 0 = cudaMemcpyAsync per stripe on one side stream per peer
 * (the only copy-engine variant);
 * MPRESS_VARIANT_AUTO (-1, default) = direct 9 when the grid is capped at
 * <= one CTA per SM (128-thread CTAs co-reside with a GEMM), else 5; bulk 3;
 * on a full grid a launch of < 16 chunks per SM (< ~74 MiB) takes the
 * deeper-ring shape instead (direct 1, bulk 0: more bytes in flight per SM
 * for a launch that is mostly ramp and tail); copy engines 0.
 * MPRESS_OPT_ORDER: chunk order inside one launch -- 0 = interleave the
 * peers by a weighted round robin, so every peer link carries its share of
 * the swap at every moment (default; needed when several sources share
 * peers); 1 = plan order (peer by peer).
 * MPRESS_OPT_PDL: programmatic dependent launch of the SM kernels, so a swap
 * kernel's launch and CTA ramp-up overlap the tail of the previous kernel on
 * its stream (each kernel still waits for that grid to complete before
 * touching memory).  1 (default) = only for an uncapped grid (MAX_CTAS 0 or
 * above the SM count); a capped swap runs beside a GEMM, and there PDL chains
 * of swap kernels cost the bf16 8192^3 cuBLAS GEMM +60% instead of +6-9%
 * (profiles/r01/pdl_gemm_ab.txt); 2 = always; 0 = never.
 * Invalid values -> MPRESS_ERR_ARG. */
#define MPRESS_OPT_PATH      1
#define MPRESS_OPT_MAX_CTAS  2
#define MPRESS_OPT_VARIANT   3
#define MPRESS_OPT_ORDER     4
#define MPRESS_OPT_PDL       7
/* MPRESS_OPT_PACE_MBPS: 0 (default) = the SM kernels move bytes as fast as
 * the links allow; R > 0 = each swap launch moves at most R MB/s: its CTAs
 * space their chunks on the GPU's global timer.  A swap is free when it
 * finishes within its tensor's live interval (fn.1 P:226), so a swap
 * beside compute needs only bytes / live-interval; pacing it there leaves
 * the rest of HBM, L2 and the issue slots to the compute.  Not applied to
 * the copy-engine path.  A paced launch keeps its CTAs resident (sleeping)
 * for longer, and a paced swap-out keeps its source tensors in use for
 * longer: pace a swap beside a long kernel whose CTAs co-reside with the
 * swap's, not a swap-out that should free memory at once (DESIGN.md §7c,
 * NEXT-2 replay). */
#define MPRESS_OPT_PACE_MBPS 12
/* MPRESS_OPT_SPLIT: how one launch's chunks (interleaved over the peers, see
 * MPRESS_OPT_ORDER) are shared by its CTAs -- MPRESS_SPLIT_BLOCKED (0):
 * each CTA takes a contiguous block of the sequence, so every CTA
 * moves the same number of chunks +- one per peer; MPRESS_SPLIT_STRIDED (1,
 * round 1): a grid stride over the sequence, whose skipped positions alias
 * with the stride (up to 1.7x the mean chunk count on one CTA);
 * MPRESS_SPLIT_DYNAMIC (2): the CTAs claim blocks of a few chunks (~128 KiB)
 * from a per-launch counter in device memory (guided self-scheduling: blocks
 * shrink as the sequence runs out), so every CTA works inside one moving
 * window of the sequence and SMs that run faster move more -- no tail.  The
 * counter slot is reset by the launch's last CTA and reused once the event
 * recorded after the launch has fired; launches of < 4 chunks per CTA and
 * launches enqueued under graph capture run BLOCKED.
 * MPRESS_SPLIT_AUTO (3, default): launches of < 32 chunks per CTA STRIDED on
 * a full grid (>= one CTA per SM; BLOCKED on a capped one), larger ones
 * DYNAMIC on the TMA (bulk) kernel and BLOCKED on the direct
 * kernel (measured on B200 loopback: bulk +3.8% at 900 MiB and 4 GiB with
 * the claims, launches of a few chunks per CTA +1-7% with the stride, the
 * direct kernel's large launches fastest blocked). */
#define MPRESS_OPT_SPLIT     13
#define MPRESS_SPLIT_BLOCKED 0
#define MPRESS_SPLIT_STRIDED 1
#define MPRESS_SPLIT_DYNAMIC 2
#define MPRESS_SPLIT_AUTO    3
/* Read-only (mpress_get_option): how the peer pools were mapped --
 * MPRESS_TRANSPORT_LOCAL (mpress_init_local), _VMM_FD (cuMem pools exported
 * as POSIX fds, passed over Unix sockets), or _LEGACY_IPC (cudaMalloc pools
 * shared with CUDA IPC handles through the all-gather; used when the fd path
 * fails on any rank, or forced with the environment variable MPRESS_IPC=legacy). */
#define MPRESS_OPT_TRANSPORT 5
#define MPRESS_OPT_LAST_PATH 6   /* read-only: path of the last swap call */
/* Read-only: the SM path MPRESS_PATH_AUTO takes for an uncapped grid, per
 * direction, for a launch moving >= MPRESS_AUTO_SMALL_BYTES (_OUT / _IN) or
 * fewer (_OUT_SMALL / _IN_SMALL).  Until mpress_autotune measures otherwise:
 * bulk for large launches, direct for small ones (one B200, CUDA-graph-
 * replayed swap pairs, 4 KiB - 4 GiB x 1/3/7 peers: direct 5-25% faster up
 * to 16 MiB over 3 or 7 peers, the two even at 64 MiB, bulk 3-8% faster from
 * 256 MiB; profiles/r01/sweep_sizes_v2.jsonl). */
#define MPRESS_OPT_AUTO_OUT  8
#define MPRESS_OPT_AUTO_IN   9
#define MPRESS_OPT_AUTO_OUT_SMALL 10
#define MPRESS_OPT_AUTO_IN_SMALL  11
#define MPRESS_AUTO_SMALL_BYTES   33554432u  /* 32 MiB */
#define MPRESS_TRANSPORT_LOCAL      0
#define MPRESS_TRANSPORT_VMM_FD     1
#define MPRESS_TRANSPORT_LEGACY_IPC 2
#define MPRESS_VARIANT_AUTO  (-1)
#define MPRESS_ORDER_INTERLEAVE 0
#define MPRESS_ORDER_PLAN       1
#define MPRESS_PATH_DIRECT   0
#define MPRESS_PATH_BULK     1
#define MPRESS_PATH_CE       2
#define MPRESS_PATH_AUTO     3
MPRESS_API int mpress_set_option(mpress_ctx_t* ctx, int key, int64_t value);

/* mpress_autotune -- not a paper operation: a B200 addition.
 * The paper's transfer mechanism is fixed (cudaMemcpyPeer over NVLink,
 * P:121); here two SM kernels and the copy engines can move a stripe, so
 * the library measures which is faster on the context's own links.
 * Measure, don't guess: which SM kernel MPRESS_PATH_AUTO should run for an
 * uncapped grid on THIS context's links (HBM loopback on one GPU, NVLink /
 * NVSwitch on several -- the kernels were only ever compared on loopback,
 * DESIGN.md §7), per direction and size class.  The probe is `probe_bytes`
 * split equally over the mapped device peers (each share a multiple of 256
 * and at most that partition's largest free block), moved out of a
 * library-owned scratch buffer into the stash partitions and back as runs of
 * back-to-back launches over successive windows of it, as a pipeline streams
 * fresh tensors: class "large" = 4 launches of probe_bytes / 4, class
 * "small" = 16 launches of 16 MiB.  Use probe_bytes >= 256 MiB so the
 * working set exceeds the 126 MB L2 and each large launch is at least
 * MPRESS_AUTO_SMALL_BYTES.  Both kernels are timed -- direct (shape 5) and
 * bulk (shape 3) -- one warm-up round then `trials` (1..64) rounds
 * alternating which goes first; per direction and class the median time per
 * launch decides, and the class's current choice stays unless the other
 * kernel is at least 2% faster (the probe's run-to-run noise is ~1%).  Read
 * the result back with MPRESS_OPT_AUTO_OUT / _IN / _OUT_SMALL / _IN_SMALL;
 * every later AUTO swap of this context with an uncapped grid uses it (a
 * capped grid or a host peer still takes the direct kernel).  Runs
 * synchronously on `stream` (NULL = legacy default stream).
 * Collective for an mpress_init context: every rank calls it with the same
 * `trials` (a rank without device peers only takes part in the barriers),
 * and each probe starts on all ranks together (barriers through the
 * exchange callback), so the probe sees the all-to-all load of a real swap.
 * ms (may be NULL): [8] = median ms per launch of {small class, large class}
 * x {direct, bulk} x {out, in} (0 when this rank probed nothing).
 * Errors: MPRESS_ERR_ARG (null ctx, trials out of range, probe_bytes 0),
 * MPRESS_ERR_STATE (a live handle: the probe uses the stash as scratch),
 * MPRESS_ERR_CUDA, MPRESS_ERR_SYS / _PEER (exchange failed, another rank
 * failed). */
MPRESS_API int mpress_autotune(mpress_ctx_t* ctx, uint64_t probe_bytes, int trials, void* stream, float* ms);
MPRESS_API int mpress_get_option(const mpress_ctx_t* ctx, int key, int64_t* value);

/* ---- the swap --------------------------------------------------------------- */

/* Handle states (R13; "record ... before the execution of the swap-out
 * operator ... updated when it completes"). */
#define MPRESS_STATE_OUT_PENDING 1  /* swap-out enqueued                      */
#define MPRESS_STATE_OUT         2  /* swap-out complete: sources reusable     */
#define MPRESS_STATE_IN_PENDING  3  /* swap-in enqueued                       */
#define MPRESS_STATE_IN          4  /* swap-in complete: stash slice released  */

/*
 * mpress_swap_out -- enqueue the move of every stripe of `plan` from the
 * caller's tensors into this source's stash slices on the peers.
 *   tensors  [plan n_tensors] device pointers, 16-byte aligned, each at least
 *            tensor_bytes long; must stay valid until the handle reaches
 *            MPRESS_STATE_OUT (mpress_wait / mpress_query)
 *   stream   cudaStream_t the kernel runs on (the "swap-out stream")
 *   after    cudaEvent_t the stream waits on first (e.g. recorded on the
 *            compute stream after the producing op), or NULL
 *   out      receives a handle holding one contiguous slice per used peer
 *            (first fit, lowest address, inside this source's partition)
 * Bytes are copied bit-exactly; nothing interprets them (R18).
 * Errors: MPRESS_ERR_ARG, MPRESS_ERR_ALIGN, MPRESS_ERR_NO_SPACE (partition
 * full), MPRESS_ERR_PEER (plan uses a peer this context has not mapped, or
 * plan.source != the context's source), MPRESS_ERR_CUDA.
 */
MPRESS_API int mpress_swap_out(mpress_ctx_t* ctx, const mpress_plan_t* plan,
                    void* const* tensors, void* stream, void* after,
                    mpress_handle_t** out);

/*
 * mpress_swap_in -- enqueue the move of every stripe back into `dst`
 * ([n_tensors] device pointers, 16-byte aligned; may differ from the
 * swap-out tensors, R14).  The stream first waits for the swap-out.  The
 * handle's slices are released for reuse once this copy completes (later
 * swap-outs into the same bytes are ordered after it by an event).
 * Errors: MPRESS_ERR_STATE unless the handle is OUT_PENDING or OUT;
 * MPRESS_ERR_ARG, MPRESS_ERR_ALIGN, MPRESS_ERR_CUDA.
 */
MPRESS_API int mpress_swap_in(mpress_ctx_t* ctx, mpress_handle_t* handle, void* const* dst,
                   void* stream);

/*
 * CUDA graph capture.  mpress_swap_out / mpress_swap_in / mpress_wait may be
 * called while their streams are being captured (cudaStreamBeginCapture,
 * torch.cuda.graph), so a pipeline step that swaps can be captured and
 * replayed as one graph launch (no per-swap host cost on the replay).  A
 * swap-out enqueued on a capturing stream makes a GRAPH HANDLE:
 *   - its stash slices are taken at capture time and stay held until
 *     mpress_handle_free (every replay writes and reads them again); eager
 *     swaps of the same context use other slices;
 *   - its swap-in must be captured into the same capture (else
 *     MPRESS_ERR_STATE), at most once; an eager handle cannot be swapped in
 *     under capture (MPRESS_ERR_STATE);
 *   - mpress_wait inside the capture joins the consumer stream on the
 *     capture's own event; outside it, waits for the latest replay;
 *   - mpress_query reports the latest replay's completion (1 before any
 *     replay) and does not advance the state; do not call it while a capture
 *     is running;
 *   - mpress_handle_free releases the slices, fenced by the latest replay's
 *     swap-in (force is needed if no swap-in was captured).  Free graph
 *     handles only once their graph will not be launched again.
 * Replays move the bytes the captured pointers hold at replay time.
 */

/* Make `consumer` wait (cudaStreamWaitEvent, enqueue-only) for the handle's
 * latest operation: the swap-out if no swap-in was issued, else the swap-in. */
MPRESS_API int mpress_wait(mpress_ctx_t* ctx, mpress_handle_t* handle, void* consumer);

/* Non-blocking: 1 = latest operation complete, 0 = pending, < 0 = error.
 * Advances the handle state (OUT_PENDING->OUT, IN_PENDING->IN). */
MPRESS_API int mpress_query(mpress_ctx_t* ctx, mpress_handle_t* handle);

/* Current state (MPRESS_STATE_*) without querying the device. */
MPRESS_API int mpress_handle_state(const mpress_handle_t* handle);

/* 1 if the handle's swap-out was captured into a CUDA graph (a graph handle,
 * see "CUDA graph capture" above), 0 if not, < 0 on error. */
MPRESS_API int mpress_handle_is_graph(const mpress_handle_t* handle);

/* Slice base of the handle inside this source's partition of each peer's
 * pool [world]; UINT64_MAX for peers the plan does not use (tests). */
MPRESS_API int mpress_handle_slices(const mpress_handle_t* handle, uint64_t* slice_off);

/* mpress_handle_free -- retire the tensor batch's metadata-table entry
 * (recorded before the swap-out, "used to guide the execution of the
 * latter swap-in operator and updated when it completes").  A handle still
 * OUT_PENDING or OUT (data only in the stash) is an error (MPRESS_ERR_STATE)
 * unless `force` is nonzero.  `force` is not in the paper (a deviation, see
 * DESIGN.md §9): it drops stashed data the caller no longer needs, e.g. when
 * a pipeline aborts a step.  An IN_PENDING handle may be freed: its slices
 * stay fenced by the swap-in event.  Errors: MPRESS_ERR_ARG (NULL, or a
 * handle of another context), MPRESS_ERR_STATE. */
MPRESS_API int mpress_handle_free(mpress_ctx_t* ctx, mpress_handle_t* handle, int force);

/* Debug / test: synchronous copy of `len` bytes at byte `offset` of this
 * source's partition on `peer` into host memory `host_dst`. */
MPRESS_API int mpress_peer_read(mpress_ctx_t* ctx, int peer, uint64_t offset, uint64_t len,
                     void* host_dst);

/* Debug / test: *out = this process's device address of byte `offset` of
 * this source's partition on `peer` (its peer mapping, P:211's "indices of
 * target GPU devices" resolved to memory), so a device-side checker can read
 * a whole stash slice in place without a host copy.  The address stays valid
 * until mpress_finalize; the bytes are defined only inside stripes of a
 * swapped-out handle.  Errors: MPRESS_ERR_ARG, MPRESS_ERR_PEER (not mapped). */
MPRESS_API int mpress_peer_ptr(const mpress_ctx_t* ctx, int peer, uint64_t offset, void** out);

/* Kernel launches the last swap_out / swap_in call enqueued (for accounting). */
MPRESS_API int mpress_last_launches(const mpress_ctx_t* ctx);

/* ---- utilities ---------------------------------------------------------------- */

/*
 * mpress_share_fds -- the fd-passing step of mpress_init, exposed for tests:
 * rank r offers `my_fd`; for every p with want[p] != 0 it receives a duplicate
 * of rank p's fd in fds_out[p] (else -1).  Collective; uses `exchange` for the
 * rendezvous and Unix-domain sockets with SCM_RIGHTS for the descriptors.
 * The caller closes the received descriptors.
 */
MPRESS_API int mpress_share_fds(int world, int rank, int my_fd, const int32_t* want,
                     mpress_exchange_fn exchange, void* exchange_user,
                     int32_t* fds_out);

MPRESS_API const char* mpress_last_error(void);
MPRESS_API int mpress_version(void);

#ifdef __cplusplus
}  /* extern "C" */
#endif
#endif  /* MPRESS_H_ */
