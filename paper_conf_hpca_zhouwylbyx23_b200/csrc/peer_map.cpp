// Peer-memory layer (SURVEY.md §8(a) row a2 "MAP"): stash pools carved from
// the importers' spare HBM (Fig. 6 line 3: spare = MEM_CAP - MEM_USE)
// and mapped into each exporter's address space so the swap kernels can load
// and store peer HBM directly over NVLink 5 / NVSwitch.
//
// The paper's memory manager takes swap space from PyTorch's allocator on the
// importer; here every importer reserves its pool once at init with
// the CUDA VMM API (cuMemCreate), so the peer's own training cannot consume
// it, and exports it as a POSIX fd; sources import + map + grant access.
// Each source owns a fixed partition of every pool (R21), so the hot path
// needs no cross-GPU lock or handshake.
#include <unistd.h>

#include <algorithm>
#include <cstdlib>
#include <cstring>
#include <mutex>

#include "ctx.h"
#include "swap_kernels.h"

namespace mpress {

int driver(const Driver** out) {
  static Driver d;
  static int rc = 1;
  static std::mutex mu;
  std::lock_guard<std::mutex> lk(mu);
  if (rc == 1) {
    rc = MPRESS_OK;
    struct Sym { const char* name; void** slot; } syms[] = {
        {"cuMemCreate", (void**)&d.mem_create},
        {"cuMemRelease", (void**)&d.mem_release},
        {"cuMemAddressReserve", (void**)&d.mem_address_reserve},
        {"cuMemAddressFree", (void**)&d.mem_address_free},
        {"cuMemMap", (void**)&d.mem_map},
        {"cuMemUnmap", (void**)&d.mem_unmap},
        {"cuMemSetAccess", (void**)&d.mem_set_access},
        {"cuMemExportToShareableHandle", (void**)&d.mem_export},
        {"cuMemImportFromShareableHandle", (void**)&d.mem_import},
        {"cuMemGetAllocationGranularity", (void**)&d.mem_granularity},
        {"cuGetErrorString", (void**)&d.get_error_string},
    };
    for (auto& s : syms) {
      cudaDriverEntryPointQueryResult q;
      cudaError_t e = cudaGetDriverEntryPoint(s.name, s.slot, cudaEnableDefault, &q);
      if (e != cudaSuccess || q != cudaDriverEntryPointSuccess || !*s.slot) {
        rc = fail(MPRESS_ERR_CUDA, "CUDA driver entry point %s unavailable (%s)", s.name,
                  cudaGetErrorString(e));
        break;
      }
    }
  }
  if (rc != MPRESS_OK) return rc;
  *out = &d;
  return MPRESS_OK;
}

int cu_fail(const Driver* d, CUresult r, const char* what) {
  const char* s = nullptr;
  if (d && d->get_error_string) d->get_error_string(r, &s);
  return fail(r == CUDA_ERROR_PEER_ACCESS_UNSUPPORTED || r == CUDA_ERROR_INVALID_DEVICE
                  ? MPRESS_ERR_PEER : MPRESS_ERR_CUDA,
              "%s: CUresult %d (%s)", what, (int)r, s ? s : "?");
}

namespace {

CUmemAllocationProp pool_prop(int owner_device, bool exportable) {
  CUmemAllocationProp prop;
  memset(&prop, 0, sizeof prop);
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = owner_device;
  prop.requestedHandleTypes = exportable ? CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR
                                         : CU_MEM_HANDLE_TYPE_NONE;
  return prop;
}

int granularity(const Driver* d, int owner_device, bool exportable, size_t* g) {
  CUmemAllocationProp prop = pool_prop(owner_device, exportable);
  CUresult r = d->mem_granularity(g, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED);
  if (r != CUDA_SUCCESS) return cu_fail(d, r, "cuMemGetAllocationGranularity");
  return MPRESS_OK;
}

// Reserve VA, map the handle, grant read/write to every device in `access`.
int map_handle(const Driver* d, Mapping* m, const int* access, int n_access) {
  CUresult r = d->mem_address_reserve(&m->va, m->size, 0, 0, 0);
  if (r != CUDA_SUCCESS) return cu_fail(d, r, "cuMemAddressReserve");
  m->reserved = true;
  r = d->mem_map(m->va, m->size, 0, m->handle, 0);
  if (r != CUDA_SUCCESS) return cu_fail(d, r, "cuMemMap");
  m->mapped = true;
  std::vector<CUmemAccessDesc> desc(n_access);
  for (int i = 0; i < n_access; ++i) {
    memset(&desc[i], 0, sizeof desc[i]);
    desc[i].location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    desc[i].location.id = access[i];
    desc[i].flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  }
  r = d->mem_set_access(m->va, m->size, desc.data(), desc.size());
  if (r != CUDA_SUCCESS) return cu_fail(d, r, "cuMemSetAccess (peer access over NVLink)");
  return MPRESS_OK;
}

void unmap(const Driver* d, Mapping* m) {
  if (m->mapped) d->mem_unmap(m->va, m->size);
  if (m->reserved) d->mem_address_free(m->va, m->size);
  if (m->has_handle) d->mem_release(m->handle);
  if (m->host) cudaFreeHost(m->host);
  if (m->ipc_opened) cudaIpcCloseMemHandle(m->ipc_opened);
  if (m->ipc_owned) cudaFree(m->ipc_owned);
  *m = Mapping();
}

// NEXT-4 (GPU-CPU swap tier): a "peer" whose pool is
// pinned host memory, allocated once ("a host pinned memory pool that is not
// part of the PyTorch runtime") and mapped into the device's address
// space, so the same stripes and kernels move bytes over PCIe.
int map_host_pool(Mapping* m, uint64_t bytes) {
  m->size = roundup(bytes, 2u << 20);
  cudaError_t e = cudaHostAlloc(&m->host, m->size, cudaHostAllocMapped | cudaHostAllocPortable);
  if (e != cudaSuccess) {
    m->host = nullptr;
    return fail(MPRESS_ERR_CUDA, "cudaHostAlloc (host stash pool, %llu B): %s", (unsigned long long)m->size,
                cudaGetErrorString(e));
  }
  void* dev = nullptr;
  e = cudaHostGetDevicePointer(&dev, m->host, 0);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "cudaHostGetDevicePointer: %s", cudaGetErrorString(e));
  m->va = reinterpret_cast<CUdeviceptr>(dev);
  return MPRESS_OK;
}

void destroy(mpress_ctx_s* c) {
  const Driver* d = nullptr;
  if (driver(&d) == MPRESS_OK) {
    for (auto& m : c->maps) unmap(d, &m);
    unmap(d, &c->own);
  }
  for (auto* h : c->handles) delete h;   // their events go back to the pool
  for (auto& p : c->parts) p.fences.clear();
  for (auto e : *c->ev_pool) cudaEventDestroy(e);
  c->ev_pool->clear();
  for (auto s : c->ce_streams) if (s) cudaStreamDestroy(s);
  table_ring_destroy(c->ring);
  counter_ring_destroy(c->counters);
  delete c;
}

void init_partition(mpress::Partition* part, uint8_t* base, uint64_t size) {
  part->base = base;
  part->size = size;
  part->free.clear();
  if (size) part->free[0] = size;
}

int check_partition(int world, const uint64_t* partition) {
  if (!partition) return fail(MPRESS_ERR_ARG, "partition is null");
  for (int s = 0; s < world; ++s) {
    if (partition[(size_t)s * world + s] != 0)
      return fail(MPRESS_ERR_ARG, "partition[%d][%d] != 0: a source cannot stash on itself", s, s);
    for (int p = 0; p < world; ++p)
      if (partition[(size_t)s * world + p] % MPRESS_ALIGN)
        return fail(MPRESS_ERR_ARG, "partition[%d][%d] is not a multiple of 256", s, p);
  }
  return MPRESS_OK;
}

}  // namespace
}  // namespace mpress

using namespace mpress;

extern "C" int mpress_init_local(int world, int source, const int* devices,
                                 const uint64_t* partition, mpress_ctx_t** out) {
  if (!out || !devices || world < 1 || source < 0 || source >= world)
    return fail(MPRESS_ERR_ARG, "mpress_init_local: bad argument");
  *out = nullptr;
  MP_TRY(check_partition(world, partition));
  if (devices[source] < 0) return fail(MPRESS_ERR_ARG, "mpress_init_local: the source must be a GPU");
  const Driver* d;
  MP_TRY(driver(&d));
  auto* c = new mpress_ctx_s();
  c->device = devices[source];
  c->world = world;
  c->source = source;
  c->local = true;
  c->partition.assign(partition, partition + (size_t)world * world);
  c->maps.resize(world);
  c->parts.resize(world);
  DeviceGuard g(c->device);
  if (cudaFree(nullptr) != cudaSuccess) {
    delete c;
    return fail(MPRESS_ERR_CUDA, "mpress_init_local: cannot initialise device %d", devices[source]);
  }
  for (int p = 0; p < world; ++p) {
    const uint64_t want = partition[(size_t)source * world + p];
    if (p == source || want == 0) continue;
    if (devices[p] == MPRESS_DEVICE_HOST) {
      const int rc = map_host_pool(&c->maps[p], want);
      c->host_peer = true;
      if (rc != MPRESS_OK) {
        destroy(c);
        return rc;
      }
      init_partition(&c->parts[p], reinterpret_cast<uint8_t*>(c->maps[p].va), want);
      continue;
    }
    size_t gran;
    int rc = granularity(d, devices[p], false, &gran);
    if (rc == MPRESS_OK) {
      Mapping& m = c->maps[p];
      m.size = roundup(want, gran);
      CUmemAllocationProp prop = pool_prop(devices[p], false);
      CUresult r = d->mem_create(&m.handle, m.size, &prop, 0);
      if (r != CUDA_SUCCESS) rc = cu_fail(d, r, "cuMemCreate (stash pool)");
      else {
        m.has_handle = true;
        int access[2] = {c->device, devices[p]};
        rc = map_handle(d, &m, access, devices[p] == c->device ? 1 : 2);
      }
    }
    if (rc != MPRESS_OK) {
      destroy(c);
      return rc;
    }
    init_partition(&c->parts[p], reinterpret_cast<uint8_t*>(c->maps[p].va), want);
  }
  int rc = preload_kernels();
  // claim counters of MPRESS_SPLIT_DYNAMIC / AUTO launches, zeroed here (a
  // blocking memset) so no swap call has to allocate or synchronise
  if (rc == MPRESS_OK) rc = counter_ring_create(c->device, &c->counters);
  if (rc != MPRESS_OK) {
    destroy(c);
    return rc;
  }
  *out = c;
  return MPRESS_OK;
}

namespace mpress {
namespace {

int init_vmm_fd(mpress_ctx_s* c, const Driver* d, int rc);

// All ranks learn whether every rank succeeded (a barrier as well).
int agree(mpress_ctx_s* c, int rc, const char* what) {
  int32_t ok = rc == MPRESS_OK;
  std::vector<int32_t> okv(c->world);
  if (c->exchange(c->exchange_user, &ok, sizeof ok, okv.data()) != 0)
    return rc != MPRESS_OK ? rc : fail(MPRESS_ERR_SYS, "mpress_init: exchange failed");
  for (int r = 0; r < c->world; ++r)
    if (!okv[r]) return rc != MPRESS_OK ? rc : fail(MPRESS_ERR_PEER, "mpress_init: rank %d failed to %s", r, what);
  return rc;
}

void reset_pools(mpress_ctx_s* c, const Driver* d) {
  for (auto& m : c->maps) unmap(d, &m);
  unmap(d, &c->own);
  for (auto& p : c->parts) p = Partition();
}

uint64_t partition_offset(const mpress_ctx_s* c, int p) {  // where my partition of p's pool starts
  uint64_t off = 0;
  for (int s = 0; s < c->source; ++s) off += c->partition[(size_t)s * c->world + p];
  return off;
}

// Transport 1 (fallback): the pools are cudaMalloc allocations shared with
// CUDA IPC handles, which travel through the all-gather itself (no sockets).
int init_legacy_ipc(mpress_ctx_s* c) {
  const int world = c->world, rank = c->source;
  uint64_t pool = 0;
  for (int s = 0; s < world; ++s) pool += c->partition[(size_t)s * world + rank];
  struct Info {
    cudaIpcMemHandle_t h;
    uint64_t size;
    int32_t ok, pad;
  } mine;
  memset(&mine, 0, sizeof mine);
  int rc = MPRESS_OK;
  if (pool > 0) {
    c->own.size = roundup(pool, 2u << 20);
    cudaError_t e = cudaMalloc(&c->own.ipc_owned, c->own.size);
    if (e == cudaSuccess) e = cudaIpcGetMemHandle(&mine.h, c->own.ipc_owned);
    if (e != cudaSuccess) rc = fail(MPRESS_ERR_CUDA, "CUDA IPC stash pool: %s", cudaGetErrorString(e));
  }
  mine.size = c->own.size;
  mine.ok = rc == MPRESS_OK;
  std::vector<Info> all(world);
  if (c->exchange(c->exchange_user, &mine, sizeof mine, all.data()) != 0 && rc == MPRESS_OK)
    rc = fail(MPRESS_ERR_SYS, "mpress_init: exchange failed");
  for (int r = 0; r < world && rc == MPRESS_OK; ++r)
    if (!all[r].ok) rc = fail(MPRESS_ERR_CUDA, "mpress_init: rank %d failed to create its pool", r);
  for (int p = 0; p < world && rc == MPRESS_OK; ++p) {
    const uint64_t want = c->partition[(size_t)rank * world + p];
    if (p == rank || want == 0) continue;
    Mapping& m = c->maps[p];
    cudaError_t e = cudaIpcOpenMemHandle(&m.ipc_opened, all[p].h, cudaIpcMemLazyEnablePeerAccess);
    if (e != cudaSuccess) {
      m.ipc_opened = nullptr;
      rc = fail(MPRESS_ERR_PEER, "cudaIpcOpenMemHandle (rank %d's pool): %s", p, cudaGetErrorString(e));
      break;
    }
    m.size = all[p].size;
    m.va = reinterpret_cast<CUdeviceptr>(m.ipc_opened);
    init_partition(&c->parts[p], reinterpret_cast<uint8_t*>(m.va) + partition_offset(c, p), want);
  }
  return rc;
}

}  // namespace
}  // namespace mpress

extern "C" int mpress_init(int device, int world, int rank, const uint64_t* partition,
                           mpress_exchange_fn exchange, void* exchange_user,
                           mpress_ctx_t** out) {
  if (!out || !exchange || world < 1 || rank < 0 || rank >= world || device < 0)
    return fail(MPRESS_ERR_ARG, "mpress_init: bad argument");
  *out = nullptr;
  MP_TRY(check_partition(world, partition));
  const Driver* d;
  MP_TRY(driver(&d));
  auto* c = new mpress_ctx_s();
  c->device = device;
  c->world = world;
  c->source = rank;
  c->exchange = exchange;
  c->exchange_user = exchange_user;
  c->partition.assign(partition, partition + (size_t)world * world);
  c->maps.resize(world);
  c->parts.resize(world);
  DeviceGuard g(device);
  int rc = cudaFree(nullptr) == cudaSuccess ? MPRESS_OK
                                            : fail(MPRESS_ERR_CUDA, "mpress_init: cannot initialise device %d", device);
  // MPRESS_IPC=legacy selects CUDA IPC handles from the start; otherwise the
  // cuMem + fd path runs first and all ranks fall back together if it fails.
  const char* ipc_env = getenv("MPRESS_IPC");
  if (ipc_env && strcmp(ipc_env, "legacy") == 0) {
    c->transport = MPRESS_TRANSPORT_LEGACY_IPC;
    rc = init_legacy_ipc(c);
  } else {
    rc = init_vmm_fd(c, d, rc);
    if (agree(c, rc, "map its peers") != MPRESS_OK) {
      reset_pools(c, d);
      c->transport = MPRESS_TRANSPORT_LEGACY_IPC;
      rc = init_legacy_ipc(c);
    }
  }
  if (rc == MPRESS_OK) rc = preload_kernels();
  if (rc == MPRESS_OK) rc = counter_ring_create(device, &c->counters);
  rc = agree(c, rc, "map its peers");
  if (rc != MPRESS_OK) {
    destroy(c);
    return rc;
  }
  *out = c;
  return MPRESS_OK;
}

namespace mpress {
namespace {

// Transport 0: cuMem pool exported as a POSIX fd, passed with SCM_RIGHTS,
// imported and mapped with peer access (no collective agreement here).
int init_vmm_fd(mpress_ctx_s* c, const Driver* d, int rc) {
  const int world = c->world, rank = c->source, device = c->device;
  const uint64_t* partition = c->partition.data();
  mpress_exchange_fn exchange = c->exchange;
  void* exchange_user = c->exchange_user;
  c->transport = MPRESS_TRANSPORT_VMM_FD;

  // 1. my pool = sum of every source's partition on me
  uint64_t pool = 0;
  for (int s = 0; s < world; ++s) pool += partition[(size_t)s * world + rank];
  int my_fd = -1;
  if (rc == MPRESS_OK && pool > 0) {
    size_t gran;
    rc = granularity(d, device, true, &gran);
    if (rc == MPRESS_OK) {
      c->own.size = roundup(pool, gran);
      CUmemAllocationProp prop = pool_prop(device, true);
      CUresult r = d->mem_create(&c->own.handle, c->own.size, &prop, 0);
      if (r != CUDA_SUCCESS) rc = cu_fail(d, r, "cuMemCreate (stash pool)");
      else {
        c->own.has_handle = true;
        r = d->mem_export(&my_fd, c->own.handle, CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR, 0);
        if (r != CUDA_SUCCESS) rc = cu_fail(d, r, "cuMemExportToShareableHandle");
      }
    }
  }

  // 2. all ranks learn every pool's mapped size (and whether everyone is OK)
  struct Info { uint64_t pool_size; int32_t ok; int32_t pad; } mine{c->own.size, rc == MPRESS_OK, 0};
  std::vector<Info> all(world);
  if (exchange(exchange_user, &mine, sizeof mine, all.data()) != 0 && rc == MPRESS_OK)
    rc = fail(MPRESS_ERR_SYS, "mpress_init: exchange failed");
  for (int r = 0; r < world && rc == MPRESS_OK; ++r)
    if (!all[r].ok) rc = fail(MPRESS_ERR_CUDA, "mpress_init: rank %d failed to create its pool", r);
  // Every rank must still take part in the fd exchange to keep the collective
  // sequence aligned; a failed rank offers nothing and wants nothing.
  std::vector<int32_t> want(world, 0), fds(world, -1);
  if (rc == MPRESS_OK)
    for (int p = 0; p < world; ++p) want[p] = (p != rank && partition[(size_t)rank * world + p] > 0);
  int rc2 = mpress_share_fds(world, rank, my_fd, want.data(), exchange, exchange_user, fds.data());
  if (my_fd >= 0) close(my_fd);
  if (rc == MPRESS_OK) rc = rc2;

  // 3. import, map, grant access to my device
  for (int p = 0; p < world && rc == MPRESS_OK; ++p) {
    if (!want[p]) continue;
    Mapping& m = c->maps[p];
    m.size = all[p].pool_size;
    CUresult r = d->mem_import(&m.handle, (void*)(uintptr_t)fds[p], CU_MEM_HANDLE_TYPE_POSIX_FILE_DESCRIPTOR);
    if (r != CUDA_SUCCESS) { rc = cu_fail(d, r, "cuMemImportFromShareableHandle"); break; }
    m.has_handle = true;
    rc = map_handle(d, &m, &device, 1);
    if (rc != MPRESS_OK) break;
    uint64_t off = 0;
    for (int s = 0; s < rank; ++s) off += partition[(size_t)s * world + p];
    init_partition(&c->parts[p], reinterpret_cast<uint8_t*>(m.va) + off,
                   partition[(size_t)rank * world + p]);
  }
  for (int p = 0; p < world; ++p)
    if (fds[p] >= 0) close(fds[p]);
  return rc;
}

}  // namespace
}  // namespace mpress

extern "C" int mpress_finalize(mpress_ctx_t* c) {
  if (!c) return MPRESS_OK;
  int rc = MPRESS_OK;
  {
    DeviceGuard g(c->device);
    cudaDeviceSynchronize();
    if (!c->local) {
      int32_t one = 1;
      std::vector<int32_t> all(c->world);
      if (c->exchange(c->exchange_user, &one, sizeof one, all.data()) != 0)
        rc = fail(MPRESS_ERR_SYS, "mpress_finalize: barrier failed");
    }
    destroy(c);
  }
  return rc;
}

extern "C" int mpress_stash_free(const mpress_ctx_t* c, uint64_t* free_bytes) {
  if (!c || !free_bytes) return fail(MPRESS_ERR_ARG, "mpress_stash_free: null argument");
  auto* cc = const_cast<mpress_ctx_s*>(c);
  std::lock_guard<std::mutex> lk(cc->mu);
  for (int p = 0; p < c->world; ++p) {
    uint64_t best = 0;
    for (auto& kv : c->parts[p].free) best = std::max(best, kv.second);
    free_bytes[p] = best;
  }
  return MPRESS_OK;
}

namespace mpress {

int set_swap_option(SwapOpts* o, int key, int64_t value) {
  switch (key) {
    case MPRESS_OPT_PATH:
      if (value != MPRESS_PATH_DIRECT && value != MPRESS_PATH_BULK && value != MPRESS_PATH_CE &&
          value != MPRESS_PATH_AUTO)
        return fail(MPRESS_ERR_ARG, "unknown path %lld", (long long)value);
      o->path = (int)value;
      o->variant = MPRESS_VARIANT_AUTO;  // variants are per path
      return MPRESS_OK;
    case MPRESS_OPT_MAX_CTAS:
      if (value < 0 || value > (1 << 20)) return fail(MPRESS_ERR_ARG, "bad max_ctas %lld", (long long)value);
      o->max_ctas = (int)value;
      return MPRESS_OK;
    case MPRESS_OPT_PDL:
      if (value < 0 || value > 2) return fail(MPRESS_ERR_ARG, "MPRESS_OPT_PDL is 0, 1 or 2, not %lld", (long long)value);
      o->pdl = (int)value;
      return MPRESS_OK;
    case MPRESS_OPT_ORDER:
      if (value != MPRESS_ORDER_INTERLEAVE && value != MPRESS_ORDER_PLAN)
        return fail(MPRESS_ERR_ARG, "unknown chunk order %lld", (long long)value);
      o->order = (int)value;
      return MPRESS_OK;
    case MPRESS_OPT_PACE_MBPS:
      if (value < 0 || value > (int64_t)100000000)
        return fail(MPRESS_ERR_ARG, "MPRESS_OPT_PACE_MBPS is 0 (off) or a rate in MB/s up to 1e8, not %lld",
                    (long long)value);
      o->pace_mbps = (uint64_t)value;
      return MPRESS_OK;
    case MPRESS_OPT_SPLIT:
      if (value < MPRESS_SPLIT_BLOCKED || value > MPRESS_SPLIT_AUTO)
        return fail(MPRESS_ERR_ARG, "MPRESS_OPT_SPLIT is 0 (blocked), 1 (strided), 2 (dynamic) or 3 (auto), not %lld",
                    (long long)value);
      o->split = (int)value;
      return MPRESS_OK;
    case MPRESS_OPT_VARIANT: {
      const int nvar = o->path == MPRESS_PATH_BULK ? kBulkVariants
                       : o->path == MPRESS_PATH_CE ? kCeVariants
                       : o->path == MPRESS_PATH_AUTO ? 0 : kDirectVariants;
      if (value != MPRESS_VARIANT_AUTO && (value < 0 || value >= nvar))
        return fail(MPRESS_ERR_ARG, "variant %lld out of range for path %d", (long long)value, o->path);
      o->variant = (int)value;
      return MPRESS_OK;
    }
  }
  return kNotSwapOption;
}

int get_swap_option(const SwapOpts& o, int key, int64_t* value) {
  switch (key) {
    case MPRESS_OPT_PATH: *value = o.path; return MPRESS_OK;
    case MPRESS_OPT_MAX_CTAS: *value = o.max_ctas; return MPRESS_OK;
    case MPRESS_OPT_VARIANT: *value = o.variant; return MPRESS_OK;
    case MPRESS_OPT_ORDER: *value = o.order; return MPRESS_OK;
    case MPRESS_OPT_PDL: *value = o.pdl; return MPRESS_OK;
    case MPRESS_OPT_PACE_MBPS: *value = (int64_t)o.pace_mbps; return MPRESS_OK;
    case MPRESS_OPT_SPLIT: *value = o.split; return MPRESS_OK;
  }
  return kNotSwapOption;
}

}  // namespace mpress

extern "C" int mpress_set_option(mpress_ctx_t* c, int key, int64_t value) {
  if (!c) return fail(MPRESS_ERR_ARG, "mpress_set_option: null ctx");
  std::lock_guard<std::mutex> lk(c->mu);
  const int rc = set_swap_option(&c->opt, key, value);
  return rc == kNotSwapOption ? fail(MPRESS_ERR_ARG, "unknown option %d", key) : rc;
}

extern "C" int mpress_get_option(const mpress_ctx_t* c, int key, int64_t* value) {
  if (!c || !value) return fail(MPRESS_ERR_ARG, "mpress_get_option: null argument");
  std::lock_guard<std::mutex> lk(const_cast<mpress_ctx_t*>(c)->mu);  // set_option/autotune/run_copy write these
  if (get_swap_option(c->opt, key, value) == MPRESS_OK) return MPRESS_OK;
  switch (key) {
    case MPRESS_OPT_TRANSPORT: *value = c->transport; return MPRESS_OK;
    case MPRESS_OPT_LAST_PATH: *value = c->last_path; return MPRESS_OK;
    case MPRESS_OPT_AUTO_OUT: *value = c->auto_path[mpress::kDirOut][1]; return MPRESS_OK;
    case MPRESS_OPT_AUTO_IN: *value = c->auto_path[mpress::kDirIn][1]; return MPRESS_OK;
    case MPRESS_OPT_AUTO_OUT_SMALL: *value = c->auto_path[mpress::kDirOut][0]; return MPRESS_OK;
    case MPRESS_OPT_AUTO_IN_SMALL: *value = c->auto_path[mpress::kDirIn][0]; return MPRESS_OK;
  }
  return fail(MPRESS_ERR_ARG, "unknown option %d", key);
}

extern "C" int mpress_peer_read(mpress_ctx_t* c, int peer, uint64_t offset, uint64_t len, void* host_dst) {
  if (!c || (!host_dst && len) || peer < 0 || peer >= c->world)
    return fail(MPRESS_ERR_ARG, "mpress_peer_read: bad argument");
  const Partition& part = c->parts[peer];
  if (!part.base) return fail(MPRESS_ERR_PEER, "mpress_peer_read: peer %d not mapped", peer);
  if (offset > part.size || len > part.size - offset)
    return fail(MPRESS_ERR_ARG, "mpress_peer_read: [%llu,+%llu) outside the partition (%llu B)",
                (unsigned long long)offset, (unsigned long long)len, (unsigned long long)part.size);
  DeviceGuard g(c->device);
  cudaError_t e = cudaMemcpy(host_dst, part.base + offset, len, cudaMemcpyDeviceToHost);
  if (e != cudaSuccess) return fail(MPRESS_ERR_CUDA, "mpress_peer_read: %s", cudaGetErrorString(e));
  return MPRESS_OK;
}

extern "C" int mpress_peer_ptr(const mpress_ctx_t* c, int peer, uint64_t offset, void** out) {
  if (!c || !out || peer < 0 || peer >= c->world) return fail(MPRESS_ERR_ARG, "mpress_peer_ptr: bad argument");
  *out = nullptr;
  const Partition& part = c->parts[peer];
  if (!part.base) return fail(MPRESS_ERR_PEER, "mpress_peer_ptr: peer %d not mapped", peer);
  if (offset > part.size)
    return fail(MPRESS_ERR_ARG, "mpress_peer_ptr: offset %llu outside the partition (%llu B)",
                (unsigned long long)offset, (unsigned long long)part.size);
  *out = part.base + offset;
  return MPRESS_OK;
}

extern "C" int mpress_last_launches(const mpress_ctx_t* c) { return c ? c->last_launches : 0; }
