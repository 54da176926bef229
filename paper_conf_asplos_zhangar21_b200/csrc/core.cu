// core.cu — host side of libvf.so: context, the type-based arena allocator
// (SharedOA, §4), the virtual range table (Fig. 3), TypePointer
// tagging (§6.1), and the C-ABI entry points declared in include/vf.h.
//
// B200 design: device memory only (no UVM objects, SURVEY A7 OUT). With
// reserve_va = 1 each (app, type) gets one reserved VA window
// (cuMemAddressReserve) and its doubling regions are mapped
// back-to-back inside it, so the paper's "merge contiguous regions" always
// fires and the COAL table has exactly one row per type. With reserve_va = 0
// every region is its own cudaMalloc and the table grows as
// T * ceil(log2(n/4096 + 1)) rows, reproducing the fragmented case.
#include <cuda.h>
#include <cuda_runtime.h>

#include <algorithm>
#include <atomic>
#include <cstdarg>
#include <cstdio>
#include <cstring>
#include <map>
#include <string>
#include <vector>

#include "vf_internal.h"

namespace vf {
static std::atomic<uint64_t> g_launches{0};
void note_launch(uint64_t k) { g_launches.fetch_add(k, std::memory_order_relaxed); }
Tuning& tuning() {
  static Tuning t;
  return t;
}

static const AppOps* app_ops(uint32_t app) {
  switch (app) {
    case VF_APP_MICRO: return app_micro();
    case VF_APP_GOL: return app_gol();
    case VF_APP_GEN: return app_gen();
    case VF_APP_GRAPH: return app_graph();
    case VF_APP_RAY: return app_ray();
    case VF_APP_TRAF: return app_traf();
    case VF_APP_NBODY: return app_nbody();
    case VF_APP_STUT: return app_stut();
    case VF_APP_COLLIDE: return app_collide();
    case VF_APP_GRAPH_EN: return app_graph_en();
    case VF_APP_EDGE: return app_edge();
  }
  return nullptr;
}

// ---- driver entry points (no link-time dependency on libcuda) -------------
struct Drv {
  decltype(&cuMemAddressReserve) reserve = nullptr;
  decltype(&cuMemAddressFree) addr_free = nullptr;
  decltype(&cuMemCreate) create = nullptr;
  decltype(&cuMemRelease) release = nullptr;
  decltype(&cuMemMap) map = nullptr;
  decltype(&cuMemUnmap) unmap = nullptr;
  decltype(&cuMemSetAccess) set_access = nullptr;
  decltype(&cuMemGetAllocationGranularity) granularity = nullptr;
  bool ok = false;
};

template <class F>
static bool get_entry(const char* name, F& f) {
  void* p = nullptr;
  cudaDriverEntryPointQueryResult q;
  if (cudaGetDriverEntryPoint(name, &p, cudaEnableDefault, &q) != cudaSuccess ||
      q != cudaDriverEntryPointSuccess || !p)
    return false;
  f = reinterpret_cast<F>(p);
  return true;
}

static Drv& drv() {
  static Drv d;
  static bool init = false;
  if (!init) {
    init = true;
    d.ok = get_entry("cuMemAddressReserve", d.reserve) && get_entry("cuMemAddressFree", d.addr_free) &&
           get_entry("cuMemCreate", d.create) && get_entry("cuMemRelease", d.release) &&
           get_entry("cuMemMap", d.map) && get_entry("cuMemUnmap", d.unmap) &&
           get_entry("cuMemSetAccess", d.set_access) &&
           get_entry("cuMemGetAllocationGranularity", d.granularity);
  }
  return d;
}

struct Arena {
  uint32_t app = 0, type = 0, obj_bytes = 0;
  uint64_t next_cap = 0;     // capacity (objects) of the next region
  int cur = -1;              // current region (index into ctx->regions)
  uint64_t used_bytes = 0;   // VMM: bytes of the window covered by regions
  CUdeviceptr va = 0;        // VMM window
  uint64_t va_size = 0;
  uint64_t mapped = 0;       // VMM: bytes mapped from the window start
  std::vector<CUmemGenericAllocationHandle> handles;
  std::vector<std::pair<CUdeviceptr, size_t>> maps;
};

struct AppTable {
  std::vector<vf_range> rows;
  uint64_t* d_start = nullptr;
  uint64_t* d_end = nullptr;
  uint32_t* d_type = nullptr;
  uint32_t d_cap = 0;
  uint32_t K = 0, P = 1;
  std::vector<uint64_t> vptr;
  uint64_t* d_vptr = nullptr;
  bool vptr_ready = false;
};

struct HeapBatch {
  uint32_t app;
  uint64_t* d_ptrs;  // untagged pointers, for delete
  uint64_t n;
};
}  // namespace vf

using namespace vf;

struct vf_ctx {
  vf_config cfg;
  std::string err;
  std::map<std::pair<uint32_t, uint32_t>, Arena> arenas;
  std::vector<vf_region> regions;
  std::vector<void*> region_malloc;  // non-VMM: cudaMalloc base per region (else null)
  std::vector<vf_range> all_rows;
  AppTable tables[VF_APP_COUNT];
  std::vector<HeapBatch> heap;
  std::vector<uint64_t> type_count[VF_APP_COUNT];  // live objects per (app, type)
  size_t gran = 2u << 20;
  // range tables replaced by a rebuild; freed only when no kernel can still
  // read them (vf_reset / vf_destroy, or after a device sync when many pile up)
  std::vector<void*> retired;
  // cuda_packed slabs (vf_alloc_packed), freed at vf_reset
  std::vector<void*> packed;
  // vf_dispatch_host: copy stream + one event per chunk (created on first use)
  cudaStream_t copy_stream = nullptr;
  std::vector<cudaEvent_t> chunk_events;
};

namespace {

vf_status fail(vf_ctx* c, vf_status s, const char* fmt, ...) {
  if (c) {
    char buf[512];
    va_list ap;
    va_start(ap, fmt);
    vsnprintf(buf, sizeof buf, fmt, ap);
    va_end(ap);
    c->err = buf;
  }
  return s;
}

#define CUDA_TRY(ctx, call)                                                                  \
  do {                                                                                       \
    cudaError_t _e = (call);                                                                 \
    if (_e != cudaSuccess)                                                                   \
      return fail(ctx, VF_ERR_CUDA, "%s: %s (%s:%d)", #call, cudaGetErrorString(_e), __FILE__, \
                  __LINE__);                                                                 \
  } while (0)

#define DRV_TRY(ctx, call)                                                                     \
  do {                                                                                         \
    CUresult _r = (call);                                                                      \
    if (_r != CUDA_SUCCESS)                                                                    \
      return fail(ctx, _r == CUDA_ERROR_OUT_OF_MEMORY ? VF_ERR_OOM : VF_ERR_CUDA,             \
                  "%s: CUresult %d (%s:%d)", #call, (int)_r, __FILE__, __LINE__);              \
  } while (0)

inline cudaStream_t S(void* s) { return reinterpret_cast<cudaStream_t>(s); }

uint64_t round_up(uint64_t x, uint64_t g) { return (x + g - 1) / g * g; }

vf_status set_device(vf_ctx* c) {
  CUDA_TRY(c, cudaSetDevice(c->cfg.device));
  return VF_OK;
}

// Ensure the (app,type) arena has a VA window (VMM mode).
vf_status ensure_window(vf_ctx* c, Arena& a) {
  if (a.va) return VF_OK;
  Drv& d = drv();
  if (!d.ok) return fail(c, VF_ERR_UNSUPPORTED, "CUDA VMM driver entry points unavailable");
  a.va_size = round_up(c->cfg.va_window_bytes, c->gran);
  DRV_TRY(c, d.reserve(&a.va, a.va_size, c->gran, 0, 0));
  return VF_OK;
}

vf_status map_upto(vf_ctx* c, Arena& a, uint64_t need_bytes) {
  if (need_bytes <= a.mapped) return VF_OK;
  if (need_bytes > a.va_size)
    return fail(c, VF_ERR_OOM, "type window of %llu bytes exhausted (need %llu)",
                (unsigned long long)a.va_size, (unsigned long long)need_bytes);
  Drv& d = drv();
  const uint64_t sz = round_up(need_bytes - a.mapped, c->gran);
  CUmemAllocationProp prop = {};
  prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
  prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  prop.location.id = c->cfg.device;
  CUmemGenericAllocationHandle h;
  DRV_TRY(c, d.create(&h, sz, &prop, 0));
  CUresult r = d.map(a.va + a.mapped, sz, 0, h, 0);
  if (r != CUDA_SUCCESS) {
    d.release(h);
    return fail(c, VF_ERR_CUDA, "cuMemMap failed: %d", (int)r);
  }
  CUmemAccessDesc acc = {};
  acc.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
  acc.location.id = c->cfg.device;
  acc.flags = CU_MEM_ACCESS_FLAGS_PROT_READWRITE;
  DRV_TRY(c, d.set_access(a.va + a.mapped, sz, &acc, 1));
  a.handles.push_back(h);
  a.maps.push_back({a.va + a.mapped, sz});
  a.mapped += sz;
  return VF_OK;
}

// New region of a.next_cap objects (start at init_chunk, double).
vf_status new_region(vf_ctx* c, Arena& a) {
  if (a.next_cap == 0) a.next_cap = c->cfg.init_chunk_objs ? c->cfg.init_chunk_objs : 4096;
  const uint64_t cap = a.next_cap;
  const uint64_t bytes = cap * a.obj_bytes;
  uint64_t start = 0;
  void* mb = nullptr;
  if (c->cfg.reserve_va) {
    vf_status s = ensure_window(c, a);
    if (s) return s;
    s = map_upto(c, a, a.used_bytes + bytes);
    if (s) return s;
    start = a.va + a.used_bytes;
    a.used_bytes += bytes;
  } else {
    cudaError_t e = cudaMalloc(&mb, bytes);
    if (e != cudaSuccess) {
      cudaGetLastError();
      return fail(c, VF_ERR_OOM, "cudaMalloc(%llu) for a region: %s", (unsigned long long)bytes,
                  cudaGetErrorString(e));
    }
    start = reinterpret_cast<uint64_t>(mb);
  }
  vf_region r = {};
  r.start = start;
  r.cap_objs = cap;
  r.used_objs = 0;
  r.obj_bytes = a.obj_bytes;
  r.type_id = a.type;
  r.app = a.app;
  c->regions.push_back(r);
  c->region_malloc.push_back(mb);
  a.cur = (int)c->regions.size() - 1;
  a.next_cap = cap * 2;  // reading G3: double the previous region of this type
  return VF_OK;
}

const uint64_t kTagMask = ~((1ull << VF_VA_BITS) - 1);

vf_status tag_check(vf_ctx* c, uint64_t addr) {
  if (addr & kTagMask)
    return fail(c, VF_ERR_TAG_BITS, "address 0x%llx uses bits 63:%u (TypePointer needs them 0)",
                (unsigned long long)addr, VF_VA_BITS);
  return VF_OK;
}

// Reserve `count` consecutive-in-allocation-order slots of (app,type); appends
// their runs as segments (first rank, first address) to `out`, ranks counted
// from `rank0`.
vf_status alloc_segments(vf_ctx* c, uint32_t app, uint32_t type, uint64_t count, uint64_t rank0,
                         std::vector<PlaceSeg>& out) {
  const AppOps* ops = app_ops(app);
  Arena& a = c->arenas[{app, type}];
  if (a.obj_bytes == 0) {
    a.app = app;
    a.type = type;
    a.obj_bytes = ops->obj_bytes[type];
  }
  while (count > 0) {
    if (a.cur < 0 || c->regions[a.cur].used_objs == c->regions[a.cur].cap_objs) {
      vf_status s = new_region(c, a);
      if (s) return s;
    }
    vf_region& r = c->regions[a.cur];
    const uint64_t take = std::min(count, r.cap_objs - r.used_objs);
    const uint64_t first = r.start + r.used_objs * r.obj_bytes;
    vf_status s = tag_check(c, first);
    if (!s) s = tag_check(c, first + take * r.obj_bytes - 1);
    if (s) return s;
    out.push_back(PlaceSeg{rank0, first, r.obj_bytes});
    r.used_objs += take;
    rank0 += take;
    count -= take;
  }
  return VF_OK;
}

vf_status ensure_vptrs(vf_ctx* c, uint32_t app) {
  AppTable& t = c->tables[app];
  if (t.vptr_ready) return VF_OK;
  const AppOps* ops = app_ops(app);
  if (!t.d_vptr) CUDA_TRY(c, cudaMalloc(&t.d_vptr, sizeof(uint64_t) * ops->ntypes));
  CUDA_TRY(c, ops->probe_vptrs(t.d_vptr, 0));
  t.vptr.resize(ops->ntypes);
  CUDA_TRY(c, cudaMemcpy(t.vptr.data(), t.d_vptr, sizeof(uint64_t) * ops->ntypes,
                         cudaMemcpyDeviceToHost));
  t.vptr_ready = true;
  return VF_OK;
}

// Fig. 3 / P:987-991: sort the app's regions by start, merge exactly-adjacent
// regions of the same type, upload the table for COAL.
vf_status rebuild_table(vf_ctx* c, uint32_t app, cudaStream_t stream) {
  vf_status s = ensure_vptrs(c, app);
  if (s) return s;
  AppTable& t = c->tables[app];
  std::vector<const vf_region*> rs;
  for (const vf_region& r : c->regions)
    if (r.app == app) rs.push_back(&r);
  std::sort(rs.begin(), rs.end(), [](const vf_region* x, const vf_region* y) { return x->start < y->start; });
  t.rows.clear();
  for (const vf_region* r : rs) {
    const uint64_t e = r->start + r->cap_objs * r->obj_bytes;
    if (!t.rows.empty() && t.rows.back().type_id == r->type_id && t.rows.back().end == r->start) {
      t.rows.back().end = e;
    } else {
      vf_range row = {r->start, e, r->type_id, app, t.vptr[r->type_id]};
      t.rows.push_back(row);
    }
  }
  t.K = (uint32_t)t.rows.size();
  t.P = 1;
  while (t.P < t.K) t.P *= 2;
  // Versioned device table: a new upload never overwrites rows a COAL kernel
  // still running on another stream may be reading; the old version is
  // retired and freed once the device is known idle. Uploaded on `stream`.
  if (t.d_start) {
    c->retired.push_back(t.d_start);
    t.d_start = t.d_end = nullptr;
    t.d_type = nullptr;
  }
  if (t.K) {
    const size_t bytes = 20ull * t.K;
    std::vector<unsigned char> host(bytes);
    uint64_t* hs = reinterpret_cast<uint64_t*>(host.data());
    uint64_t* he = hs + t.K;
    uint32_t* ht = reinterpret_cast<uint32_t*>(he + t.K);
    for (uint32_t j = 0; j < t.K; ++j) {
      hs[j] = t.rows[j].start;
      he[j] = t.rows[j].end;
      ht[j] = t.rows[j].type_id;
    }
    void* d = nullptr;
    CUDA_TRY(c, cudaMalloc(&d, bytes));
    t.d_start = static_cast<uint64_t*>(d);
    t.d_end = t.d_start + t.K;
    t.d_type = reinterpret_cast<uint32_t*>(t.d_end + t.K);
    CUDA_TRY(c, cudaMemcpyAsync(d, host.data(), bytes, cudaMemcpyHostToDevice, stream));
    CUDA_TRY(c, cudaStreamSynchronize(stream));  // `host` goes out of scope
  }
  t.d_cap = t.K;
  if (c->retired.size() > 64) {
    CUDA_TRY(c, cudaDeviceSynchronize());
    for (void* p : c->retired) cudaFree(p);
    c->retired.clear();
  }
  c->all_rows.clear();
  for (uint32_t a = 0; a < VF_APP_COUNT; ++a)
    c->all_rows.insert(c->all_rows.end(), c->tables[a].rows.begin(), c->tables[a].rows.end());
  std::sort(c->all_rows.begin(), c->all_rows.end(),
            [](const vf_range& x, const vf_range& y) { return x.start < y.start; });
  return VF_OK;
}

DevTable dev_table(vf_ctx* c, uint32_t app) {
  AppTable& t = c->tables[app];
  DevTable d;
  d.start = t.d_start;
  d.end = t.d_end;
  d.type = t.d_type;
  d.K = t.K;
  d.P = t.P;
  d.vptr = t.d_vptr;
  d.ntypes = app_ops(app)->ntypes;
  d.active_types = 0;
  for (uint64_t k : c->type_count[app]) d.active_types += (k != 0);
  d.inl = t.K <= kTableInline && (int)t.K <= tuning().coal_inline ? 1u : 0u;
  for (uint32_t j = 0; j < kTableInline; ++j) {
    const bool v = j < t.K && t.K <= kTableInline;  // (rows are filled whenever they fit)
    d.in_start[j] = v ? t.rows[j].start : ~0ull;
    d.in_len[j] = v ? t.rows[j].end - t.rows[j].start : 0ull;
    d.in_type[j] = v ? t.rows[j].type_id : VF_NOT_FOUND;
  }
  return d;
}

vf_status check_app(vf_ctx* c, uint32_t app) {
  if (!c) return VF_ERR_INVALID;
  if (!app_ops(app)) return fail(c, VF_ERR_INVALID, "unknown app %u", app);
  return VF_OK;
}

inline uint64_t tag_ptr(uint64_t addr, uint32_t type) {
  return addr | ((uint64_t)(type + 1) << VF_VA_BITS);
}

}  // namespace

extern "C" {

void vf_config_default(vf_config* cfg) {
  if (!cfg) return;
  cfg->device = 0;
  cfg->init_chunk_objs = 4096;
  cfg->reserve_va = 1;
  cfg->va_window_bytes = 64ull << 30;
  cfg->cuda_heap_bytes = 8ull << 30;
}

const char* vf_status_str(vf_status s) {
  switch (s) {
    case VF_OK: return "VF_OK";
    case VF_ERR_INVALID: return "VF_ERR_INVALID";
    case VF_ERR_OOM: return "VF_ERR_OOM";
    case VF_ERR_CUDA: return "VF_ERR_CUDA";
    case VF_ERR_TAG_BITS: return "VF_ERR_TAG_BITS";
    case VF_ERR_TOO_MANY_TYPES: return "VF_ERR_TOO_MANY_TYPES";
    case VF_ERR_TABLE_FULL: return "VF_ERR_TABLE_FULL";
    case VF_ERR_UNSUPPORTED: return "VF_ERR_UNSUPPORTED";
  }
  return "VF_ERR_?";
}

const char* vf_last_error(const vf_ctx* c) { return c ? c->err.c_str() : "null ctx"; }

uint64_t vf_launch_count(void) { return g_launches.load(); }

vf_status vf_set_tuning(const char* key, int value) {
  if (!key) return VF_ERR_INVALID;
  if (!strcmp(key, "unroll")) {
    if (value != -1 && value != 1 && value != 2 && value != 4) return VF_ERR_INVALID;
    tuning().unroll = value;
  } else if (!strcmp(key, "prefetch")) {
    if (value < -1 || value > 3) return VF_ERR_INVALID;
    tuning().prefetch = value;
  } else if (!strcmp(key, "regroup")) {
    if (value < 0 || value > 2) return VF_ERR_INVALID;
    tuning().regroup = value;
  } else if (!strcmp(key, "pipeline")) {
    if (value < 0 || value > 1) return VF_ERR_INVALID;
    tuning().pipeline = value;
  } else if (!strcmp(key, "call")) {
    if (value < 0 || value > 1) return VF_ERR_INVALID;
    tuning().call = value;
  } else if (!strcmp(key, "persistent")) {
    if (value < -1 || value > 1) return VF_ERR_INVALID;
    tuning().persistent = value;
  } else if (!strcmp(key, "cluster")) {
    if (value < 0 || value > 1) return VF_ERR_INVALID;
    tuning().cluster = value;
  } else if (!strcmp(key, "coal_inline")) {
    if (value < 0 || value > (int)kTableInline) return VF_ERR_INVALID;
    tuning().coal_inline = value;
  } else if (!strcmp(key, "gsort")) {
    if (value < -1 || value > 1) return VF_ERR_INVALID;
    tuning().gsort = value;
  } else if (!strcmp(key, "ray_rays")) {
    if (value != 2 && value != 4) return VF_ERR_INVALID;
    tuning().ray_rays = value;
  } else if (!strcmp(key, "ray_parts")) {
    if (value != -1 && (value < 1 || value > 16)) return VF_ERR_INVALID;
    tuning().ray_parts = value;
  } else {
    return VF_ERR_INVALID;
  }
  return VF_OK;
}

vf_status vf_app_info(uint32_t app, uint32_t* ntypes, uint32_t* obj_bytes, uint32_t* nmethods) {
  const AppOps* ops = app_ops(app);
  if (!ops) return VF_ERR_INVALID;
  if (ntypes) *ntypes = ops->ntypes;
  if (nmethods) *nmethods = ops->nmethods;
  if (obj_bytes)
    for (uint32_t k = 0; k < ops->ntypes; ++k) obj_bytes[k] = ops->obj_bytes[k];
  return VF_OK;
}

vf_status vf_create(const vf_config* cfg, vf_ctx** out) {
  if (!out) return VF_ERR_INVALID;
  *out = nullptr;
  vf_ctx* c = new vf_ctx();
  if (cfg) c->cfg = *cfg;
  else vf_config_default(&c->cfg);
  if (c->cfg.init_chunk_objs == 0) c->cfg.init_chunk_objs = 4096;
  if (c->cfg.va_window_bytes == 0) c->cfg.va_window_bytes = 64ull << 30;
  int ndev = 0;
  cudaError_t e = cudaGetDeviceCount(&ndev);
  if (e != cudaSuccess || c->cfg.device < 0 || c->cfg.device >= ndev) {
    cudaGetLastError();
    delete c;
    return e != cudaSuccess ? VF_ERR_CUDA : VF_ERR_INVALID;
  }
  if (cudaSetDevice(c->cfg.device) != cudaSuccess || cudaFree(0) != cudaSuccess) {
    delete c;
    return VF_ERR_CUDA;
  }
  if (c->cfg.reserve_va) {
    Drv& d = drv();
    if (!d.ok) {
      delete c;
      return VF_ERR_UNSUPPORTED;
    }
    CUmemAllocationProp prop = {};
    prop.type = CU_MEM_ALLOCATION_TYPE_PINNED;
    prop.location.type = CU_MEM_LOCATION_TYPE_DEVICE;
    prop.location.id = c->cfg.device;
    size_t g = 0;
    if (d.granularity(&g, &prop, CU_MEM_ALLOC_GRANULARITY_RECOMMENDED) == CUDA_SUCCESS && g)
      c->gran = g;
  }
  // Stream-ordered scratch (cudaMallocAsync: batched allocation, the grid-level
  // type sort) comes from the device's default pool; keep what it has mapped
  // instead of returning it at every synchronisation (threshold 0 would make
  // each dispatch re-map its scratch).
  {
    cudaMemPool_t pool;
    if (cudaDeviceGetDefaultMemPool(&pool, c->cfg.device) == cudaSuccess) {
      uint64_t keep = ~0ull;
      cudaMemPoolSetAttribute(pool, cudaMemPoolAttrReleaseThreshold, &keep);
    }
    cudaGetLastError();
  }
  // Device heap for the CUDA baseline. The limit can only grow
  // before the first device-malloc kernel of the process; failure here is
  // reported later by vf_alloc_cuda.
  if (c->cfg.cuda_heap_bytes) {
    size_t cur = 0;
    cudaDeviceGetLimit(&cur, cudaLimitMallocHeapSize);
    if (cur < c->cfg.cuda_heap_bytes) {
      if (cudaDeviceSetLimit(cudaLimitMallocHeapSize, c->cfg.cuda_heap_bytes) != cudaSuccess)
        cudaGetLastError();
    }
  }
  *out = c;
  return VF_OK;
}

vf_status vf_reset(vf_ctx* c) {
  if (!c) return VF_ERR_INVALID;
  vf_status st = set_device(c);
  if (st) return st;
  CUDA_TRY(c, cudaDeviceSynchronize());
  for (HeapBatch& h : c->heap) {
    app_ops(h.app)->delete_cuda(h.d_ptrs, h.n, 0);
    cudaDeviceSynchronize();
    cudaFree(h.d_ptrs);
  }
  c->heap.clear();
  for (void* p : c->retired) cudaFree(p);
  c->retired.clear();
  for (void* p : c->packed) cudaFree(p);
  c->packed.clear();
  for (size_t r = 0; r < c->region_malloc.size(); ++r)
    if (c->region_malloc[r]) cudaFree(c->region_malloc[r]);
  Drv& d = drv();
  for (auto& kv : c->arenas) {
    Arena& a = kv.second;
    for (auto& m : a.maps) d.unmap(m.first, m.second);
    for (auto h : a.handles) d.release(h);
    a.maps.clear();
    a.handles.clear();
    a.mapped = 0;
    a.used_bytes = 0;
    a.cur = -1;
    a.next_cap = 0;
  }
  c->regions.clear();
  c->region_malloc.clear();
  c->all_rows.clear();
  for (uint32_t app = 0; app < VF_APP_COUNT; ++app) {
    c->type_count[app].clear();
    c->tables[app].rows.clear();
    c->tables[app].K = 0;
    c->tables[app].P = 1;
  }
  return VF_OK;
}

void vf_destroy(vf_ctx* c) {
  if (!c) return;
  vf_reset(c);
  Drv& d = drv();
  for (auto& kv : c->arenas)
    if (kv.second.va) d.addr_free(kv.second.va, kv.second.va_size);
  for (AppTable& t : c->tables) {
    cudaFree(t.d_start);  // one allocation holds start, end and type
    cudaFree(t.d_vptr);
  }
  for (void* p : c->retired) cudaFree(p);
  for (cudaEvent_t e : c->chunk_events) cudaEventDestroy(e);
  if (c->copy_stream) cudaStreamDestroy(c->copy_stream);
  delete c;
}

vf_status vf_alloc_typed_batch(vf_ctx* c, uint32_t app, const uint32_t* type_ids_dev,
                               uint64_t count, const void* ctor_args_dev, uint32_t ctor_arg_bytes,
                               uint64_t* out_ptrs_dev, int tag, void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if (count == 0) return VF_OK;
  if (!type_ids_dev || !out_ptrs_dev) return fail(c, VF_ERR_INVALID, "null device pointer");
  if ((st = set_device(c))) return st;
  const AppOps* ops = app_ops(app);
  if (ops->ntypes > 32) return fail(c, VF_ERR_TOO_MANY_TYPES, "device ranking handles <= 32 types");
  cudaStream_t s = S(stream);
  // (1) per-type exclusive prefix counts on the device (alloc.cu); only the
  // T totals come back to the host, which sizes and maps the regions
  const uint64_t nch = rank_chunks(count);
  unsigned char* scratch = nullptr;
  const size_t hist_bytes = 128ull * nch;
  CUDA_TRY(c, cudaMallocAsync(reinterpret_cast<void**>(&scratch), hist_bytes + 8 * 32 + 16, s));
  uint32_t* hist = reinterpret_cast<uint32_t*>(scratch);
  unsigned long long* totals = reinterpret_cast<unsigned long long*>(scratch + hist_bytes);
  uint32_t* bad = reinterpret_cast<uint32_t*>(scratch + hist_bytes + 8 * 32);
  struct Guard {
    unsigned char* p;
    cudaStream_t s;
    ~Guard() { cudaFreeAsync(p, s); }
  } guard{scratch, s};
  CUDA_TRY(c, cudaMemsetAsync(bad, 0, 4, s));
  CUDA_TRY(c, rank_hist(type_ids_dev, count, ops->ntypes, hist, bad, totals, s));
  unsigned long long h_tot[32] = {0};
  uint32_t h_bad = 0;
  CUDA_TRY(c, cudaMemcpyAsync(h_tot, totals, 8ull * ops->ntypes, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(c, cudaMemcpyAsync(&h_bad, bad, 4, cudaMemcpyDeviceToHost, s));
  CUDA_TRY(c, cudaStreamSynchronize(s));
  if (h_bad) return fail(c, VF_ERR_INVALID, "a type id >= ntypes %u", ops->ntypes);
  if (tag && ops->ntypes > 127) return fail(c, VF_ERR_TOO_MANY_TYPES, "7-bit tag holds 127 types");
  // (2) regions: each type's slots as segments (rank range -> first address)
  std::vector<PlaceSeg> segs;
  std::vector<uint32_t> first(ops->ntypes + 1, 0);
  for (uint32_t t = 0; t < ops->ntypes; ++t) {
    first[t] = (uint32_t)segs.size();
    if (h_tot[t] && (st = alloc_segments(c, app, t, h_tot[t], 0, segs))) return st;
  }
  first[ops->ntypes] = (uint32_t)segs.size();
  c->type_count[app].resize(ops->ntypes, 0);
  for (uint32_t t = 0; t < ops->ntypes; ++t) c->type_count[app][t] += h_tot[t];
  // (3) place every object at its slot (device), then construct it there
  const size_t seg_bytes = sizeof(PlaceSeg) * segs.size(), first_bytes = 4ull * first.size();
  unsigned char* d_seg = nullptr;
  CUDA_TRY(c, cudaMallocAsync(reinterpret_cast<void**>(&d_seg), seg_bytes + first_bytes, s));
  Guard guard2{d_seg, s};
  CUDA_TRY(c, cudaMemcpyAsync(d_seg, segs.data(), seg_bytes, cudaMemcpyHostToDevice, s));
  CUDA_TRY(c, cudaMemcpyAsync(d_seg + seg_bytes, first.data(), first_bytes, cudaMemcpyHostToDevice, s));
  CUDA_TRY(c, rank_place(type_ids_dev, count, hist, reinterpret_cast<const PlaceSeg*>(d_seg),
                         reinterpret_cast<const uint32_t*>(d_seg + seg_bytes), tag, out_ptrs_dev, s));
  CUDA_TRY(c, ops->construct(type_ids_dev, out_ptrs_dev, ctor_args_dev, ctor_arg_bytes, count, s));
  CUDA_TRY(c, cudaStreamSynchronize(s));
  return rebuild_table(c, app, s);
}

vf_status vf_alloc_typed(vf_ctx* c, uint32_t app, uint32_t type_id, uint64_t count,
                         const void* ctor_args_dev, uint32_t ctor_arg_bytes, uint64_t* out_ptrs_dev,
                         int tag, void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if (type_id >= app_ops(app)->ntypes) return fail(c, VF_ERR_INVALID, "type id %u", type_id);
  if (count == 0) return VF_OK;
  if ((st = set_device(c))) return st;
  uint32_t* d_types = nullptr;
  CUDA_TRY(c, cudaMallocAsync(&d_types, 4ull * count, S(stream)));
  cudaError_t e = fill_u32(d_types, count, type_id, S(stream));
  if (e == cudaSuccess)
    st = vf_alloc_typed_batch(c, app, d_types, count, ctor_args_dev, ctor_arg_bytes, out_ptrs_dev,
                              tag, stream);
  cudaFreeAsync(d_types, S(stream));
  cudaStreamSynchronize(S(stream));
  if (e != cudaSuccess) return fail(c, VF_ERR_CUDA, "%s", cudaGetErrorString(e));
  return st;
}

vf_status vf_alloc_packed(vf_ctx* c, uint32_t app, const uint32_t* type_ids_dev, uint64_t count,
                          const void* ctor_args_dev, uint32_t ctor_arg_bytes, uint64_t* out_ptrs_dev,
                          void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if (count == 0) return VF_OK;
  if (!type_ids_dev || !out_ptrs_dev) return fail(c, VF_ERR_INVALID, "null device pointer");
  if ((st = set_device(c))) return st;
  const AppOps* ops = app_ops(app);
  uint64_t stride = 0;
  for (uint32_t t = 0; t < ops->ntypes; ++t) stride = std::max<uint64_t>(stride, ops->obj_bytes[t]);
  stride = (stride + 15) & ~15ull;
  void* slab = nullptr;
  cudaError_t e = cudaMalloc(&slab, stride * count);
  if (e != cudaSuccess) {
    cudaGetLastError();
    return fail(c, VF_ERR_OOM, "cudaMalloc(%llu) for a packed slab: %s",
                (unsigned long long)(stride * count), cudaGetErrorString(e));
  }
  c->packed.push_back(slab);
  cudaStream_t s = S(stream);
  CUDA_TRY(c, place_packed(reinterpret_cast<uint64_t>(slab), stride, count, out_ptrs_dev, s));
  CUDA_TRY(c, ops->construct(type_ids_dev, out_ptrs_dev, ctor_args_dev, ctor_arg_bytes, count, s));
  CUDA_TRY(c, cudaStreamSynchronize(s));
  c->type_count[app].resize(ops->ntypes, 0);
  c->type_count[app][0] += count;  // types unknown on the host: marks the app live (launch heuristics)
  return ensure_vptrs(c, app);
}

vf_status vf_alloc_cuda(vf_ctx* c, uint32_t app, const uint32_t* type_ids_dev, uint64_t count,
                        const void* ctor_args_dev, uint32_t ctor_arg_bytes, uint64_t* out_ptrs_dev,
                        int tag, void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if (count == 0) return VF_OK;
  if (!type_ids_dev || !out_ptrs_dev) return fail(c, VF_ERR_INVALID, "null device pointer");
  if ((st = set_device(c))) return st;
  const AppOps* ops = app_ops(app);
  if (tag && ops->ntypes > 127) return fail(c, VF_ERR_TOO_MANY_TYPES, "7-bit tag holds 127 types");
  CUDA_TRY(c, ops->new_cuda(type_ids_dev, ctor_args_dev, ctor_arg_bytes, count, out_ptrs_dev, S(stream)));
  CUDA_TRY(c, cudaStreamSynchronize(S(stream)));
  std::vector<uint64_t> ptrs(count);
  CUDA_TRY(c, cudaMemcpy(ptrs.data(), out_ptrs_dev, 8ull * count, cudaMemcpyDeviceToHost));
  uint64_t nulls = 0;
  for (uint64_t p : ptrs) nulls += (p == 0);
  // keep an untagged copy for delete
  HeapBatch hb{app, nullptr, count};
  CUDA_TRY(c, cudaMalloc(&hb.d_ptrs, 8ull * count));
  CUDA_TRY(c, cudaMemcpy(hb.d_ptrs, out_ptrs_dev, 8ull * count, cudaMemcpyDeviceToDevice));
  c->heap.push_back(hb);
  if (nulls)
    return fail(c, VF_ERR_OOM, "device heap exhausted: %llu of %llu `new` returned null (raise cuda_heap_bytes before the first device-malloc kernel)",
                (unsigned long long)nulls, (unsigned long long)count);
  for (uint64_t p : ptrs)
    if ((st = tag_check(c, p))) return st;
  std::vector<uint32_t> types(count);
  CUDA_TRY(c, cudaMemcpy(types.data(), type_ids_dev, 4ull * count, cudaMemcpyDeviceToHost));
  c->type_count[app].resize(ops->ntypes, 0);
  for (uint32_t t : types)
    if (t < ops->ntypes) ++c->type_count[app][t];
  if (tag) {
    for (uint64_t i = 0; i < count; ++i) ptrs[i] = tag_ptr(ptrs[i], types[i]);
    CUDA_TRY(c, cudaMemcpy(out_ptrs_dev, ptrs.data(), 8ull * count, cudaMemcpyHostToDevice));
  }
  return ensure_vptrs(c, app);
}

vf_status vf_range_table(const vf_ctx* c, uint32_t app, const vf_range** out, uint32_t* n) {
  if (!c || !out || !n) return VF_ERR_INVALID;
  if (app == 0xFFFFFFFFu) {
    *out = c->all_rows.data();
    *n = (uint32_t)c->all_rows.size();
    return VF_OK;
  }
  if (app >= VF_APP_COUNT) return VF_ERR_INVALID;
  *out = c->tables[app].rows.data();
  *n = (uint32_t)c->tables[app].rows.size();
  return VF_OK;
}

vf_status vf_regions(const vf_ctx* c, const vf_region** out, uint32_t* n) {
  if (!c || !out || !n) return VF_ERR_INVALID;
  *out = c->regions.data();
  *n = (uint32_t)c->regions.size();
  return VF_OK;
}

vf_status vf_type_vptrs(vf_ctx* c, uint32_t app, uint64_t* vptrs_out) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if ((st = set_device(c)) || (st = ensure_vptrs(c, app))) return st;
  if (vptrs_out)
    std::copy(c->tables[app].vptr.begin(), c->tables[app].vptr.end(), vptrs_out);
  return VF_OK;
}

vf_status vf_resolve(vf_ctx* c, uint32_t app, vf_variant v, const uint64_t* ptrs_dev, uint64_t n,
                     uint32_t* types_out_dev, void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if ((unsigned)v > VF_CONCORD) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if ((st = set_device(c)) || (st = ensure_vptrs(c, app))) return st;
  if (v == VF_COAL && c->tables[app].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[app].K, VF_MAX_RANGES);
  CUDA_TRY(c, app_ops(app)->resolve((int)v, ptrs_dev, n, types_out_dev, dev_table(c, app), S(stream)));
  return VF_OK;
}

vf_status vf_verify_types(vf_ctx* c, uint32_t app, vf_variant v, const uint64_t* ptrs_dev,
                          uint64_t n, unsigned long long* mism_dev, void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if ((unsigned)v > VF_CONCORD) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if ((st = set_device(c)) || (st = ensure_vptrs(c, app))) return st;
  if (v == VF_COAL && c->tables[app].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[app].K, VF_MAX_RANGES);
  CUDA_TRY(c, app_ops(app)->verify((int)v, ptrs_dev, n, mism_dev, dev_table(c, app), S(stream)));
  return VF_OK;
}

vf_status vf_dispatch(vf_ctx* c, vf_variant v, uint32_t app, uint32_t method,
                      const uint64_t* objs_dev, uint64_t n, const void* args, size_t args_bytes,
                      void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  const AppOps* ops = app_ops(app);
  if ((unsigned)v > VF_CONCORD) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if (method >= ops->nmethods) return fail(c, VF_ERR_INVALID, "method %u of app %s", method, ops->name);
  if (args_bytes > VF_MAX_ARGS_BYTES || (args_bytes && !args))
    return fail(c, VF_ERR_INVALID, "args_bytes %zu", args_bytes);
  if (args_bytes < ops->method_args_bytes[method])
    return fail(c, VF_ERR_INVALID, "method %u needs %u argument bytes, got %zu", method,
                ops->method_args_bytes[method], args_bytes);
  if (n && !objs_dev) return fail(c, VF_ERR_INVALID, "null objs");
  if (v == VF_COAL && c->tables[app].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[app].K, VF_MAX_RANGES);
  ArgBlob blob;
  memset(&blob, 0, sizeof blob);
  if (args_bytes) memcpy(blob.b, args, args_bytes);
  const cudaError_t e = ops->dispatch((int)v, method, objs_dev, n, blob, dev_table(c, app), S(stream));
  if (e == cudaErrorNotSupported)
    return fail(c, VF_ERR_UNSUPPORTED, "app %s has no embedded type tag (Concord)", ops->name);
  CUDA_TRY(c, e);
  return VF_OK;
}

vf_status vf_dispatch_host(vf_ctx* c, vf_variant v, uint32_t app, uint32_t method, const uint64_t* objs_host,
                           uint64_t n, const void* args, size_t args_bytes, uint64_t* staging_dev, uint64_t chunk,
                           void* stream) {
  vf_status st = check_app(c, app);
  if (st) return st;
  if (!n) return VF_OK;
  if (!objs_host || !staging_dev) return fail(c, VF_ERR_INVALID, "null host array or staging buffer");
  if ((st = set_device(c))) return st;
  if (!chunk) chunk = 1ull << 22;
  const uint64_t nchunks = (n + chunk - 1) / chunk;
  if (!c->copy_stream) CUDA_TRY(c, cudaStreamCreateWithFlags(&c->copy_stream, cudaStreamNonBlocking));
  while (c->chunk_events.size() < nchunks + 1) {
    cudaEvent_t e;
    CUDA_TRY(c, cudaEventCreateWithFlags(&e, cudaEventDisableTiming));
    c->chunk_events.push_back(e);
  }
  cudaStream_t us = S(stream);
  // the staging buffer may still be read by earlier work on `stream`
  CUDA_TRY(c, cudaEventRecord(c->chunk_events[nchunks], us));
  CUDA_TRY(c, cudaStreamWaitEvent(c->copy_stream, c->chunk_events[nchunks], 0));
  for (uint64_t k = 0; k < nchunks; ++k) {
    const uint64_t off = k * chunk, m = n - off < chunk ? n - off : chunk;
    CUDA_TRY(c, cudaMemcpyAsync(staging_dev + off, objs_host + off, 8 * m, cudaMemcpyHostToDevice, c->copy_stream));
    CUDA_TRY(c, cudaEventRecord(c->chunk_events[k], c->copy_stream));
  }
  for (uint64_t k = 0; k < nchunks; ++k) {
    const uint64_t off = k * chunk, m = n - off < chunk ? n - off : chunk;
    CUDA_TRY(c, cudaStreamWaitEvent(us, c->chunk_events[k], 0));
    if ((st = vf_dispatch(c, v, app, method, staging_dev + off, m, args, args_bytes, stream))) return st;
  }
  return VF_OK;
}

vf_status vf_dispatch_concord(vf_ctx* c, uint32_t app, uint32_t m, const uint64_t* o, uint64_t n, const void* a,
                              size_t ab, void* s) {
  return vf_dispatch(c, VF_CONCORD, app, m, o, n, a, ab, s);
}

vf_status vf_ray_render(vf_ctx* c, vf_variant v, const uint64_t* shapes_dev, uint32_t S, uint32_t W,
                        uint32_t H, uint32_t row0, uint32_t nrows, const float* cam, const float* albedo,
                        float* rgb_dev, int32_t* hit_dev, void* stream) {
  vf_status st = check_app(c, VF_APP_RAY);
  if (st) return st;
  if ((unsigned)v > VF_TYPEPTR) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if (!cam || !albedo || !rgb_dev || !hit_dev || (S && !shapes_dev) || row0 + nrows > H)
    return fail(c, VF_ERR_INVALID, "ray_render arguments");
  if ((st = set_device(c)) || (st = ensure_vptrs(c, VF_APP_RAY))) return st;
  if (v == VF_COAL && c->tables[VF_APP_RAY].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[VF_APP_RAY].K, VF_MAX_RANGES);
  CUDA_TRY(c, ray_render((int)v, shapes_dev, S, W, H, row0, nrows, cam, albedo, rgb_dev, hit_dev,
                         dev_table(c, VF_APP_RAY), reinterpret_cast<cudaStream_t>(stream)));
  return VF_OK;
}

vf_status vf_gol_step(vf_ctx* c, vf_variant v, uint32_t W, uint32_t H, int torus, const uint8_t* prev_dev,
                      uint8_t* next_dev, uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* alive_dev,
                      const uint64_t* dead_dev, void* stream) {
  vf_status st = check_app(c, VF_APP_GOL);
  if (st) return st;
  if ((unsigned)v > VF_TYPEPTR) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if ((uint64_t)W * H > 0xFFFFFFFFull) return fail(c, VF_ERR_INVALID, "W*H > 2^32-1 cells");
  if ((uint64_t)W * H && (!prev_dev || !next_dev || !nbr_dev || !grid_dev || !alive_dev || !dead_dev))
    return fail(c, VF_ERR_INVALID, "gol_step arguments");
  if ((st = set_device(c)) || (st = ensure_vptrs(c, VF_APP_GOL))) return st;
  if (v == VF_COAL && c->tables[VF_APP_GOL].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[VF_APP_GOL].K, VF_MAX_RANGES);
  CUDA_TRY(c, gol_step((int)v, W, H, torus, prev_dev, next_dev, nbr_dev, grid_dev, alive_dev, dead_dev,
                       dev_table(c, VF_APP_GOL), reinterpret_cast<cudaStream_t>(stream)));
  return VF_OK;
}

vf_status vf_gol_run(vf_ctx* c, vf_variant v, uint32_t W, uint32_t H, int torus, uint8_t* state0_dev,
                     uint8_t* state1_dev, uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* alive_dev,
                     const uint64_t* dead_dev, uint32_t gens, uint32_t* barrier_dev, void* stream) {
  vf_status st = check_app(c, VF_APP_GOL);
  if (st) return st;
  if ((unsigned)v > VF_TYPEPTR) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if ((uint64_t)W * H > 0xFFFFFFFFull) return fail(c, VF_ERR_INVALID, "W*H > 2^32-1 cells");
  if ((uint64_t)W * H && gens &&
      (!state0_dev || !state1_dev || !nbr_dev || !grid_dev || !alive_dev || !dead_dev || !barrier_dev))
    return fail(c, VF_ERR_INVALID, "gol_run arguments");
  if ((st = set_device(c)) || (st = ensure_vptrs(c, VF_APP_GOL))) return st;
  if (v == VF_COAL && c->tables[VF_APP_GOL].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[VF_APP_GOL].K, VF_MAX_RANGES);
  CUDA_TRY(c, gol_run((int)v, W, H, torus, state0_dev, state1_dev, nbr_dev, grid_dev, alive_dev, dead_dev, gens,
                      barrier_dev, dev_table(c, VF_APP_GOL), reinterpret_cast<cudaStream_t>(stream)));
  return VF_OK;
}

vf_status vf_gen_step_rows(vf_ctx* c, vf_variant v, uint32_t W, uint32_t H, int torus, uint32_t row0,
                           uint32_t nrows, const uint8_t* prev_dev, uint8_t* next_dev, uint8_t* nbr_dev,
                           uint64_t* grid_dev, const uint64_t* dead_dev, const uint64_t* alive_dev,
                           const uint64_t* dying_dev, uint32_t born_mask, uint32_t survive_mask, uint32_t C,
                           void* stream) {
  vf_status st = check_app(c, VF_APP_GEN);
  if (st) return st;
  if ((unsigned)v > VF_TYPEPTR) return fail(c, VF_ERR_INVALID, "variant %d", (int)v);
  if ((uint64_t)W * H > 0xFFFFFFFFull) return fail(c, VF_ERR_INVALID, "W*H = %llu > 2^32-1 cells",
                                                  (unsigned long long)W * H);
  if ((uint64_t)row0 + nrows > H) return fail(c, VF_ERR_INVALID, "rows [%u, %u) outside H = %u", row0, row0 + nrows, H);
  if ((uint64_t)W * nrows && (!prev_dev || !next_dev || !nbr_dev || !grid_dev || !dead_dev || !alive_dev || !dying_dev))
    return fail(c, VF_ERR_INVALID, "gen_step arguments");
  if (C < 2 || C > 255) return fail(c, VF_ERR_INVALID, "C = %u", C);
  if ((st = set_device(c)) || (st = ensure_vptrs(c, VF_APP_GEN))) return st;
  if (v == VF_COAL && c->tables[VF_APP_GEN].K > VF_MAX_RANGES)
    return fail(c, VF_ERR_TABLE_FULL, "K = %u > %u", c->tables[VF_APP_GEN].K, VF_MAX_RANGES);
  CUDA_TRY(c, gen_step((int)v, W, H, torus, row0, nrows, prev_dev, next_dev, nbr_dev, grid_dev, dead_dev, alive_dev,
                       dying_dev, born_mask, survive_mask, C, dev_table(c, VF_APP_GEN),
                       reinterpret_cast<cudaStream_t>(stream)));
  return VF_OK;
}

vf_status vf_gen_step(vf_ctx* c, vf_variant v, uint32_t W, uint32_t H, int torus, const uint8_t* prev_dev,
                      uint8_t* next_dev, uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* dead_dev,
                      const uint64_t* alive_dev, const uint64_t* dying_dev, uint32_t born_mask,
                      uint32_t survive_mask, uint32_t C, void* stream) {
  return vf_gen_step_rows(c, v, W, H, torus, 0, H, prev_dev, next_dev, nbr_dev, grid_dev, dead_dev, alive_dev,
                          dying_dev, born_mask, survive_mask, C, stream);
}

vf_status vf_dispatch_cuda(vf_ctx* c, uint32_t app, uint32_t m, const uint64_t* o, uint64_t n,
                           const void* a, size_t ab, void* s) {
  return vf_dispatch(c, VF_CUDA, app, m, o, n, a, ab, s);
}
vf_status vf_dispatch_sharedoa(vf_ctx* c, uint32_t app, uint32_t m, const uint64_t* o, uint64_t n,
                               const void* a, size_t ab, void* s) {
  return vf_dispatch(c, VF_SHAREDOA, app, m, o, n, a, ab, s);
}
vf_status vf_dispatch_coal(vf_ctx* c, uint32_t app, uint32_t m, const uint64_t* o, uint64_t n,
                           const void* a, size_t ab, void* s) {
  return vf_dispatch(c, VF_COAL, app, m, o, n, a, ab, s);
}
vf_status vf_dispatch_typeptr(vf_ctx* c, uint32_t app, uint32_t m, const uint64_t* o, uint64_t n,
                              const void* a, size_t ab, void* s) {
  return vf_dispatch(c, VF_TYPEPTR, app, m, o, n, a, ab, s);
}

}  // extern "C"
