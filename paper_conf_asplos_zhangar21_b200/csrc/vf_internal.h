// vf_internal.h — internal interface between the host core (core.cu) and the
// per-app device modules (app_*.cu). Not part of the public ABI (include/vf.h).
//
// GPUs cannot load code dynamically: every virtual function a kernel may call
// must be compiled into that kernel's module, and a vTable* is only
// meaningful inside the module whose kernel constructed the object. So each app
// is ONE translation unit holding its class hierarchy, its construction kernels
// and its dispatch kernels, and exports an AppOps table to the core.
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include "../../include/vf.h"

namespace vf {

// Method argument blob, copied by value into kernel parameters.
struct __align__(16) ArgBlob {
  unsigned char b[VF_MAX_ARGS_BYTES];
};

// Device view of one app's virtual range table (sorted, merged) and vTables.
// Tables of <= kTableInline rows also travel inline in the kernel parameters
// (constant bank), so a COAL CTA stages them into shared memory without a
// dependent global load at its start (the paper keeps the table in
// constant / shared memory).
constexpr uint32_t kTableInline = 8;
struct DevTable {
  const uint64_t* start;  // K entries, sorted
  const uint64_t* end;    // K entries
  const uint32_t* type;   // K entries
  uint32_t K;
  uint32_t P;             // K rounded up to a power of two (>= 1); smem table size
  const uint64_t* vptr;   // ntypes entries: device vTable* per concrete type
  uint32_t ntypes;
  uint32_t active_types;  // concrete types with live objects (launch heuristics)
  uint32_t inl;           // 1: COAL tests the inline rows below (K <= min(kTableInline, tuning coal_inline))
  uint64_t in_start[kTableInline];  // rows 0..K-1 when K <= kTableInline
  uint64_t in_len[kTableInline];    // end - start (0 for padding rows)
  uint32_t in_type[kTableInline];
};

struct AppOps {
  const char* name;
  uint32_t ntypes;
  const uint32_t* obj_bytes;  // per type, sizeof(class)
  uint32_t nmethods;
  const uint32_t* method_args_bytes;  // per method: sizeof(args struct)
  // vTable* of each type -> out_dev[ntypes] (placement-new into scratch).
  cudaError_t (*probe_vptrs)(uint64_t* out_dev, cudaStream_t s);
  // placement-new object i of class types[i] at strip(ptrs[i]).
  cudaError_t (*construct)(const uint32_t* types_dev, const uint64_t* ptrs_dev,
                           const void* ctor_args_dev, uint32_t ctor_arg_bytes, uint64_t n,
                           cudaStream_t s);
  // device-heap new (CUDA baseline); out_ptrs[i] = new T(types[i]) or 0.
  cudaError_t (*new_cuda)(const uint32_t* types_dev, const void* ctor_args_dev,
                          uint32_t ctor_arg_bytes, uint64_t n, uint64_t* out_ptrs_dev,
                          cudaStream_t s);
  // delete of device-heap objects (untagged pointers).
  cudaError_t (*delete_cuda)(const uint64_t* ptrs_dev, uint64_t n, cudaStream_t s);
  cudaError_t (*dispatch)(int variant, uint32_t method, const uint64_t* objs_dev, uint64_t n,
                          const ArgBlob& args, const DevTable& tbl, cudaStream_t s);
  cudaError_t (*resolve)(int variant, const uint64_t* ptrs_dev, uint64_t n, uint32_t* out_dev,
                         const DevTable& tbl, cudaStream_t s);
  cudaError_t (*verify)(int variant, const uint64_t* ptrs_dev, uint64_t n,
                        unsigned long long* mism_dev, const DevTable& tbl, cudaStream_t s);
};

const AppOps* app_micro();
const AppOps* app_gol();
const AppOps* app_gen();
const AppOps* app_graph();
const AppOps* app_ray();
const AppOps* app_traf();
const AppOps* app_nbody();
const AppOps* app_stut();
const AppOps* app_collide();
const AppOps* app_graph_en();
const AppOps* app_edge();

// config 3 renderer (app_ray.cu): rows [row0, row0+nrows) of a W x H image
cudaError_t ray_render(int variant, const uint64_t* objs, uint32_t S, uint32_t W, uint32_t H, uint32_t row0,
                       uint32_t nrows, const float* cam5, const float* albedo12, float* rgb, int32_t* hid,
                       const DevTable& tbl, cudaStream_t s);

// fused cellular-automaton generations (app_gol.cu / app_gen.cu)
cudaError_t gol_step(int variant, uint32_t W, uint32_t H, int torus, const uint8_t* prev, uint8_t* next, uint8_t* nbr,
                     uint64_t* grid, const uint64_t* alive, const uint64_t* dead, const DevTable& tbl,
                     cudaStream_t s);
cudaError_t gol_run(int variant, uint32_t W, uint32_t H, int torus, uint8_t* buf0, uint8_t* buf1, uint8_t* nbr,
                    uint64_t* grid, const uint64_t* alive, const uint64_t* dead, uint32_t gens, unsigned* bar,
                    const DevTable& tbl, cudaStream_t s);
cudaError_t gen_step(int variant, uint32_t W, uint32_t H, int torus, uint32_t row0, uint32_t nrows,
                     const uint8_t* prev, uint8_t* next, uint8_t* nbr, uint64_t* grid, const uint64_t* dead,
                     const uint64_t* alive, const uint64_t* dying, uint32_t born, uint32_t survive, uint32_t C,
                     const DevTable& tbl, cudaStream_t s);

// Batched typed allocation on the device (alloc.cu). A type's free slots, in
// allocation order, are a list of segments: ranks [rank0, next segment's
// rank0) live at addr + (rank - rank0) * obj_bytes.
struct PlaceSeg {
  uint64_t rank0;
  uint64_t addr;
  uint64_t obj_bytes;
};
uint64_t rank_chunks(uint64_t n);  // hist rows (32 u32 each) needed for n objects
// per-chunk type histogram -> in-place exclusive scan per type; totals[t] =
// objects of type t; *bad != 0 if a type id >= ntypes (ntypes <= 32)
cudaError_t rank_hist(const uint32_t* types, uint64_t n, uint32_t ntypes, uint32_t* hist, uint32_t* bad,
                      unsigned long long* totals, cudaStream_t s);
// out[i] = slot of object i (its rank among same-type objects of lower index), tagged if tag
cudaError_t rank_place(const uint32_t* types, uint64_t n, const uint32_t* hist, const PlaceSeg* segs,
                       const uint32_t* seg_first, int tag, uint64_t* out, cudaStream_t s);
cudaError_t place_packed(uint64_t base, uint64_t stride, uint64_t n, uint64_t* out, cudaStream_t s);
cudaError_t fill_u32(uint32_t* x, uint64_t n, uint32_t v, cudaStream_t s);

// Benchmark / ablation knobs set through vf_set_tuning (-1 = app default).
struct Tuning {
  int unroll = -1;    // objects per thread in the grouped kernels (1, 2, 4)
  int prefetch = -1;  // 0 none, 1 prefetch.global.L1, 2 L1-allocating warm load
  int pipeline = 0;   // 1: TMA-pipelined pointer stream (k_dispatch_pipe), 0: plain loads
  int regroup = 1;    // 1: CTA-level counting sort of each tile by type (k_dispatch_sorted)
  int call = 0;       // COAL / TypePointer: 0 grouped direct call, 1 indirect CALL via vFunc* table
  int persistent = -1; // grouped kernels: 1 persistent grid, 0 one tile per CTA, -1 app default (kHeavyMask)
  int cluster = 0;     // vf_gol_run: 1 one thread-block cluster (state in DSMEM) when the grid fits
  int ray_rays = 4;       // ray kernels: pixels (rays) per thread, 2 or 4
  int ray_parts = -1;     // ray COAL / TypePointer: shape parts per pixel block (1..16; -1: balance the last wave)
  int coal_inline = 8;    // COAL: largest table (rows) tested from the kernel parameters (0: always shared memory)
  int gsort = -1;         // COAL / TypePointer heavy methods: 1 = sort the whole dispatch list by type
                          // first, 0 = per CTA tile only, -1 = app default (App::kGridSort)
};
Tuning& tuning();

// launch accounting (bench: gpu_launches)
void note_launch(uint64_t k = 1);

}  // namespace vf
