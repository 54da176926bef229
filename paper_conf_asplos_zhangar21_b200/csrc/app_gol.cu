// app_gol.cu — config 1: Game of Life over polymorphic cells (Table 2,
// P:1518-1522). Readings: G12 dead border (torus optional), G13
// abstract Cell + concrete Alive / Dead, G14 p = 0.5 soup. Every cell owns one
// object in each type's arena (slot = cell id), so a type change is a pointer
// swap and the type-contiguous arenas stay valid for COAL / TypePointer.
//
// Object layout (16 B): { vTable* (8 B), u32 cell, u16 counter, u16 pad }.
// counter = age (Alive) / dead_for (Dead): incremented by next(), reset to 0
// when the cell switches to this object.
#include <cooperative_groups.h>
#include <cstring>

#include "dispatch.cuh"

namespace vf {
namespace gol {

struct Cell {
  __device__ explicit Cell(const void* arg) : cell(arg ? *static_cast<const uint32_t*>(arg) : 0) {}
  __device__ virtual ~Cell() {}
  __device__ virtual void next(vf_gol_next_args a) = 0;
  __device__ virtual void get(vf_gol_get_args a) = 0;
  uint32_t cell;
  uint16_t counter = 0;
  uint16_t pad = 0;
};

struct Alive final : Cell {
  __device__ explicit Alive(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gol_next_args a) override {
    const uint8_t n = a.nbr_dev[cell];
    ++counter;
    a.state_out_dev[cell] = (n == 2 || n == 3) ? 1 : 0;
  }
  __device__ void get(vf_gol_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 1;
  }
};

struct Dead final : Cell {
  __device__ explicit Dead(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gol_next_args a) override {
    const uint8_t n = a.nbr_dev[cell];
    ++counter;
    a.state_out_dev[cell] = n == 3 ? 1 : 0;
  }
  __device__ void get(vf_gol_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 0;
  }
};

template <int K>
struct TypeOf;
template <>
struct TypeOf<0> { using T = Dead; };
template <>
struct TypeOf<1> { using T = Alive; };

struct App {
  static constexpr int kTypes = 2;  // 0 = Dead, 1 = Alive
  static constexpr int kMethods = 2;
  static constexpr int kUnroll = 1;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 0;
  static constexpr bool kLean = true;  // default launch configuration only (knob sweeps: micro)
  using Base = Cell;
  template <int K>
  using Type = typename TypeOf<K>::T;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_GOL_NEXT) o->next(blob_as<vf_gol_next_args>(b));
    else o->get(blob_as<vf_gol_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_GOL_NEXT) o->Type<K>::next(blob_as<vf_gol_next_args>(b));
    else o->Type<K>::get(blob_as<vf_gol_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(Alive) == 16 && sizeof(Dead) == 16, "cell layout");

__global__ void k_neighbors(uint32_t W, uint32_t H, int torus, const uint8_t* __restrict__ st,
                            uint8_t* __restrict__ nb) {
  const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= (uint64_t)W * H) return;
  nb[c] = count_live(W, H, torus, st, c);
}

__global__ void k_swap(uint64_t n, const uint8_t* __restrict__ prev, const uint8_t* __restrict__ next,
                       uint64_t* __restrict__ grid, const uint64_t* __restrict__ alive,
                       const uint64_t* __restrict__ dead) {
  const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  const uint8_t s = next[c];
  if (s != prev[c]) {
    const uint64_t p = s ? alive[c] : dead[c];
    grid[c] = p;
    reinterpret_cast<Cell*>(strip(p))->counter = 0;
  }
}

// Fused generation (vf_gol_step): neighbours -> virtual next() -> swap per cell.
struct Step {
  uint32_t W, H;
  int torus;
  const uint8_t* prev;
  const uint8_t* next;
  uint8_t* nbr;
  uint64_t* grid;
  const uint64_t* alive;
  const uint64_t* dead;
  __device__ __forceinline__ void pre(uint64_t c) const { nbr[c] = count_live(W, H, torus, prev, c); }
  __device__ __forceinline__ uint64_t ptr(uint64_t c) const { return grid[c]; }
  // the body reads nbr[cell] (just written by pre) and the object's counter
  __device__ __forceinline__ uint32_t warm(uint64_t c, uint64_t a) const {
    uint32_t v, w;
    asm volatile("ld.global.ca.u8 %0, [%1];" : "=r"(v) : "l"(nbr + c));
    asm volatile("ld.global.ca.u32 %0, [%1];" : "=r"(w) : "l"(a + 8));
    return v ^ w;
  }
  __device__ __forceinline__ uint64_t* ptr_base() const { return grid; }
  __device__ __forceinline__ void post(uint64_t c) const {
    const uint8_t s = next[c];
    if (s != prev[c]) {
      const uint64_t p = s ? alive[c] : dead[c];
      grid[c] = p;
      reinterpret_cast<Cell*>(strip(p))->counter = 0;
    }
  }
};


// ---------------------------------------------------------------------------
// Persistent multi-generation run (vf_gol_run). At 256 x 256 one generation is
// a few microseconds of work, so a launch per generation is launch-latency
// bound. Here ONE cooperative launch runs all generations: every cell is
// owned by a fixed thread (grid-stride mapping with a fixed grid), generations
// are separated by a grid barrier, and COAL's range table is staged into
// shared memory once for all of them. State arrays written by other CTAs are
// read with ld.global.cg (L2; L1 is not coherent across SMs); everything else
// a thread touches (its cells' nbr, grid entries and objects) is its own.
// Same variants, same bodies, same results as vf_gol_step per generation.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint8_t ldcg_u8(const uint8_t* p) { return __ldcg(p); }

__device__ __forceinline__ uint8_t count_live_cg(uint32_t W, uint32_t H, int torus, const uint8_t* st, uint32_t c) {
  const uint32_t yq = c / W;  // 32-bit (W*H < 2^32): no u64 division subroutine
  const int y = (int)yq, x = (int)(c - yq * W);
  int n = 0;
#pragma unroll
  for (int dy = -1; dy <= 1; ++dy)
#pragma unroll
    for (int dx = -1; dx <= 1; ++dx) {
      if (dx == 0 && dy == 0) continue;
      int yy = y + dy, xx = x + dx;
      if (torus) {
        yy = (yy + (int)H) % (int)H;
        xx = (xx + (int)W) % (int)W;
      } else if (yy < 0 || yy >= (int)H || xx < 0 || xx >= (int)W) {
        continue;
      }
      n += ldcg_u8(st + (uint64_t)yy * W + xx) == 1;
    }
  return (uint8_t)n;
}

__device__ __forceinline__ uint32_t ld_acquire_u32(const unsigned* p) {
  uint32_t v;
  asm volatile("ld.acquire.gpu.global.u32 %0, [%1];" : "=r"(v) : "l"(p) : "memory");
  return v;
}

// Monotonic grid barrier: after the g-th barrier *ctr == g * gridDim.x
// (zeroed before the launch; all CTAs are co-resident: cooperative launch).
__device__ __forceinline__ void grid_barrier(unsigned* ctr, uint32_t& target) {
  __syncthreads();
  target += gridDim.x;
  if (threadIdx.x == 0) {
    __threadfence();
    atomicAdd(ctr, 1u);
    while (ld_acquire_u32(ctr) < target) {
    }
  }
  __syncthreads();
}

struct RunArgs {
  uint32_t W, H;
  int torus;
  uint32_t gens;
  uint8_t* buf[2];  // state buffers: generation g reads buf[g & 1], writes buf[(g + 1) & 1]
  uint8_t* nbr;
  uint64_t* grid;
  const uint64_t* alive;
  const uint64_t* dead;
  unsigned* bar;
};

__device__ __forceinline__ void post_cg(const RunArgs& r, const uint8_t* prev, const uint8_t* next, uint64_t c) {
  const uint8_t s = __ldcg(next + c);
  if (s != __ldcg(prev + c)) {
    const uint64_t p = s ? r.alive[c] : r.dead[c];
    r.grid[c] = p;
    reinterpret_cast<Cell*>(strip(p))->counter = 0;
  }
}

template <class R>
__global__ void __launch_bounds__(kBlock) k_run_grouped(RunArgs r, DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  const uint64_t n = (uint64_t)r.W * r.H;
  uint32_t hint = 0, target = 0;
  for (uint32_t g = 0; g < r.gens; ++g) {
    const uint8_t* prev = r.buf[g & 1];
    uint8_t* next = r.buf[(g + 1) & 1];
    ArgBlob args{};
    const vf_gol_next_args a{r.nbr, next};
    *reinterpret_cast<vf_gol_next_args*>(args.b) = a;
    for (uint64_t base = (uint64_t)blockIdx.x * kBlock; base < n; base += (uint64_t)gridDim.x * kBlock) {
      const uint64_t c = base + threadIdx.x;
      const bool valid = c < n;
      uint64_t p = 0, ad = 0;
      uint32_t t = kNF;
      if (valid) {
        r.nbr[c] = count_live_cg(r.W, r.H, r.torus, prev, c);
        p = r.grid[c];
      }
      if (p) t = R::resolve(smem, tbl, p, ad, hint);
      group_call<App, VF_GOL_NEXT>(t, ad, p, c, args, tbl);
      if (valid) post_cg(r, prev, next, c);
    }
    grid_barrier(r.bar, target);
  }
}

__global__ void __launch_bounds__(kBlock) k_run_virtual(RunArgs r) {
  const uint64_t n = (uint64_t)r.W * r.H;
  uint32_t target = 0;
  for (uint32_t g = 0; g < r.gens; ++g) {
    const uint8_t* prev = r.buf[g & 1];
    uint8_t* next = r.buf[(g + 1) & 1];
    const vf_gol_next_args a{r.nbr, next};
    for (uint64_t c = (uint64_t)blockIdx.x * kBlock + threadIdx.x; c < n; c += (uint64_t)gridDim.x * kBlock) {
      r.nbr[c] = count_live_cg(r.W, r.H, r.torus, prev, c);
      const uint64_t p = r.grid[c];
      if (p) reinterpret_cast<Cell*>(p)->next(a);  // the compiler's virtual call
      post_cg(r, prev, next, c);
    }
    grid_barrier(r.bar, target);
  }
}

// Cluster variant (small grids, e.g. config 1's 256 x 256): ONE thread-block
// cluster of C CTAs (up to 16, non-portable size) runs every generation. CTA r
// keeps its block of rows of the state in shared memory (double-buffered);
// neighbour rows owned by other CTAs are read through distributed shared
// memory, and generations are separated by the hardware cluster barrier
// (barrier.cluster, ~0.2 us, which also orders the DSMEM writes). The method
// still writes its next state to global memory (its contract); the owning
// thread reads its own write back into shared memory for the neighbours.
constexpr int kClusterBlock = 1024;

template <class R>
__global__ void __launch_bounds__(kClusterBlock, 1) k_run_cluster(RunArgs r, DevTable tbl, uint32_t rows_per) {
  extern __shared__ __align__(16) unsigned char smem[];
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  const uint32_t rank = cluster.block_rank();
  const size_t tbytes = R::kNeedsTable ? (table_smem_dev(tbl.P) + 15) / 16 * 16 : 0;
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  uint8_t* const sb0 = smem + tbytes;
  uint8_t* const sb1 = smem + tbytes + (size_t)rows_per * r.W;
  const uint32_t W = r.W, H = r.H;
  const uint32_t y0 = rank * rows_per;
  const uint32_t y1 = min(H, y0 + rows_per);
  const uint32_t own = y1 > y0 ? (y1 - y0) * W : 0u;
  // initial state of the owned rows
  for (uint32_t k = threadIdx.x; k < own; k += kClusterBlock) sb0[k] = r.buf[0][(uint64_t)y0 * W + k];
  cluster.sync();
  uint32_t hint = 0;
  for (uint32_t g = 0; g < r.gens; ++g) {
    const uint8_t* cur = (g & 1) ? sb1 : sb0;
    uint8_t* nxt_s = (g & 1) ? sb0 : sb1;
    uint8_t* next = (g & 1) ? r.buf[0] : r.buf[1];
    ArgBlob args{};
    const vf_gol_next_args a{r.nbr, next};
    *reinterpret_cast<vf_gol_next_args*>(args.b) = a;
    const uint32_t iters = (own + kClusterBlock - 1) / kClusterBlock;  // CTA-uniform
    for (uint32_t it = 0; it < iters; ++it) {
      const uint32_t k = it * kClusterBlock + threadIdx.x;
      const bool valid = k < own;
      uint64_t c = 0, p = 0, ad = 0;
      uint32_t t = kNF;
      uint8_t prev_s = 0;
      if (valid) {
        const uint32_t y = y0 + k / W, x = k % W;
        c = (uint64_t)y * W + x;
        int n = 0;
#pragma unroll
        for (int dy = -1; dy <= 1; ++dy) {
          int yy = (int)y + dy;
          if (r.torus) yy = (yy + (int)H) % (int)H;
          else if (yy < 0 || yy >= (int)H) continue;
          const uint32_t owner = (uint32_t)yy / rows_per;
          const uint8_t* row = (owner == rank ? const_cast<uint8_t*>(cur)
                                              : cluster.map_shared_rank(const_cast<uint8_t*>(cur), owner)) +
                               (size_t)((uint32_t)yy - owner * rows_per) * W;
#pragma unroll
          for (int dx = -1; dx <= 1; ++dx) {
            if (dx == 0 && dy == 0) continue;
            int xx = (int)x + dx;
            if (r.torus) xx = (xx + (int)W) % (int)W;
            else if (xx < 0 || xx >= (int)W) continue;
            n += row[xx] == 1;
          }
        }
        r.nbr[c] = (uint8_t)n;
        prev_s = cur[k];
        p = r.grid[c];
      }
      if (p) t = R::resolve(smem, tbl, p, ad, hint);
      group_call<App, VF_GOL_NEXT>(t, ad, p, c, args, tbl);
      if (valid) {
        const uint8_t s = *(volatile const uint8_t*)(next + c);  // this thread's own write
        if (s != prev_s) {
          const uint64_t q = s ? r.alive[c] : r.dead[c];
          r.grid[c] = q;
          reinterpret_cast<Cell*>(strip(q))->counter = 0;
        }
        nxt_s[k] = s;
      }
    }
    cluster.sync();
  }
}

template <class R>
__global__ void __launch_bounds__(kClusterBlock, 1) k_run_cluster_virtual(RunArgs r, DevTable tbl,
                                                                        uint32_t rows_per) {
  (void)tbl;
  extern __shared__ __align__(16) unsigned char smem[];
  namespace cg = cooperative_groups;
  cg::cluster_group cluster = cg::this_cluster();
  const uint32_t rank = cluster.block_rank();
  uint8_t* const sb0 = smem;
  uint8_t* const sb1 = smem + (size_t)rows_per * r.W;
  const uint32_t W = r.W, H = r.H;
  const uint32_t y0 = rank * rows_per;
  const uint32_t y1 = min(H, y0 + rows_per);
  const uint32_t own = y1 > y0 ? (y1 - y0) * W : 0u;
  for (uint32_t k = threadIdx.x; k < own; k += kClusterBlock) sb0[k] = r.buf[0][(uint64_t)y0 * W + k];
  cluster.sync();
  for (uint32_t g = 0; g < r.gens; ++g) {
    const uint8_t* cur = (g & 1) ? sb1 : sb0;
    uint8_t* nxt_s = (g & 1) ? sb0 : sb1;
    uint8_t* next = (g & 1) ? r.buf[0] : r.buf[1];
    const vf_gol_next_args a{r.nbr, next};
    for (uint32_t k = threadIdx.x; k < own; k += kClusterBlock) {
      const uint32_t y = y0 + k / W, x = k % W;
      const uint64_t c = (uint64_t)y * W + x;
      int n = 0;
#pragma unroll
      for (int dy = -1; dy <= 1; ++dy) {
        int yy = (int)y + dy;
        if (r.torus) yy = (yy + (int)H) % (int)H;
        else if (yy < 0 || yy >= (int)H) continue;
        const uint32_t owner = (uint32_t)yy / rows_per;
        const uint8_t* row = (owner == rank ? const_cast<uint8_t*>(cur)
                                            : cluster.map_shared_rank(const_cast<uint8_t*>(cur), owner)) +
                             (size_t)((uint32_t)yy - owner * rows_per) * W;
#pragma unroll
        for (int dx = -1; dx <= 1; ++dx) {
          if (dx == 0 && dy == 0) continue;
          int xx = (int)x + dx;
          if (r.torus) xx = (xx + (int)W) % (int)W;
          else if (xx < 0 || xx >= (int)W) continue;
          n += row[xx] == 1;
        }
      }
      r.nbr[c] = (uint8_t)n;
      const uint8_t prev_s = cur[k];
      const uint64_t p = r.grid[c];
      if (p) reinterpret_cast<Cell*>(p)->next(a);  // the compiler's virtual call
      const uint8_t s = *(volatile const uint8_t*)(next + c);
      if (s != prev_s) {
        const uint64_t q = s ? r.alive[c] : r.dead[c];
        r.grid[c] = q;
        reinterpret_cast<Cell*>(strip(q))->counter = 0;
      }
      nxt_s[k] = s;
    }
    cluster.sync();
  }
}

// Launch one cluster of C CTAs if the grid's rows fit; returns
// cudaErrorNotSupported (caller falls back to the grid-barrier kernels) if not.
template <class K>
static cudaError_t cluster_launch(K kern, const RunArgs& r, const DevTable& tbl, size_t table_bytes, cudaStream_t s) {
  const uint64_t n = (uint64_t)r.W * r.H;
  if (n > (1u << 17)) return cudaErrorNotSupported;  // bigger grids: the whole GPU, not one cluster
  for (int C : {16, 8}) {
    const uint32_t rows_per = (r.H + C - 1) / C;
    const size_t sm = (table_bytes + 15) / 16 * 16 + 2 * (size_t)rows_per * r.W;
    if (sm > 200 * 1024) continue;
    cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    if (C > 8) cudaFuncSetAttribute(kern, cudaFuncAttributeNonPortableClusterSizeAllowed, 1);
    cudaLaunchConfig_t cfg{};
    cfg.gridDim = dim3(C);
    cfg.blockDim = dim3(kClusterBlock);
    cfg.dynamicSmemBytes = sm;
    cfg.stream = s;
    cudaLaunchAttribute attr[1];
    attr[0].id = cudaLaunchAttributeClusterDimension;
    attr[0].val.clusterDim.x = C;
    attr[0].val.clusterDim.y = 1;
    attr[0].val.clusterDim.z = 1;
    cfg.attrs = attr;
    cfg.numAttrs = 1;
    int nclusters = 0;
    if (cudaOccupancyMaxActiveClusters(&nclusters, (const void*)kern, &cfg) != cudaSuccess || nclusters < 1) {
      cudaGetLastError();
      continue;
    }
    const cudaError_t e = cudaLaunchKernelEx(&cfg, kern, r, tbl, rows_per);
    note_launch();
    return e;
  }
  return cudaErrorNotSupported;
}

template <class K>
static cudaError_t coop_launch(K kern, uint64_t n, size_t sm, void** params, cudaStream_t s) {
  int occ = 0;
  if (sm > 48 * 1024) cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  cudaError_t e = cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, sm);
  if (e != cudaSuccess) return e;
  if (occ < 1) return cudaErrorCooperativeLaunchTooLarge;
  const uint64_t tiles = (n + kBlock - 1) / kBlock;
  const uint64_t cap = (uint64_t)num_sms() * occ;
  const unsigned grid = (unsigned)(tiles < cap ? (tiles ? tiles : 1) : cap);
  e = cudaLaunchCooperativeKernel((const void*)kern, dim3(grid), dim3(kBlock), params, sm, s);
  note_launch();
  return e;
}
}  // namespace gol

cudaError_t gol_step(int variant, uint32_t W, uint32_t H, int torus, const uint8_t* prev, uint8_t* next, uint8_t* nbr,
                     uint64_t* grid, const uint64_t* alive, const uint64_t* dead, const DevTable& tbl,
                     cudaStream_t s) {
  vf_gol_next_args a{nbr, next};
  ArgBlob blob{};
  memcpy(blob.b, &a, sizeof a);
  const gol::Step st{W, H, torus, prev, next, nbr, grid, alive, dead};
  return launch_step<gol::App, VF_GOL_NEXT>(variant, (uint64_t)W * H, blob, tbl, st, s);
}

cudaError_t gol_run(int variant, uint32_t W, uint32_t H, int torus, uint8_t* buf0, uint8_t* buf1, uint8_t* nbr,
                    uint64_t* grid, const uint64_t* alive, const uint64_t* dead, uint32_t gens, unsigned* bar,
                    const DevTable& tbl, cudaStream_t s) {
  const uint64_t n = (uint64_t)W * H;
  if (!gens || !n) return cudaSuccess;
  cudaError_t e = cudaMemsetAsync(bar, 0, sizeof(unsigned), s);
  if (e != cudaSuccess) return e;
  gol::RunArgs r{W, H, torus, gens, {buf0, buf1}, nbr, grid, alive, dead, bar};
  DevTable t = tbl;
  void* params[2] = {&r, &t};
  // small grids: one thread-block cluster, state in distributed shared memory
  if (tuning().cluster != 0) {
    cudaError_t ce = cudaErrorNotSupported;
    switch (variant) {
      case VF_CUDA:
      case VF_SHAREDOA:
        ce = gol::cluster_launch(gol::k_run_cluster_virtual<ResolveTP>, r, t, 0, s);
        break;
      case VF_COAL:
        ce = gol::cluster_launch(gol::k_run_cluster<ResolveCOAL>, r, t, table_smem(tbl), s);
        break;
      case VF_TYPEPTR:
        ce = gol::cluster_launch(gol::k_run_cluster<ResolveTP>, r, t, 0, s);
        break;
    }
    if (ce != cudaErrorNotSupported) return ce;
  }
  switch (variant) {
    case VF_CUDA:
    case VF_SHAREDOA:
      return gol::coop_launch(gol::k_run_virtual, n, 0, params, s);
    case VF_COAL:
      return gol::coop_launch(gol::k_run_grouped<ResolveCOAL>, n, table_smem(tbl), params, s);
    case VF_TYPEPTR:
      return gol::coop_launch(gol::k_run_grouped<ResolveTP>, n, 0, params, s);
  }
  return cudaErrorInvalidValue;
}

static const uint32_t kGolBytes[2] = {16, 16};
static const uint32_t kGolArgs[2] = {sizeof(vf_gol_next_args), sizeof(vf_gol_get_args)};

const AppOps* app_gol() {
  static const AppOps ops = make_ops<gol::App>("gol", kGolBytes, kGolArgs);
  return &ops;
}

}  // namespace vf

extern "C" vf_status vf_gol_neighbors(uint32_t W, uint32_t H, int torus, const uint8_t* state_dev,
                                      uint8_t* nbr_dev, void* stream) {
  const uint64_t n = (uint64_t)W * H;
  if (!n) return VF_OK;
  if (!state_dev || !nbr_dev) return VF_ERR_INVALID;
  vf::gol::k_neighbors<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      W, H, torus, state_dev, nbr_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}

extern "C" vf_status vf_gol_swap(vf_ctx*, uint64_t ncells, const uint8_t* prev, const uint8_t* next,
                                 uint64_t* grid, const uint64_t* alive, const uint64_t* dead,
                                 void* stream) {
  if (!ncells) return VF_OK;
  if (!prev || !next || !grid || !alive || !dead) return VF_ERR_INVALID;
  vf::gol::k_swap<<<(unsigned)((ncells + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      ncells, prev, next, grid, alive, dead);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
