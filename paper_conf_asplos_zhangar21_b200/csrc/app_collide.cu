// app_collide.cu — config 5 "collision" at 16M bodies over polymorphic bodies
// (BASELINE north_star "collision/N-body"; DynaSOAr's collision app [46], not
// in this paper: readings G18 / G19 in DESIGN.md). Classes: abstract Body,
// concrete Star / Planet / Dust. One step, from the state P at its start:
//   (0) vf_collide_grid (non-virtual): a uniform grid of cells of side rc over
//       the active bodies, ids ascending per cell, a cell-sorted copy Ps of
//       the positions, and the dispatch order (owned objects in cell order);
//   (1) virtual update(): softened gravity over the bodies within rc found in
//       the 27 neighbour cells, nearest body within rm, integrate;
//   (2) virtual merge(): mutual-nearest pairs merge into the smaller id.
// Double-buffered (reading G8): update reads P and writes Pm / Vm / near;
// merge reads those and writes P, so no call reads what another call of the
// same launch writes.
//
// Built with -fmad=false -prec-div=true -prec-sqrt=true -ftz=false: every FMA
// is the explicit fmaf of the formula (vf.h), bit-identical to the oracle.
//
// Layout: {vptr, u32 idx, f32 vx, vy, vz} = 24 B; positions + masses are the
// caller's float4 arrays indexed by idx (the state a multi-GPU run exchanges).
#include "dispatch.cuh"
#include "ieee_fast.cuh"

namespace vf {
namespace collide {

// Cell coordinate of one axis: floor(x / rc) clamped to [0, G) (NaN -> 0),
// the oracle's cell_coord. IEEE division (-prec-div=true, and __fdiv_rn).
__device__ __forceinline__ int cell_coord(float x, float rc, int G) {
  const float f = floorf(__fdiv_rn(x, rc));
  if (!(f >= 0.0f)) return 0;
  if (f >= (float)G) return G - 1;
  return (int)f;
}

struct Body {
  uint32_t idx;
  float vx, vy, vz;
  __device__ explicit Body(const void* arg) {
    const uint32_t* q = static_cast<const uint32_t*>(arg);
    idx = q ? q[0] : 0;
    vx = q ? __uint_as_float(q[1]) : 0.f;
    vy = q ? __uint_as_float(q[2]) : 0.f;
    vz = q ? __uint_as_float(q[3]) : 0.f;
  }
  __device__ virtual ~Body() {}
  __device__ virtual void update(const vf_collide_update_args& a) = 0;
  __device__ virtual void merge(const vf_collide_merge_args& a) = 0;
  __device__ virtual void get(const vf_collide_get_args& a) = 0;

 protected:
  // Forces from the bodies within rc and the nearest body within rm. The
  // three cells x-1, x, x+1 of one (z, y) row are consecutive in the cell
  // index, so their bodies are ONE contiguous run of list / Ps in exactly the
  // oracle's order (x ascending, ids ascending within a cell): 9 runs per body.
  // "j != me" compares slots (slot[me]), so the id array is read only for
  // candidates within rm. (Measured on B200: batching 4 candidates for ILP,
  // with or without a predicated force term, raises registers 48 -> 71 and
  // costs occupancy: 1.6x slower.)
  __device__ __forceinline__ void update_with(const vf_collide_update_args& a, float eps2, bool damped) {
    const uint32_t me = idx;
    const float4 pi = __ldg(a.P_dev + me);
    const uint32_t es = __ldg(a.slot_dev + me);
    const int G = (int)a.G;
    const int cx = cell_coord(pi.x, a.rc, G), cy = cell_coord(pi.y, a.rc, G), cz = cell_coord(pi.z, a.rc, G);
    const int x0 = cx > 0 ? cx - 1 : 0, x1 = cx + 1 < G ? cx + 1 : G - 1;
    float ax = 0.0f, ay = 0.0f, az = 0.0f;
    float best = 0.0f;
    int32_t bestj = -1;
    const float rc2 = a.rc2, rm2 = a.rm2;
    for (int z = cz - 1; z <= cz + 1; ++z) {
      if (z < 0 || z >= G) continue;
      for (int y = cy - 1; y <= cy + 1; ++y) {
        if (y < 0 || y >= G) continue;
        const uint32_t row = ((uint32_t)z * (uint32_t)G + (uint32_t)y) * (uint32_t)G;
        const uint32_t e0 = __ldg(a.cell_start_dev + row + x0);
        const uint32_t e1 = __ldg(a.cell_start_dev + row + x1 + 1);
#pragma unroll 2
        for (uint32_t e = e0; e < e1; ++e) {
          const float4 pj = __ldg(a.Ps_dev + e);
          const float dx = pj.x - pi.x, dy = pj.y - pi.y, dz = pj.z - pi.z;
          const float d2 = fmaf(dx, dx, fmaf(dy, dy, dz * dz));
          const bool other = e != es;
          if (other && d2 < rc2) {  // ~1 candidate in 6 (sphere / 27 cells)
            const float r2 = fmaf(dx, dx, fmaf(dy, dy, fmaf(dz, dz, eps2)));
            const float sc = pj.w * rcp_rn_fast(r2 * sqrt_rn_fast(r2));  // m_j * (1.0f / (r2 * sqrtf(r2)))
            ax = fmaf(dx, sc, ax);
            ay = fmaf(dy, sc, ay);
            az = fmaf(dz, sc, az);
          }
          if (other && d2 < rm2 && (bestj < 0 || d2 <= best)) {  // rare: read the id
            const int32_t j = (int32_t)__ldg(a.list_dev + e);
            if (bestj < 0 || d2 < best || j < bestj) {
              best = d2;
              bestj = j;
            }
          }
        }
      }
    }
    float ux = vx, uy = vy, uz = vz;
    if (damped) {
      ux = ux * a.damp;
      uy = uy * a.damp;
      uz = uz * a.damp;
    }
    ux = fmaf(a.dt, ax, ux);
    uy = fmaf(a.dt, ay, uy);
    uz = fmaf(a.dt, az, uz);
    vx = ux;
    vy = uy;
    vz = uz;
    a.Pm_dev[me] = make_float4(fmaf(a.dt, ux, pi.x), fmaf(a.dt, uy, pi.y), fmaf(a.dt, uz, pi.z), pi.w);
    a.near_dev[me] = bestj;
    if (bestj >= 0) a.Vm_dev[me] = make_float4(ux, uy, uz, 0.0f);  // read only by a mutual partner
  }

  __device__ __forceinline__ void merge_common(const vf_collide_merge_args& a) {
    const uint32_t i = idx;
    const int32_t j = __ldg(a.near_dev + i);
    const float4 pm = __ldg(a.Pm_dev + i);
    if (j < 0 || __ldg(a.near_dev + j) != (int32_t)i) {
      a.P_dev[i] = pm;
      return;
    }
    if ((uint32_t)j > i) {  // i absorbs j
      const float4 pj = __ldg(a.Pm_dev + j);
      const float4 vj = __ldg(a.Vm_dev + j);
      const float mi = pm.w, mj = pj.w;
      const float m = mi + mj;
      const float px = __fdiv_rn(fmaf(mi, pm.x, mj * pj.x), m);
      const float py = __fdiv_rn(fmaf(mi, pm.y, mj * pj.y), m);
      const float pz = __fdiv_rn(fmaf(mi, pm.z, mj * pj.z), m);
      const float ux = __fdiv_rn(fmaf(mi, vx, mj * vj.x), m);
      const float uy = __fdiv_rn(fmaf(mi, vy, mj * vj.y), m);
      const float uz = __fdiv_rn(fmaf(mi, vz, mj * vj.z), m);
      vx = ux;
      vy = uy;
      vz = uz;
      a.P_dev[i] = make_float4(px, py, pz, m);
    } else {  // absorbed by j < i: inactive from now on, position kept
      a.P_dev[i] = make_float4(pm.x, pm.y, pm.z, 0.0f);
      vx = vy = vz = 0.0f;
    }
  }

  __device__ __forceinline__ void get_vel(const vf_collide_get_args& a) const {
    float* o = a.vel_out_dev + 3ull * (idx - a.idx_base);
    o[0] = vx;
    o[1] = vy;
    o[2] = vz;
  }
};

struct Star final : Body {
  __device__ explicit Star(const void* arg) : Body(arg) {}
  __device__ void update(const vf_collide_update_args& a) override { update_with(a, a.eps2[0], false); }
  __device__ void merge(const vf_collide_merge_args& a) override { merge_common(a); }
  __device__ void get(const vf_collide_get_args& a) override { get_vel(a); }
};

struct Planet final : Body {
  __device__ explicit Planet(const void* arg) : Body(arg) {}
  __device__ void update(const vf_collide_update_args& a) override { update_with(a, a.eps2[1], false); }
  __device__ void merge(const vf_collide_merge_args& a) override { merge_common(a); }
  __device__ void get(const vf_collide_get_args& a) override { get_vel(a); }
};

struct Dust final : Body {
  __device__ explicit Dust(const void* arg) : Body(arg) {}
  __device__ void update(const vf_collide_update_args& a) override { update_with(a, a.eps2[2], true); }
  __device__ void merge(const vf_collide_merge_args& a) override { merge_common(a); }
  __device__ void get(const vf_collide_get_args& a) override { get_vel(a); }
};

template <int K>
struct TypeOf;
template <>
struct TypeOf<0> { using T = Star; };
template <>
struct TypeOf<1> { using T = Planet; };
template <>
struct TypeOf<2> { using T = Dust; };

struct App {
  static constexpr int kTypes = 3;
  static constexpr int kMethods = 3;
  static constexpr int kUnroll = 1;
  static constexpr int kUnrollSorted = 1;
  static constexpr int kPrefetch = 0;
  static constexpr bool kLean = true;  // default launch configuration only (knob sweeps: micro)
  static constexpr bool kGridSort = true;  // heavy update: grid-level type sort (measured)
  static constexpr uint32_t kHeavyMask = 1u << VF_COLLIDE_UPDATE;  // one tile per CTA (dispatch.cuh grid_cap)
  static constexpr int kMinBlocks = 5;  // <= 48 registers: 40 warps per SM hide the gather latency
  using Base = Body;
  template <int K>
  using Type = typename TypeOf<K>::T;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_COLLIDE_UPDATE) o->update(blob_as<vf_collide_update_args>(b));
    else if constexpr (M == VF_COLLIDE_MERGE) o->merge(blob_as<vf_collide_merge_args>(b));
    else o->get(blob_as<vf_collide_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_COLLIDE_UPDATE) o->Type<K>::update(blob_as<vf_collide_update_args>(b));
    else if constexpr (M == VF_COLLIDE_MERGE) o->Type<K>::merge(blob_as<vf_collide_merge_args>(b));
    else o->Type<K>::get(blob_as<vf_collide_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(Star) == 24 && sizeof(Planet) == 24 && sizeof(Dust) == 24, "layouts");

// ---------------------------------------------------------------------------
// Step (0): the grid (non-virtual kernels).
// ---------------------------------------------------------------------------
constexpr int kScanThreads = 256;
constexpr int kScanPer = 16;
constexpr uint32_t kScanTile = kScanThreads * kScanPer;  // 4096 elements per block

// cell of every active body, per-cell counts, owned active count
__global__ void k_cells(uint32_t N, const float4* __restrict__ P, int G, float rc, uint32_t* __restrict__ cell_of,
                        uint32_t* __restrict__ count, uint32_t id_lo, uint32_t id_hi,
                        unsigned long long* active) {
  const uint32_t stride = gridDim.x * blockDim.x;
  uint32_t owned = 0;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < N; i += stride) {
    const float4 p = __ldg(P + i);
    uint32_t c = 0xFFFFFFFFu;
    if (p.w > 0.0f) {
      const uint32_t x = cell_coord(p.x, rc, G), y = cell_coord(p.y, rc, G), z = cell_coord(p.z, rc, G);
      c = (z * (uint32_t)G + y) * (uint32_t)G + x;
      atomicAdd(count + c, 1u);
      owned += (i >= id_lo && i < id_hi);
    }
    cell_of[i] = c;
  }
  if (active) {
    for (int o = 16; o > 0; o >>= 1) owned += __shfl_xor_sync(0xffffffffu, owned, o);
    if ((threadIdx.x & 31) == 0 && owned) atomicAdd(active, (unsigned long long)owned);
  }
}

__device__ __forceinline__ uint32_t block_exclusive_scan(uint32_t v, uint32_t* warp_sums, uint32_t& total) {
  const int lane = threadIdx.x & 31, w = threadIdx.x >> 5;
  uint32_t x = v;
  for (int o = 1; o < 32; o <<= 1) {
    const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
    if (lane >= o) x += y;
  }
  if (lane == 31) warp_sums[w] = x;
  __syncthreads();
  if (w == 0) {
    const int nw = blockDim.x >> 5;
    uint32_t s = lane < nw ? warp_sums[lane] : 0;
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, s, o);
      if (lane >= o) s += y;
    }
    if (lane < nw) warp_sums[lane] = s;  // inclusive
  }
  __syncthreads();
  total = warp_sums[(blockDim.x >> 5) - 1];
  const uint32_t before = w ? warp_sums[w - 1] : 0;
  __syncthreads();
  return before + x - v;
}

// pass 1: per-tile sums
__global__ void __launch_bounds__(kScanThreads) k_scan_reduce(const uint32_t* __restrict__ in, uint64_t n,
                                                              uint32_t* __restrict__ bsum) {
  __shared__ uint32_t ws[kScanThreads / 32];
  const uint64_t base = (uint64_t)blockIdx.x * kScanTile;
  uint32_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanPer; ++k) {
    const uint64_t i = base + (uint64_t)k * kScanThreads + threadIdx.x;
    if (i < n) s += in[i];
  }
  uint32_t total;
  block_exclusive_scan(s, ws, total);
  if (threadIdx.x == 0) bsum[blockIdx.x] = total;
}

// pass 2: one block scans the tile sums in place (exclusive); out[n] = total
__global__ void __launch_bounds__(1024) k_scan_tiles(uint32_t* __restrict__ bsum, uint32_t nb,
                                                     uint32_t* __restrict__ out, uint64_t n) {
  __shared__ uint32_t ws[32];
  uint32_t carry = 0;
  for (uint32_t b0 = 0; b0 < nb; b0 += blockDim.x) {
    const uint32_t b = b0 + threadIdx.x;
    const uint32_t v = b < nb ? bsum[b] : 0;
    uint32_t total;
    const uint32_t ex = block_exclusive_scan(v, ws, total);
    if (b < nb) bsum[b] = carry + ex;
    carry += total;
  }
  if (threadIdx.x == 0) out[n] = carry;
}

// pass 3: per-tile exclusive scan + tile offset (in may alias out)
__global__ void __launch_bounds__(kScanThreads) k_scan_apply(const uint32_t* in, uint64_t n,
                                                             const uint32_t* __restrict__ bsum, uint32_t* out) {
  __shared__ uint32_t ws[kScanThreads / 32];
  const uint64_t base = (uint64_t)blockIdx.x * kScanTile + (uint64_t)threadIdx.x * kScanPer;
  uint32_t v[kScanPer];
  uint32_t s = 0;
#pragma unroll
  for (int k = 0; k < kScanPer; ++k) {
    v[k] = base + k < n ? in[base + k] : 0;
    s += v[k];
  }
  uint32_t total;
  uint32_t run = block_exclusive_scan(s, ws, total) + bsum[blockIdx.x];
#pragma unroll
  for (int k = 0; k < kScanPer; ++k) {
    if (base + k < n) out[base + k] = run;
    run += v[k];
  }
}

// list[start[c] + ..] = ids of cell c (any order); counts return to zero
__global__ void k_fill(uint32_t N, const uint32_t* __restrict__ cell_of, uint32_t* __restrict__ count,
                       const uint32_t* __restrict__ start, uint32_t* __restrict__ list) {
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t i = blockIdx.x * blockDim.x + threadIdx.x; i < N; i += stride) {
    const uint32_t c = cell_of[i];
    if (c != 0xFFFFFFFFu) {
      const uint32_t k = atomicSub(count + c, 1u) - 1u;
      list[start[c] + k] = i;
    }
  }
}

// per cell: ids ascending (insertion sort; ~per_cell entries), then Ps
__global__ void k_sort_cells(uint32_t ncell, const uint32_t* __restrict__ start, uint32_t* __restrict__ list,
                             const float4* __restrict__ P, float4* __restrict__ Ps, uint32_t* __restrict__ slot) {
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t c = blockIdx.x * blockDim.x + threadIdx.x; c < ncell; c += stride) {
    const uint32_t s = start[c], e = start[c + 1];
    for (uint32_t k = s + 1; k < e; ++k) {
      const uint32_t x = list[k];
      uint32_t m = k;
      while (m > s && list[m - 1] > x) {
        list[m] = list[m - 1];
        --m;
      }
      list[m] = x;
    }
    for (uint32_t k = s; k < e; ++k) {
      const uint32_t id = list[k];
      Ps[k] = __ldg(P + id);
      slot[id] = k;
    }
  }
}

// single rank: order[e] = objs[list[e]] (cell order), null past the active count
__global__ void k_order_all(uint32_t N, const uint32_t* __restrict__ list, const uint32_t* __restrict__ total,
                            const uint64_t* __restrict__ objs, uint64_t* __restrict__ order) {
  const uint32_t nact = *total;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < N; e += stride)
    order[e] = e < nact ? __ldg(objs + __ldg(list + e)) : 0ull;
}

// several ranks: flag[e] = list[e] is owned (then scanned into positions)
__global__ void k_order_flags(uint32_t N, const uint32_t* __restrict__ list, const uint32_t* __restrict__ total,
                              uint32_t id_lo, uint32_t id_hi, uint32_t* __restrict__ flag) {
  const uint32_t nact = *total;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < N; e += stride) {
    uint32_t f = 0;
    if (e < nact) {
      const uint32_t id = __ldg(list + e);
      f = id >= id_lo && id < id_hi;
    }
    flag[e] = f;
  }
}

__global__ void k_order_scatter(uint32_t N, const uint32_t* __restrict__ list, const uint32_t* __restrict__ total,
                                const uint32_t* __restrict__ pos, uint32_t id_lo, uint32_t id_hi,
                                const uint64_t* __restrict__ objs, uint64_t* __restrict__ order) {
  const uint32_t nact = *total, nown = pos[N], cap = id_hi - id_lo;
  const uint32_t stride = gridDim.x * blockDim.x;
  for (uint32_t e = blockIdx.x * blockDim.x + threadIdx.x; e < N; e += stride) {
    if (e < nact) {
      const uint32_t id = __ldg(list + e);
      if (id >= id_lo && id < id_hi) order[pos[e]] = __ldg(objs + (id - id_lo));
    }
    if (e >= nown && e < cap) order[e] = 0ull;
  }
}

}  // namespace collide

static const uint32_t kCollideBytes[3] = {24, 24, 24};
static const uint32_t kCollideArgs[3] = {sizeof(vf_collide_update_args), sizeof(vf_collide_merge_args),
                                         sizeof(vf_collide_get_args)};

const AppOps* app_collide() {
  static const AppOps ops = make_ops<collide::App>("collide", kCollideBytes, kCollideArgs);
  return &ops;
}

// exclusive scan of in[0, n) into out[0, n] (out[n] = total); in may equal out.
static cudaError_t scan_u32(const uint32_t* in, uint32_t* out, uint64_t n, uint32_t* bsum, cudaStream_t s) {
  const uint32_t nb = (uint32_t)((n + collide::kScanTile - 1) / collide::kScanTile);
  if (nb) {
    collide::k_scan_reduce<<<nb, collide::kScanThreads, 0, s>>>(in, n, bsum);
    note_launch();
  }
  collide::k_scan_tiles<<<1, 1024, 0, s>>>(bsum, nb, out, n);
  note_launch();
  if (nb) {
    collide::k_scan_apply<<<nb, collide::kScanThreads, 0, s>>>(in, n, bsum, out);
    note_launch();
  }
  return cudaGetLastError();
}

}  // namespace vf

namespace vf {
namespace collide {
// Multi-GPU exchange after update: merge() on body i reads
// near[j], Pm[j], Vm[j] of its nearest body j = near[i] only when j has a
// partner (near[j] >= 0), so only those bodies' entries travel.
__global__ void k_pack_near(uint32_t lo, uint32_t hi, const int32_t* __restrict__ near, const float4* __restrict__ Pm,
                            const float4* __restrict__ Vm, vf_collide_near_entry* __restrict__ out,
                            uint32_t* __restrict__ count) {
  const uint32_t lane = threadIdx.x & 31u;
  for (uint64_t b = lo + (uint64_t)blockIdx.x * blockDim.x; b < hi; b += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t i = b + threadIdx.x;
    const bool take = i < hi && near[i] >= 0;
    const uint32_t m = __ballot_sync(0xffffffffu, take);
    if (!m) continue;
    const uint32_t leader = __ffs(m) - 1;
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(count, (uint32_t)__popc(m));
    base = __shfl_sync(0xffffffffu, base, leader);
    if (take) {
      vf_collide_near_entry e;
      e.id = (uint32_t)i;
      e.near = near[i];
      e.pad[0] = e.pad[1] = 0;
      const float4 pm = Pm[i], vm = Vm[i];
      e.Pm[0] = pm.x; e.Pm[1] = pm.y; e.Pm[2] = pm.z; e.Pm[3] = pm.w;
      e.Vm[0] = vm.x; e.Vm[1] = vm.y; e.Vm[2] = vm.z; e.Vm[3] = vm.w;
      out[base + __popc(m & ((1u << lane) - 1u))] = e;
    }
  }
}
// near[] of every body outside [lo, hi) back to -1 (no partner) ...
__global__ void k_reset_near(uint32_t N, uint32_t lo, uint32_t hi, int32_t* __restrict__ near) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < N; i += (uint64_t)gridDim.x * blockDim.x)
    if (i < lo || i >= hi) near[i] = -1;
}
// ... then the received entries: slot k of rank r's segment is valid iff k < counts[r]
__global__ void k_unpack_near(const vf_collide_near_entry* __restrict__ in, uint32_t nseg, uint32_t seg,
                              const int64_t* __restrict__ counts, uint32_t lo, uint32_t hi, int32_t* __restrict__ near,
                              float4* __restrict__ Pm, float4* __restrict__ Vm) {
  for (uint64_t k = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; k < (uint64_t)nseg * seg;
       k += (uint64_t)gridDim.x * blockDim.x) {
    if ((int64_t)(k % seg) >= counts[k / seg]) continue;
    const vf_collide_near_entry e = in[k];
    if (e.id >= lo && e.id < hi) continue;  // own entries are already in place
    near[e.id] = e.near;
    Pm[e.id] = make_float4(e.Pm[0], e.Pm[1], e.Pm[2], e.Pm[3]);
    Vm[e.id] = make_float4(e.Vm[0], e.Vm[1], e.Vm[2], e.Vm[3]);
  }
}
}  // namespace collide
}  // namespace vf

extern "C" vf_status vf_collide_pack_near(uint32_t lo, uint32_t hi, const int32_t* near_dev, const float* Pm_dev,
                                          const float* Vm_dev, vf_collide_near_entry* out_dev, uint32_t* count_dev,
                                          void* stream) {
  if (hi < lo || (hi > lo && (!near_dev || !Pm_dev || !Vm_dev || !out_dev || !count_dev))) return VF_ERR_INVALID;
  if (hi == lo) return VF_OK;
  vf::collide::k_pack_near<<<(unsigned)vf::num_sms() * 4, 256, 0, (cudaStream_t)stream>>>(
      lo, hi, near_dev, reinterpret_cast<const float4*>(Pm_dev), reinterpret_cast<const float4*>(Vm_dev), out_dev,
      count_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}

extern "C" vf_status vf_collide_unpack_near(const vf_collide_near_entry* in_dev, uint32_t nseg, uint32_t seg,
                                            const int64_t* counts_dev, uint32_t N, uint32_t lo, uint32_t hi,
                                            int32_t* near_dev, float* Pm_dev, float* Vm_dev, void* stream) {
  if (!near_dev || !Pm_dev || !Vm_dev || (nseg && seg && (!in_dev || !counts_dev)) || hi < lo || hi > N)
    return VF_ERR_INVALID;
  const cudaStream_t s = (cudaStream_t)stream;
  const unsigned grid = (unsigned)vf::num_sms() * 4;
  if (N) {
    vf::collide::k_reset_near<<<grid, 256, 0, s>>>(N, lo, hi, near_dev);
    vf::note_launch();
  }
  if (nseg && seg) {
    vf::collide::k_unpack_near<<<grid, 256, 0, s>>>(in_dev, nseg, seg, counts_dev, lo, hi, near_dev,
                                                     reinterpret_cast<float4*>(Pm_dev),
                                                     reinterpret_cast<float4*>(Vm_dev));
    vf::note_launch();
  }
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}

extern "C" uint64_t vf_collide_tmp_words(uint32_t N, uint32_t G) {
  const uint64_t ncell = (uint64_t)G * G * G;
  const uint64_t big = ncell > N ? ncell : N;
  return (uint64_t)N + 1 + (big + vf::collide::kScanTile - 1) / vf::collide::kScanTile + 1;
}

extern "C" vf_status vf_collide_grid(const vf_collide_grid_args* a, void* stream) {
  if (!a || a->G < 1 || a->G > 1024 || !(a->rc > 0.0f) || a->id_lo > a->id_hi || a->id_hi > a->N) return VF_ERR_INVALID;
  if (a->N && (!a->P_dev || !a->cell_of_dev || !a->cell_count_dev || !a->cell_start_dev || !a->list_dev ||
               !a->Ps_dev || !a->slot_dev || !a->tmp_dev))
    return VF_ERR_INVALID;
  if (a->id_hi > a->id_lo && (!a->objs_dev || !a->order_dev)) return VF_ERR_INVALID;
  const cudaStream_t s = (cudaStream_t)stream;
  const uint32_t N = a->N, G = a->G;
  const uint64_t ncell = (uint64_t)G * G * G;
  const unsigned grid = (unsigned)vf::num_sms() * 8;
  using namespace vf::collide;
  if (N) {
    k_cells<<<grid, 256, 0, s>>>(N, a->P_dev, (int)G, a->rc, a->cell_of_dev, a->cell_count_dev, a->id_lo, a->id_hi,
                                 a->active_dev);
    vf::note_launch();
  }
  uint32_t* flags = a->tmp_dev;            // N + 1
  uint32_t* bsum = a->tmp_dev + N + 1;     // tile sums
  cudaError_t e = vf::scan_u32(a->cell_count_dev, a->cell_start_dev, ncell, bsum, s);
  if (e != cudaSuccess) return VF_ERR_CUDA;
  if (N) {
    k_fill<<<grid, 256, 0, s>>>(N, a->cell_of_dev, a->cell_count_dev, a->cell_start_dev, a->list_dev);
    k_sort_cells<<<grid, 256, 0, s>>>((uint32_t)ncell, a->cell_start_dev, a->list_dev, a->P_dev, a->Ps_dev,
                                        a->slot_dev);
    vf::note_launch(2);
  }
  const uint32_t* total = a->cell_start_dev + ncell;
  if (a->id_hi > a->id_lo) {
    if (a->id_lo == 0 && a->id_hi == N) {
      k_order_all<<<grid, 256, 0, s>>>(N, a->list_dev, total, a->objs_dev, a->order_dev);
      vf::note_launch();
    } else {
      k_order_flags<<<grid, 256, 0, s>>>(N, a->list_dev, total, a->id_lo, a->id_hi, flags);
      vf::note_launch();
      e = vf::scan_u32(flags, flags, N, bsum, s);
      if (e != cudaSuccess) return VF_ERR_CUDA;
      k_order_scatter<<<grid, 256, 0, s>>>(N, a->list_dev, total, flags, a->id_lo, a->id_hi, a->objs_dev,
                                           a->order_dev);
      vf::note_launch();
    }
  }
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
