// graph_common.cuh — CSR work-entry helpers shared by the vertex-only graph
// apps (app_graph.cu, GraphChi-vE style) and the virtual-edge apps
// (app_graph_en.cu, GraphChi-vEN style). Work entries: vf.h VF_APP_GRAPH.
#pragma once
#include "dispatch.cuh"

namespace vf {
namespace graph {

// L2 residency (B200: 126 MB of L2). The per-vertex state a body gathers at
// random (PageRank contributions, CC labels, BFS depths / frontier bits: 64-
// 134 MB at RMAT-24) is loaded with an evict_last policy so the adjacency
// stream `col` (2 GB, read once per sweep) does not push it out of L2. (An
// evict_first policy on `col` itself was measured worse on B200: a lane reads
// its row 4 B at a time, and the sector was evicted between its reads.)
__device__ __forceinline__ uint64_t l2_keep() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_last.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint64_t l2_stream() {
  uint64_t p;
  asm("createpolicy.fractional.L2::evict_first.b64 %0, 1.0;" : "=l"(p));
  return p;
}
__device__ __forceinline__ uint32_t ld_hint(const uint32_t* a, uint64_t pol) {
  uint32_t v;
  asm("ld.global.nc.L2::cache_hint.u32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ int32_t ld_hint(const int32_t* a, uint64_t pol) {
  int32_t v;
  asm("ld.global.nc.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ float ld_hint(const float* a, uint64_t pol) {
  float v;
  asm("ld.global.nc.L2::cache_hint.f32 %0, [%1], %2;" : "=f"(v) : "l"(a), "l"(pol));
  return v;
}
__device__ __forceinline__ double ld_hint(const double* a, uint64_t pol) {
  double v;
  asm("ld.global.nc.L2::cache_hint.f64 %0, [%1], %2;" : "=d"(v) : "l"(a), "l"(pol));
  return v;
}

// coherent (non-.nc) load with a policy: state this kernel also writes
__device__ __forceinline__ int32_t ld_hint_rw(const int32_t* a, uint64_t pol) {
  int32_t v;
  asm volatile("ld.global.L2::cache_hint.s32 %0, [%1], %2;" : "=r"(v) : "l"(a), "l"(pol));
  return v;
}

// Neighbour loop with U independent lanes of work (U = 1: plain loop).
template <int U, class F>
__device__ __forceinline__ void for_neighbors(const uint32_t* __restrict__ col, uint64_t b, uint64_t e, F&& f) {
  uint64_t k = b;
  if constexpr (U > 1) {
    for (; k + U <= e; k += U) {
      uint32_t u[U];
#pragma unroll
      for (int j = 0; j < U; ++j) u[j] = __ldg(col + k + j);
#pragma unroll
      for (int j = 0; j < U; ++j) f(u[j]);
    }
  }
  for (; k < e; ++k) f(__ldg(col + k));
}

// Visit col[b..e) with f(j, u): the 16 B-aligned middle with 16 B vector
// loads, U neighbour ids per step (U / 4 loads in flight, then U independent
// bodies, f's j = 0..U-1 a compile-time lane of independent work after
// unrolling), the unaligned head and the tail one id at a time with j = 0.
// (Per-lane 4 B loads cost one L1 wavefront each: RMAT-24 PageRank was bound
// by L1 throughput, 75% of peak, with half of the wavefronts on `col`.)
template <int U, class F>
__device__ __forceinline__ void for_edges_v(const uint32_t* __restrict__ col, uint64_t b, uint64_t e, F&& f) {
  static_assert(U % 4 == 0, "U is a multiple of 4");
  uint64_t k = b;
  uint64_t h = b + ((4u - (uint32_t)((reinterpret_cast<uintptr_t>(col + b) >> 2) & 3u)) & 3u);
  if (h > e) h = e;
  for (; k < h; ++k) f(0, __ldg(col + k));
  for (; k + U <= e; k += U) {
    uint4 v[U / 4];
#pragma unroll
    for (int j = 0; j < U / 4; ++j) v[j] = __ldg(reinterpret_cast<const uint4*>(col + k) + j);
#pragma unroll
    for (int j = 0; j < U / 4; ++j) {
      f(4 * j, v[j].x);
      f(4 * j + 1, v[j].y);
      f(4 * j + 2, v[j].z);
      f(4 * j + 3, v[j].w);
    }
  }
  if (k + 4 <= e && U > 4) {
    const uint4 v = __ldg(reinterpret_cast<const uint4*>(col + k));
    f(0, v.x);
    f(1, v.y);
    f(2, v.z);
    f(3, v.w);
    k += 4;
  }
  for (; k < e; ++k) f(0, __ldg(col + k));
}

// Is there a neighbour u in col[b..e) with pred(u)? 4 ids per 16 B vector
// load and their 4 predicate loads in flight; stops after the first step
// that holds a hit (bottom-up BFS: the answer, not the neighbour, matters).
template <class P>
__device__ __forceinline__ bool any_edge_v(const uint32_t* __restrict__ col, uint64_t b, uint64_t e, P&& pred) {
  uint64_t k = b;
  uint64_t h = b + ((4u - (uint32_t)((reinterpret_cast<uintptr_t>(col + b) >> 2) & 3u)) & 3u);
  if (h > e) h = e;
  for (; k < h; ++k)
    if (pred(__ldg(col + k))) return true;
  for (; k + 4 <= e; k += 4) {
    const uint4 v = __ldg(reinterpret_cast<const uint4*>(col + k));
    const bool p0 = pred(v.x), p1 = pred(v.y), p2 = pred(v.z), p3 = pred(v.w);
    if (p0 | p1 | p2 | p3) return true;
  }
  for (; k < e; ++k)
    if (pred(__ldg(col + k))) return true;
  return false;
}

__device__ __forceinline__ uint32_t nchunks(uint32_t deg, uint32_t C) { return deg <= C ? 1u : (deg + C - 1) / C; }

// The edge range of work entry i of vertex (vid, deg): chunk c of <= C edges.
// Single-chunk vertices (deg <= C, nearly all) never read the chunk array.
struct Work {
  uint64_t b, e;
  uint32_t c, nch;
};
__device__ __forceinline__ Work work_of(const uint64_t* offs, const uint32_t* chunk, uint64_t i, uint32_t vid,
                                        uint32_t deg, uint32_t C) {
  Work w;
  w.nch = nchunks(deg, C);
  w.c = w.nch > 1 ? __ldg(chunk + i) : 0u;
  const uint64_t b0 = __ldg(offs + vid);
  w.b = b0 + (uint64_t)w.c * C;
  const uint64_t e0 = b0 + deg;
  w.e = w.b + C < e0 ? w.b + C : e0;
  return w;
}

// Append vertex u's work entries to the next BFS frontier. Single-chunk
// vertices reserve their slots with one warp-aggregated atomic per group of
// lanes that claim at the same time, multi-chunk ones alone.
template <class BfsArgs>
__device__ __forceinline__ void enqueue(const BfsArgs& a, uint32_t u) {
  const uint32_t d = (uint32_t)(__ldg(a.offs_dev + u + 1) - __ldg(a.offs_dev + u));
  const uint32_t n = nchunks(d, a.C);
  const uint64_t obj = __ldg(a.vobj_dev + u);
  if (n == 1) {
    const uint32_t m = __activemask();
    const uint32_t lane = threadIdx.x & 31u;
    const uint32_t leader = __ffs(m) - 1;
    uint32_t base = 0;
    if (lane == leader) base = atomicAdd(a.next_count_dev, (uint32_t)__popc(m));
    base = __shfl_sync(m, base, leader) + __popc(m & ((1u << lane) - 1u));
    a.next_queue_dev[base] = obj;
    a.next_chunk_dev[base] = 0;
  } else {
    const uint32_t base = atomicAdd(a.next_count_dev, n);
    for (uint32_t j = 0; j < n; ++j) {
      a.next_queue_dev[base + j] = obj;
      a.next_chunk_dev[base + j] = j;
    }
  }
}

}  // namespace graph
}  // namespace vf
