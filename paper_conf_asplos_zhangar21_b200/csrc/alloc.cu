// alloc.cu — device side of the batched typed allocation (vf_alloc_typed_batch,
// SURVEY §8(b)): object i of class types[i] takes the next free slot of its
// type's arena IN INDEX ORDER (SharedOA; regions P:979-999), i.e.
// its slot is its rank among the objects of the same type with a smaller
// index. The ranks are an exclusive per-type prefix count over the type
// array, computed here on the device so a 2^26-object batch never brings the
// type array (or the pointers) back to the host:
//   1. k_type_hist   per 4096-object chunk, count each type       (chunk x T)
//   2. k_hist_scan   per type, exclusive scan over the chunks     (+ totals)
//   -- host reads back the T totals (T x 8 B), maps regions, uploads the
//      per-type segment list (rank range -> first address)
//   3. k_place       per chunk, recompute each object's rank in index order
//      (warp match_any + per-warp counts in shared memory), look up its
//      type's segment and write the (tagged) pointer
// plus k_place_packed for the cuda_packed sensitivity variant (placement into
// one index-ordered slab, SURVEY §7 "A fair CUDA baseline").
#include <cuda_runtime.h>
#include <stdint.h>

#include "vf_internal.h"

namespace vf {
namespace alloc {

constexpr int kThreads = 256;
constexpr int kRounds = 16;
constexpr uint32_t kChunk = kThreads * kRounds;  // objects per chunk (one CTA)

__global__ void __launch_bounds__(kThreads) k_type_hist(const uint32_t* __restrict__ types, uint64_t n,
                                                        uint32_t ntypes, uint32_t* __restrict__ hist,
                                                        uint32_t* __restrict__ bad) {
  __shared__ uint32_t h[32];
  if (threadIdx.x < 32) h[threadIdx.x] = 0;
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * kChunk;
  const uint32_t lane = threadIdx.x & 31u;
  for (int r = 0; r < kRounds; ++r) {
    const uint64_t i = base + (uint64_t)r * kThreads + threadIdx.x;
    uint32_t t = i < n ? __ldg(types + i) : 0xFFFFu;
    if (i < n && t >= ntypes) {
      atomicOr(bad, 1u);
      t = 0xFFFFu;
    }
    const uint32_t peers = __match_any_sync(0xffffffffu, t);
    if (t < 32u && lane == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&h[t], (uint32_t)__popc(peers));
  }
  __syncthreads();
  if (threadIdx.x < 32) hist[(uint64_t)blockIdx.x * 32 + threadIdx.x] = h[threadIdx.x];
}

// one warp per type: exclusive scan of hist[.][t] over the chunks (in place)
__global__ void k_hist_scan(uint32_t* __restrict__ hist, uint64_t nchunks, uint32_t ntypes,
                            unsigned long long* __restrict__ totals) {
  const uint32_t t = threadIdx.x >> 5, lane = threadIdx.x & 31u;
  if (t >= ntypes) return;
  unsigned long long run = 0;
  for (uint64_t b0 = 0; b0 < nchunks; b0 += 32) {
    const uint64_t b = b0 + lane;
    const uint32_t v = b < nchunks ? hist[b * 32 + t] : 0u;
    uint32_t x = v;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= (uint32_t)o) x += y;
    }
    if (b < nchunks) hist[b * 32 + t] = (uint32_t)(run + x - v);  // ranks < 2^32 per type
    run += __shfl_sync(0xffffffffu, x, 31);
  }
  if (lane == 0) totals[t] = run;
}

__global__ void __launch_bounds__(kThreads) k_place(const uint32_t* __restrict__ types, uint64_t n,
                                                    const uint32_t* __restrict__ offs, const PlaceSeg* __restrict__ segs,
                                                    const uint32_t* __restrict__ seg_first, int tag,
                                                    uint64_t* __restrict__ out) {
  constexpr int kWarps = kThreads / 32;
  __shared__ uint32_t run[32];
  __shared__ uint32_t wcnt[kWarps][32];
  __shared__ uint32_t boff[32];
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  if (threadIdx.x < 32) {
    run[threadIdx.x] = 0;
    boff[threadIdx.x] = offs[(uint64_t)blockIdx.x * 32 + threadIdx.x];
  }
  const uint64_t base = (uint64_t)blockIdx.x * kChunk;
  for (int r = 0; r < kRounds; ++r) {
    const uint64_t i = base + (uint64_t)r * kThreads + threadIdx.x;
    const bool v = i < n;
    const uint32_t t = v ? __ldg(types + i) : 0xFFFFu;  // validated by k_type_hist
    wcnt[warp][lane] = 0;
    __syncwarp();
    const uint32_t peers = __match_any_sync(0xffffffffu, t);
    const uint32_t within = __popc(peers & ((1u << lane) - 1u));
    if (v && lane == (uint32_t)(__ffs(peers) - 1)) wcnt[warp][t] = __popc(peers);
    __syncthreads();
    if (v) {
      uint32_t before = run[t];
      for (uint32_t w = 0; w < warp; ++w) before += wcnt[w][t];
      const uint64_t rank = (uint64_t)boff[t] + before + within;
      // the type's segments are consecutive and sorted by first rank
      uint32_t k = seg_first[t];
      const uint32_t kend = seg_first[t + 1];
      while (k + 1 < kend && segs[k + 1].rank0 <= rank) ++k;
      const PlaceSeg s = segs[k];
      uint64_t a = s.addr + (rank - s.rank0) * s.obj_bytes;
      if (tag) a |= (uint64_t)(t + 1) << VF_VA_BITS;
      out[i] = a;
    }
    __syncthreads();
    if (threadIdx.x < 32) {
      uint32_t s = 0;
      for (int w = 0; w < kWarps; ++w) s += wcnt[w][threadIdx.x];
      run[threadIdx.x] += s;
    }
    __syncthreads();
  }
}

__global__ void k_place_packed(uint64_t base, uint64_t stride, uint64_t n, uint64_t* __restrict__ out) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = base + i * stride;
}

__global__ void k_fill_u32(uint32_t* __restrict__ x, uint64_t n, uint32_t v) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n; i += (uint64_t)gridDim.x * blockDim.x)
    x[i] = v;
}

}  // namespace alloc

uint64_t rank_chunks(uint64_t n) { return (n + alloc::kChunk - 1) / alloc::kChunk; }

cudaError_t rank_hist(const uint32_t* types, uint64_t n, uint32_t ntypes, uint32_t* hist, uint32_t* bad,
                      unsigned long long* totals, cudaStream_t s) {
  const uint64_t nb = rank_chunks(n);
  if (nb > 0x7FFFFFFFull) return cudaErrorInvalidValue;
  alloc::k_type_hist<<<(unsigned)nb, alloc::kThreads, 0, s>>>(types, n, ntypes, hist, bad);
  note_launch();
  alloc::k_hist_scan<<<1, 32 * 32, 0, s>>>(hist, nb, ntypes, totals);
  note_launch();
  return cudaGetLastError();
}

cudaError_t scan_type_hist(uint32_t* hist, uint64_t nchunks, uint32_t ntypes, unsigned long long* totals,
                           cudaStream_t s) {
  alloc::k_hist_scan<<<1, 32 * 32, 0, s>>>(hist, nchunks, ntypes, totals);
  note_launch();
  return cudaGetLastError();
}

cudaError_t rank_place(const uint32_t* types, uint64_t n, const uint32_t* hist, const PlaceSeg* segs,
                       const uint32_t* seg_first, int tag, uint64_t* out, cudaStream_t s) {
  const uint64_t nb = rank_chunks(n);
  alloc::k_place<<<(unsigned)nb, alloc::kThreads, 0, s>>>(types, n, hist, segs, seg_first, tag, out);
  note_launch();
  return cudaGetLastError();
}

cudaError_t place_packed(uint64_t base, uint64_t stride, uint64_t n, uint64_t* out, cudaStream_t s) {
  alloc::k_place_packed<<<1184, 256, 0, s>>>(base, stride, n, out);
  note_launch();
  return cudaGetLastError();
}

cudaError_t fill_u32(uint32_t* x, uint64_t n, uint32_t v, cudaStream_t s) {
  alloc::k_fill_u32<<<1184, 256, 0, s>>>(x, n, v);
  note_launch();
  return cudaGetLastError();
}

}  // namespace vf
