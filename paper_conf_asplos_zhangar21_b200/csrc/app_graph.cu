// app_graph.cu — config 4: BFS / CC / PageRank over polymorphic vertices
// (Table 2 GraphChi apps; BASELINE north_star: polymorphic
// vertices on a synthetic RMAT graph, reading G22). Vertex classes by degree
// bucket: Leaf (deg <= 1), Low (2..15), Mid (16..255), Hub (>= 256). All four
// implement the same semantics (the oracle's plain loops); each picks the
// loop shape that suits its degree: U independent neighbour ids per step (16 B
// vector loads of the row, for_edges_v) and U independent accumulators, U = 4
// for Leaf / Low, 8 for Mid / Hub.
// High-degree vertices are split into work entries of <= C edges (vf.h), so no
// lane walks a hub's whole row. (Measured on B200: sharing one member's row
// across the group's lanes in turn — coalesced but serial per vertex — was
// 1.2-1.5x SLOWER than these per-lane loops at RMAT-24.)
//
// Object layout (16 B): { vTable* (8 B), u32 vid, u32 deg }.
#include "graph_common.cuh"

namespace vf {
namespace graph {

struct CtorArg {
  uint32_t vid, deg;
};

struct Vertex {
  __device__ explicit Vertex(const void* arg)
      : vid(arg ? static_cast<const CtorArg*>(arg)->vid : 0),
        deg(arg ? static_cast<const CtorArg*>(arg)->deg : 0) {}
  __device__ virtual ~Vertex() {}
  // i = index of this call's work entry in the dispatched array (its chunk)
  __device__ virtual void bfs_expand(vf_graph_bfs_args a, uint64_t i) = 0;
  __device__ virtual void bfs_probe(vf_graph_bfs_args a, uint64_t i) = 0;
  __device__ virtual void cc_update(vf_graph_cc_args a, uint64_t i) = 0;
  __device__ virtual void pr_contrib(vf_graph_pr_args a, uint64_t i) = 0;
  __device__ virtual void pr_update(vf_graph_pr_args a, uint64_t i) = 0;
  __device__ virtual void bfs_probe_bits(vf_graph_bfs_bits_args a, uint64_t i) = 0;
  uint32_t vid;
  uint32_t deg;
};

template <int KIND>
struct VertexK final : Vertex {
  static constexpr int U = KIND <= 1 ? 4 : 8;
  __device__ explicit VertexK(const void* arg) : Vertex(arg) {}

  __device__ void bfs_expand(vf_graph_bfs_args a, uint64_t i) {
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    const uint64_t keep = l2_keep();
    for_edges_v<U>(a.col_dev, w.b, w.e, [&](int, uint32_t u) {
      if (ld_hint_rw(a.depth_dev + u, keep) == -1 && atomicCAS(a.depth_dev + u, -1, a.level + 1) == -1) enqueue(a, u);
    });
  }
  // bottom-up step: an unvisited vertex joins level+1 if a neighbour is at `level`
  __device__ void bfs_probe(vf_graph_bfs_args a, uint64_t i) {
    if (*(volatile int32_t*)(a.depth_dev + vid) != -1) return;
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    const uint64_t keep = l2_keep();
    for (uint64_t k = w.b; k < w.e; ++k) {
      // depth values of earlier levels are final: a stale read of this
      // launch's updates (level + 1) cannot equal `level`
      if (ld_hint(a.depth_dev + __ldg(a.col_dev + k), keep) == a.level) {
        if (atomicCAS(a.depth_dev + vid, -1, a.level + 1) == -1) *(volatile uint32_t*)a.next_count_dev = 1u;
        return;
      }
    }
  }
  // bottom-up step over a frontier bitmap (multi-GPU exchange unit)
  __device__ void bfs_probe_bits(vf_graph_bfs_bits_args a, uint64_t i) {
    if (*(volatile int32_t*)(a.depth_dev + vid) != -1) return;
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    const uint64_t keep = l2_keep();
    for (uint64_t k = w.b; k < w.e; ++k) {
      const uint32_t u = __ldg(a.col_dev + k);
      if ((ld_hint(a.frontier_dev + (u >> 5), keep) >> (u & 31u)) & 1u) {
        if (atomicCAS(a.depth_dev + vid, -1, a.level + 1) == -1) {
          atomicOr(a.next_dev + (vid >> 5), 1u << (vid & 31u));
          *(volatile uint32_t*)a.next_count_dev = 1u;
        }
        return;
      }
    }
  }
  __device__ void cc_update(vf_graph_cc_args a, uint64_t i) {
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    const uint32_t own = __ldg(a.label_in_dev + vid);
    const uint64_t keep = l2_keep();
    uint32_t acc[U];
#pragma unroll
    for (int j = 0; j < U; ++j) acc[j] = own;
    for_edges_v<U>(a.col_dev, w.b, w.e,
                   [&](int j, uint32_t u) { acc[j] = min(acc[j], ld_hint(a.label_in_dev + u, keep)); });
    uint32_t m = own;
#pragma unroll
    for (int j = 0; j < U; ++j) m = min(m, acc[j]);
    if (w.nch == 1) a.label_out_dev[vid] = m;
    else atomicMin(a.label_out_dev + vid, m);
    // "some label changed": millions of lanes set one flag in the first
    // iterations, and same-address stores serialise in L2 (measured: the
    // first CC sweeps took 3.3 ms against 2.2 ms once labels settle), so a
    // lane stores only while the flag still reads 0 from L2
    if (m != own && __ldcg(a.changed_dev) == 0u) a.changed_dev[0] = 1u;
  }
  __device__ void pr_contrib(vf_graph_pr_args a, uint64_t i) {
    if (nchunks(deg, a.C) > 1 && __ldg(a.chunk_dev + i) != 0) return;  // once per vertex
    const float r = a.rank_in_dev[vid];
    a.contrib_dev[vid] = deg ? (float)((double)r / (double)deg) : 0.0f;
    if (!deg) {
      // dangling mass: one fp64 atomic per group of lanes that get here together
      // (RMAT graphs have millions of isolated vertices: per-lane atomics on one
      // address serialise in L2); the group sum is taken in lane order
      const uint32_t m = __activemask();
      const double x = (double)r;
      double total = 0.0;
      for (uint32_t mm = m; mm; mm &= mm - 1) total += __shfl_sync(m, x, __ffs(mm) - 1);
      if ((threadIdx.x & 31u) == (uint32_t)(__ffs(m) - 1)) atomicAdd(a.dangling_dev, total);
    }
  }
  __device__ void pr_update(vf_graph_pr_args a, uint64_t i) {
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    const uint64_t keep = l2_keep();
    double acc[4] = {0.0, 0.0, 0.0, 0.0};  // U gathers in flight, 4 fp64 chains (64 registers)
    for_edges_v<U>(a.col_dev, w.b, w.e,
                   [&](int j, uint32_t u) { acc[j & 3] += (double)ld_hint(a.contrib_dev + u, keep); });
    double s = (acc[0] + acc[1]) + (acc[2] + acc[3]);
    if (w.nch > 1) {
      // last-finisher combine, in chunk order (deterministic)
      a.partial_dev[i] = s;
      __threadfence();
      if (atomicAdd(a.counter_dev + vid, 1u) != w.nch - 1) return;
      __threadfence();
      const uint64_t first = i - w.c;
      s = 0.0;
      for (uint32_t j = 0; j < w.nch; ++j) s += __ldcg(a.partial_dev + first + j);
      a.counter_dev[vid] = 0;
    }
    const double D = *a.dangling_dev;
    // (1-d)/V + d*(s + D/V), the oracle's operation order, IEEE fp64 (no contraction)
    a.rank_out_dev[vid] = (float)__dadd_rn(a.base, __dmul_rn(a.d, __dadd_rn(s, __ddiv_rn(D, a.Vd))));
  }
};

struct App {
  static constexpr int kTypes = 4;
  static constexpr int kMethods = 6;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  static constexpr bool kLean = true;  // default launch configuration only (knob sweeps: micro)
  static constexpr uint32_t kHeavyMask = 0x3Fu;  // one tile per CTA (dispatch.cuh grid_cap)
  static constexpr int kMinBlocks = 5;           // <= 48 registers: random gathers need resident warps
  using Base = Vertex;
  template <int K>
  using Type = VertexK<K>;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_GRAPH_BFS_EXPAND) o->bfs_expand(blob_as<vf_graph_bfs_args>(b), i);
    else if constexpr (M == VF_GRAPH_BFS_PROBE) o->bfs_probe(blob_as<vf_graph_bfs_args>(b), i);
    else if constexpr (M == VF_GRAPH_CC_UPDATE) o->cc_update(blob_as<vf_graph_cc_args>(b), i);
    else if constexpr (M == VF_GRAPH_PR_CONTRIB) o->pr_contrib(blob_as<vf_graph_pr_args>(b), i);
    else if constexpr (M == VF_GRAPH_PR_UPDATE) o->pr_update(blob_as<vf_graph_pr_args>(b), i);
    else o->bfs_probe_bits(blob_as<vf_graph_bfs_bits_args>(b), i);
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_GRAPH_BFS_EXPAND) o->Type<K>::bfs_expand(blob_as<vf_graph_bfs_args>(b), i);
    else if constexpr (M == VF_GRAPH_BFS_PROBE) o->Type<K>::bfs_probe(blob_as<vf_graph_bfs_args>(b), i);
    else if constexpr (M == VF_GRAPH_CC_UPDATE) o->Type<K>::cc_update(blob_as<vf_graph_cc_args>(b), i);
    else if constexpr (M == VF_GRAPH_PR_CONTRIB) o->Type<K>::pr_contrib(blob_as<vf_graph_pr_args>(b), i);
    else if constexpr (M == VF_GRAPH_PR_UPDATE) o->Type<K>::pr_update(blob_as<vf_graph_pr_args>(b), i);
    else o->Type<K>::bfs_probe_bits(blob_as<vf_graph_bfs_bits_args>(b), i);
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(VertexK<0>) == 16, "vertex layout");

__global__ void k_bfs_init(uint64_t V, int32_t* depth, uint32_t src, const uint64_t* vobj, const uint64_t* offs,
                           uint32_t C, uint64_t* queue, uint32_t* qchunk, uint32_t* count) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v < V) depth[v] = v == src ? 0 : -1;
  const uint32_t n = nchunks((uint32_t)(offs[src + 1] - offs[src]), C);
  if (v < n) {
    queue[v] = vobj[src];
    qchunk[v] = (uint32_t)v;
  }
  if (v == 0) *count = n;
}

__global__ void k_iota(uint64_t V, uint32_t* x) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v < V) x[v] = (uint32_t)v;
}

__global__ void k_fill_f32(uint64_t V, float* x, float val) {
  const uint64_t v = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (v < V) x[v] = val;
}

}  // namespace graph

static const uint32_t kGraphBytes[4] = {16, 16, 16, 16};
static const uint32_t kGraphArgs[6] = {sizeof(vf_graph_bfs_args), sizeof(vf_graph_bfs_args),
                                       sizeof(vf_graph_cc_args), sizeof(vf_graph_pr_args),
                                       sizeof(vf_graph_pr_args), sizeof(vf_graph_bfs_bits_args)};

const AppOps* app_graph() {
  static const AppOps ops = make_ops<graph::App>("graph", kGraphBytes, kGraphArgs);
  return &ops;
}

}  // namespace vf

extern "C" vf_status vf_graph_bfs_init(uint64_t V, int32_t* depth_dev, uint32_t src, const uint64_t* vobj_dev,
                                       const uint64_t* offs_dev, uint32_t C, uint64_t* queue_dev,
                                       uint32_t* queue_chunk_dev, uint32_t* count_dev, void* stream) {
  if (!V || src >= V || !depth_dev || !vobj_dev || !offs_dev || !C || !queue_dev || !queue_chunk_dev || !count_dev)
    return VF_ERR_INVALID;
  // V threads also cover src's chunks: nch <= deg <= V
  vf::graph::k_bfs_init<<<(unsigned)((V + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      V, depth_dev, src, vobj_dev, offs_dev, C, queue_dev, queue_chunk_dev, count_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}

extern "C" vf_status vf_iota_u32(uint64_t n, uint32_t* x_dev, void* stream) {
  if (!n) return VF_OK;
  if (!x_dev) return VF_ERR_INVALID;
  vf::graph::k_iota<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(n, x_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}

extern "C" vf_status vf_fill_f32(uint64_t n, float* x_dev, float value, void* stream) {
  if (!n) return VF_OK;
  if (!x_dev) return VF_ERR_INVALID;
  vf::graph::k_fill_f32<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(n, x_dev, value);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
