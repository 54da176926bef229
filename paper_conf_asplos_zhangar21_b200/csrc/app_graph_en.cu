// app_graph_en.cu — GraphChi-vEN style graph apps: BFS / CC / PageRank where
// vertices AND edges are polymorphic objects and every edge access is a
// virtual call on an edge object (Table 2: "also defines an
// abstract base class for vertex, ChiVertex ... both virtual edges and
// nodes"; edges ChiEdge / Edge P:1542-1546; readings G32/G33).
//
// Two apps live in this ONE module (a vTable* is only valid in the module
// that constructed the object, and vertex methods call edge
// methods): VF_APP_GRAPH_EN (ChiVertex; Leaf / Low / Mid / Hub by degree, as
// app_graph.cu) and VF_APP_EDGE (ChiEdge; Edge / HubEdge by source degree).
//
// Nested edge calls. The vertex methods are written once, templated on
// DIRECT:
//   * DIRECT = false is what the virtual vertex method runs (VF_CUDA /
//     VF_SHAREDOA, and the indirect-call ablation): each edge access is the
//     compiler's virtual call — vTable* load, vFunc* load, indirect CALL.
//   * DIRECT = true is what the COAL / TypePointer kernels call by qualified
//     name: each edge pointer is typed from its value (er.rule: the edge
//     app's range table, or the tag), the lanes of a batch of edges are
//     grouped by edge type, and each present type's accessor runs once,
//     inlined (no CALL). Unresolvable pointers fall back to the embedded
//     vTable* (P:1305-1311).
//
// Object layouts: vertex 16 B { vTable*, u32 vid, u32 deg };
// edge 32 B { vTable*, u32 src, u32 dst, union { f64 f[2]; u32 u[2]; } }.
#include <type_traits>

#include "graph_common.cuh"

namespace vf {
namespace graph_en {

using graph::nchunks;
using graph::Work;
using graph::work_of;

// ------------------------------------------------------------------ edges
struct EdgeCtor {
  uint32_t src, dst;
};

struct ChiEdge {
  __device__ explicit ChiEdge(const void* arg)
      : src(arg ? static_cast<const EdgeCtor*>(arg)->src : 0), dst(arg ? static_cast<const EdgeCtor*>(arg)->dst : 0) {
    val.f[0] = 0.0;
    val.f[1] = 0.0;
  }
  __device__ virtual ~ChiEdge() {}
  // dispatched over the edge arrays (VF_EDGE_*)
  __device__ virtual void pull_pr(vf_edge_args a, uint64_t i) = 0;
  __device__ virtual void pull_label(vf_edge_args a, uint64_t i) = 0;
  __device__ virtual void get(vf_edge_args a, uint64_t i) = 0;
  // called from vertex methods
  __device__ virtual uint32_t target() const = 0;
  __device__ virtual double get_pr(uint32_t b) const = 0;
  __device__ virtual uint32_t get_label(uint32_t b) const = 0;
  uint32_t src, dst;
  union {
    double f[2];
    uint32_t u[2];
  } val;
};

template <int KIND>
struct EdgeK final : ChiEdge {
  __device__ explicit EdgeK(const void* arg) : ChiEdge(arg) {}
  __device__ void pull_pr(vf_edge_args a, uint64_t) override { val.f[a.slot] = __ldg(a.contrib_dev + src); }
  __device__ void pull_label(vf_edge_args a, uint64_t) override { val.u[a.slot] = __ldg(a.label_dev + src); }
  __device__ void get(vf_edge_args a, uint64_t i) override { a.out_dev[i] = (uint64_t)src << 32 | dst; }
  __device__ uint32_t target() const override { return dst; }
  __device__ double get_pr(uint32_t b) const override { return val.f[b]; }
  __device__ uint32_t get_label(uint32_t b) const override { return val.u[b]; }
};
static_assert(sizeof(EdgeK<0>) == 32, "edge layout");

struct EdgeApp {
  static constexpr int kTypes = 2;
  static constexpr int kMethods = 3;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  static constexpr bool kLean = true;
  using Base = ChiEdge;
  template <int K>
  using Type = EdgeK<K>;
  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_EDGE_PULL_PR) o->pull_pr(blob_as<vf_edge_args>(b), i);
    else if constexpr (M == VF_EDGE_PULL_LABEL) o->pull_label(blob_as<vf_edge_args>(b), i);
    else o->get(blob_as<vf_edge_args>(b), i);
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_EDGE_PULL_PR) o->Type<K>::pull_pr(blob_as<vf_edge_args>(b), i);
    else if constexpr (M == VF_EDGE_PULL_LABEL) o->Type<K>::pull_label(blob_as<vf_edge_args>(b), i);
    else o->Type<K>::get(blob_as<vf_edge_args>(b), i);
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) { construct_switch<EdgeApp>(t, mem, arg); }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<EdgeApp>(t, arg); }
};

// Accessors: a ChiEdge* is a virtual call; an EdgeK<K>* a direct, qualified one.
__device__ __forceinline__ uint32_t e_target(const ChiEdge* e) { return e->target(); }
__device__ __forceinline__ double e_get_pr(const ChiEdge* e, uint32_t b) { return e->get_pr(b); }
__device__ __forceinline__ uint32_t e_get_label(const ChiEdge* e, uint32_t b) { return e->get_label(b); }
template <int K>
__device__ __forceinline__ uint32_t e_target(const EdgeK<K>* e) { return e->EdgeK<K>::target(); }
template <int K>
__device__ __forceinline__ double e_get_pr(const EdgeK<K>* e, uint32_t b) { return e->EdgeK<K>::get_pr(b); }
template <int K>
__device__ __forceinline__ uint32_t e_get_label(const EdgeK<K>* e, uint32_t b) { return e->EdgeK<K>::get_label(b); }

// COAL for edges: the two most recently hit ranges of the edge app's table are
// kept in registers (an out-edge list is all one type; an in-edge list mixes
// the two edge types), so the branch-free search over the table (L1-resident,
// global memory) runs only on a miss.
struct EdgeRangeCache {
  uint64_t s0 = ~0ull, e0 = 0, s1 = ~0ull, e1 = 0;
  uint32_t t0 = kNF, t1 = kNF;
};

// Type of edge pointer p from its value (COAL: cached ranges, else the range
// search; TypePointer: the tag), else from the embedded vTable*. a = the
// address to dereference.
__device__ __forceinline__ uint32_t edge_type(const vf_edge_resolver& r, EdgeRangeCache& rc, uint64_t p,
                                              uint64_t& a) {
  uint32_t t;
  if (r.rule == VF_TYPEPTR) {
    a = strip(p);
    t = ((uint32_t)(p >> 32) >> (VF_VA_BITS - 32)) - 1u;
  } else {
    a = p;
    if ((rc.s0 <= p) & (p < rc.e0)) {
      t = rc.t0;
    } else if ((rc.s1 <= p) & (p < rc.e1)) {
      t = rc.t1;
    } else {
      uint32_t j = 0;
      for (uint32_t step = r.P >> 1; step > 0; step >>= 1) {
        const uint32_t c = j + step;
        j = (c < r.K && __ldg(r.start_dev + c) <= p) ? c : j;
      }
      const uint64_t s = __ldg(r.start_dev + j), e = __ldg(r.end_dev + j);
      t = (s <= p && p < e) ? __ldg(r.type_dev + j) : kNF;
      if (t != kNF) {
        rc.s1 = rc.s0, rc.e1 = rc.e0, rc.t1 = rc.t0;
        rc.s0 = s, rc.e0 = e, rc.t0 = t;
      }
    }
  }
  if (t >= (uint32_t)EdgeApp::kTypes) {  // fallback
    const uint64_t vp = *reinterpret_cast<const uint64_t*>(a);
    t = vp == __ldg(r.vptr_dev) ? 0u : vp == __ldg(r.vptr_dev + 1) ? 1u : kNF;
  }
  return t;
}

// A batch of U edge pointers (one per unrolled slot of this lane): resolve
// all, then run each edge type present among the active lanes' batches once,
// over every slot of that type (independent loads stay in flight together).
template <int U, class F>
__device__ __forceinline__ void visit_direct(const vf_edge_resolver& r, EdgeRangeCache& rc, const uint64_t (&p)[U],
                                             F&& f) {
  uint64_t a[U];
  uint32_t t[U];
  uint32_t mine = 0;
#pragma unroll
  for (int j = 0; j < U; ++j) {
    t[j] = edge_type(r, rc, p[j], a[j]);
    mine |= t[j] < (uint32_t)EdgeApp::kTypes ? 1u << t[j] : 0u;
  }
  const uint32_t present = __reduce_or_sync(__activemask(), mine);
  if (present & 1u) {
#pragma unroll
    for (int j = 0; j < U; ++j)
      if (t[j] == 0u) f(j, reinterpret_cast<const EdgeK<0>*>(a[j]));
  }
  if (present & 2u) {
#pragma unroll
    for (int j = 0; j < U; ++j)
      if (t[j] == 1u) f(j, reinterpret_cast<const EdgeK<1>*>(a[j]));
  }
}

template <bool DIRECT, int U, class F>
__device__ __forceinline__ void visit(const vf_edge_resolver& r, EdgeRangeCache& rc, const uint64_t (&p)[U], F&& f) {
  if constexpr (DIRECT) {
    visit_direct<U>(r, rc, p, f);
  } else {
#pragma unroll
    for (int j = 0; j < U; ++j) f(j, reinterpret_cast<const ChiEdge*>(p[j]));
  }
}

// Edge k in [b, e) of a pointer array (out- or in-edges), U per batch: the
// edge call `get` (an accessor: target / get_label / get_pr) yields one value
// per slot inside the type groups; `use(j, value)` then consumes the slots in
// edge order outside them (one copy of the vertex's own logic, all lanes
// converged, whatever mix of edge types the batch held).
template <class T, bool DIRECT, int U, class G, class C>
__device__ __forceinline__ void for_edges(const vf_edge_resolver& r, const uint64_t* __restrict__ ptrs, uint64_t b,
                                          uint64_t e, G&& get, C&& use) {
  EdgeRangeCache rc;
  uint64_t k = b;
  if constexpr (U > 1) {
    for (; k + U <= e; k += U) {
      uint64_t p[U];
#pragma unroll
      for (int j = 0; j < U; ++j) p[j] = ldg_u64(ptrs + k + j);
      T v[U];
      visit<DIRECT, U>(r, rc, p, [&](int j, auto* ed) { v[j] = get(ed); });
#pragma unroll
      for (int j = 0; j < U; ++j) use(j, v[j]);
    }
  }
  for (; k < e; ++k) {
    const uint64_t p[1] = {ldg_u64(ptrs + k)};
    T v[1];
    visit<DIRECT, 1>(r, rc, p, [&](int j, auto* ed) { v[j] = get(ed); });
    use(0, v[0]);
  }
}

// ------------------------------------------------------------------ vertices
struct VCtor {
  uint32_t vid, deg;
};

struct ChiVertex {
  __device__ explicit ChiVertex(const void* arg)
      : vid(arg ? static_cast<const VCtor*>(arg)->vid : 0), deg(arg ? static_cast<const VCtor*>(arg)->deg : 0) {}
  __device__ virtual ~ChiVertex() {}
  __device__ virtual void bfs_expand(vf_graph_en_bfs_args a, uint64_t i) = 0;
  __device__ virtual void cc_update(vf_graph_en_cc_args a, uint64_t i) = 0;
  __device__ virtual void pr_init(vf_graph_en_pr_args a, uint64_t i) = 0;
  __device__ virtual void pr_gather(vf_graph_en_pr_args a, uint64_t i) = 0;
  uint32_t vid;
  uint32_t deg;
};

// dangling mass: one fp64 atomic per group of lanes that get here together
__device__ __forceinline__ void add_dangling(double* D, float r) {
  const uint32_t m = __activemask();
  const double x = (double)r;
  double total = 0.0;
  for (uint32_t mm = m; mm; mm &= mm - 1) total += __shfl_sync(m, x, __ffs(mm) - 1);
  if ((threadIdx.x & 31u) == (uint32_t)(__ffs(m) - 1)) atomicAdd(D, total);
}

template <int KIND>
struct VertexK final : ChiVertex {
  static constexpr int U = KIND <= 1 ? 1 : 4;
  __device__ explicit VertexK(const void* arg) : ChiVertex(arg) {}

  template <bool D>
  __device__ __forceinline__ void bfs_expand_t(const vf_graph_en_bfs_args& a, uint64_t i) {
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    for_edges<uint32_t, D, U>(
        a.er, a.out_edges_dev, w.b, w.e, [](auto* e) { return e_target(e); },  // edge call
        [&](int, uint32_t u) {
          if (a.depth_dev[u] == -1 && atomicCAS(a.depth_dev + u, -1, a.level + 1) == -1) graph::enqueue(a, u);
        });
  }
  template <bool D>
  __device__ __forceinline__ void cc_update_t(const vf_graph_en_cc_args& a, uint64_t i) {
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    const uint32_t own = __ldg(a.label_in_dev + vid);
    uint32_t acc[U];
#pragma unroll
    for (int j = 0; j < U; ++j) acc[j] = own;
    const uint32_t b = a.b;
    for_edges<uint32_t, D, U>(
        a.er, a.in_edges_dev, w.b, w.e, [b](auto* e) { return e_get_label(e, b); },  // edge call
        [&](int j, uint32_t x) { acc[j] = min(acc[j], x); });
    uint32_t m = own;
#pragma unroll
    for (int j = 0; j < U; ++j) m = min(m, acc[j]);
    if (w.nch == 1) a.label_out_dev[vid] = m;
    else atomicMin(a.label_out_dev + vid, m);
    if (m != own && __ldcg(a.changed_dev) == 0u) a.changed_dev[0] = 1u;  // (see app_graph.cu cc_update)
  }
  __device__ __forceinline__ void pr_init_t(const vf_graph_en_pr_args& a, uint64_t i) {
    if (nchunks(deg, a.C) > 1 && __ldg(a.chunk_dev + i) != 0) return;  // once per vertex
    const float r = a.rank_in_dev[vid];
    a.contrib_dev[vid] = deg ? (double)r / (double)deg : 0.0;
    if (!deg) add_dangling(a.dangling_out_dev, r);
  }
  template <bool D>
  __device__ __forceinline__ void pr_gather_t(const vf_graph_en_pr_args& a, uint64_t i) {
    const Work w = work_of(a.offs_dev, a.chunk_dev, i, vid, deg, a.C);
    double acc[U];
#pragma unroll
    for (int j = 0; j < U; ++j) acc[j] = 0.0;
    const uint32_t b = a.b;
    for_edges<double, D, U>(
        a.er, a.in_edges_dev, w.b, w.e, [b](auto* e) { return e_get_pr(e, b); },  // edge call
        [&](int j, double x) { acc[j] += x; });
    double s = 0.0;
#pragma unroll
    for (int j = 0; j < U; ++j) s += acc[j];
    if (w.nch > 1) {
      // last-finisher combine, in chunk order (deterministic), as VF_GRAPH_PR_UPDATE
      a.partial_dev[i] = s;
      __threadfence();
      if (atomicAdd(a.counter_dev + vid, 1u) != w.nch - 1) return;
      __threadfence();
      const uint64_t first = i - w.c;
      s = 0.0;
      for (uint32_t j = 0; j < w.nch; ++j) s += __ldcg(a.partial_dev + first + j);
      a.counter_dev[vid] = 0;
    }
    const double Dt = *a.dangling_in_dev;
    const float r = (float)__dadd_rn(a.base, __dmul_rn(a.d, __dadd_rn(s, __ddiv_rn(Dt, a.Vd))));
    a.rank_out_dev[vid] = r;
    a.contrib_dev[vid] = deg ? (double)r / (double)deg : 0.0;
    if (!deg) add_dangling(a.dangling_out_dev, r);
  }

  // virtual methods: edge accesses are virtual calls
  __device__ void bfs_expand(vf_graph_en_bfs_args a, uint64_t i) override { bfs_expand_t<false>(a, i); }
  __device__ void cc_update(vf_graph_en_cc_args a, uint64_t i) override { cc_update_t<false>(a, i); }
  __device__ void pr_init(vf_graph_en_pr_args a, uint64_t i) override { pr_init_t(a, i); }
  __device__ void pr_gather(vf_graph_en_pr_args a, uint64_t i) override { pr_gather_t<false>(a, i); }
};
static_assert(sizeof(VertexK<0>) == 16, "vertex layout");

struct VtxApp {
  static constexpr int kTypes = 4;
  static constexpr int kMethods = 4;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  static constexpr uint32_t kHeavyMask = 0xBu;  // bfs, cc, gather: one tile per CTA
  static constexpr bool kLean = true;           // default launch configuration only
  static constexpr int kMinBlocks = 3;          // <= 80 registers: random edge gathers need warps
  using Base = ChiVertex;
  template <int K>
  using Type = VertexK<K>;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_GRAPH_EN_BFS_EXPAND) o->bfs_expand(blob_as<vf_graph_en_bfs_args>(b), i);
    else if constexpr (M == VF_GRAPH_EN_CC_UPDATE) o->cc_update(blob_as<vf_graph_en_cc_args>(b), i);
    else if constexpr (M == VF_GRAPH_EN_PR_INIT) o->pr_init(blob_as<vf_graph_en_pr_args>(b), i);
    else o->pr_gather(blob_as<vf_graph_en_pr_args>(b), i);
  }
  // devirtualised vertex call (COAL / TypePointer): the edge calls inside are
  // devirtualised too
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_GRAPH_EN_BFS_EXPAND)
      o->Type<K>::template bfs_expand_t<true>(blob_as<vf_graph_en_bfs_args>(b), i);
    else if constexpr (M == VF_GRAPH_EN_CC_UPDATE)
      o->Type<K>::template cc_update_t<true>(blob_as<vf_graph_en_cc_args>(b), i);
    else if constexpr (M == VF_GRAPH_EN_PR_INIT)
      o->Type<K>::pr_init_t(blob_as<vf_graph_en_pr_args>(b), i);
    else
      o->Type<K>::template pr_gather_t<true>(blob_as<vf_graph_en_pr_args>(b), i);
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) { construct_switch<VtxApp>(t, mem, arg); }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<VtxApp>(t, arg); }
};

}  // namespace graph_en

static const uint32_t kEnVtxBytes[4] = {16, 16, 16, 16};
static const uint32_t kEnVtxArgs[4] = {sizeof(vf_graph_en_bfs_args), sizeof(vf_graph_en_cc_args),
                                       sizeof(vf_graph_en_pr_args), sizeof(vf_graph_en_pr_args)};
static const uint32_t kEdgeBytes[2] = {32, 32};
static const uint32_t kEdgeArgs[3] = {sizeof(vf_edge_args), sizeof(vf_edge_args), sizeof(vf_edge_args)};

const AppOps* app_graph_en() {
  static const AppOps ops = make_ops<graph_en::VtxApp>("graph_en", kEnVtxBytes, kEnVtxArgs);
  return &ops;
}
const AppOps* app_edge() {
  static const AppOps ops = make_ops<graph_en::EdgeApp>("edge", kEdgeBytes, kEdgeArgs);
  return &ops;
}

}  // namespace vf
