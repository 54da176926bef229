// oracle/graph_en.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// GraphChi-vEN-style graph apps (Table 2):
// BFS / CC / PageRank where BOTH vertices and edges are polymorphic objects
// and every edge access is a virtual call on an edge object (GraphChi's
// ChiEdge / Edge hierarchy: "also defines an
// abstract base class for vertex ... both virtual edges and nodes").
//
// Written the GraphChi way (vertex-centric update over edge objects that
// carry the data):
//   * one edge object per arc (u -> v) of the symmetric CSR, from plain `new`
//     in arc order; it holds src, dst and a double-buffered value (reading
//     G33: Jacobi iterations read buffer t&1 and write buffer (t+1)&1);
//   * every vertex keeps its in-edge list (pointers to the arcs (u -> v),
//     built here by walking the arcs in order, so ascending u) and its
//     out-edge list (its own arcs, ascending v);
//   * an update reads its in-edges through virtual get_*() and writes its
//     out-edges through virtual set_*(); BFS visits out-edges through the
//     virtual target().
// Edge classes (reading G32): abstract ChiEdge + Edge (source not a Hub) and
// HubEdge (source vertex of type Hub, deg >= 256), same semantics.
// Vertex classes: the four degree buckets of graph.cpp (reading G22).
#include "oracle.h"

#include <chrono>
#include <vector>

namespace {

struct ChiEdge {
  ChiEdge(uint32_t s, uint32_t d) : src(s), dst(d) { val.f[0] = val.f[1] = 0.0; }
  virtual ~ChiEdge() {}
  virtual uint32_t target() const = 0;
  virtual double get_pr(int buf) const = 0;
  virtual void set_pr(int buf, double x) = 0;
  virtual uint32_t get_label(int buf) const = 0;
  virtual void set_label(int buf, uint32_t x) = 0;
  uint32_t src, dst;
  union {
    double f[2];
    uint32_t u[2];
  } val;
};

template <int KIND>
struct EdgeK final : ChiEdge {
  EdgeK(uint32_t s, uint32_t d) : ChiEdge(s, d) {}
  uint32_t target() const override { return dst; }
  double get_pr(int buf) const override { return val.f[buf]; }
  void set_pr(int buf, double x) override { val.f[buf] = x; }
  uint32_t get_label(int buf) const override { return val.u[buf]; }
  void set_label(int buf, uint32_t x) override { val.u[buf] = x; }
};

struct Net {
  uint64_t V = 0;
  std::vector<ChiEdge*> edges;                 // arc order
  std::vector<std::vector<ChiEdge*>> in, out;  // per vertex
  ~Net() {
    for (ChiEdge* e : edges) delete e;
  }
};

struct ChiVertex {
  explicit ChiVertex(uint32_t v) : vid(v) {}
  virtual ~ChiVertex() {}
  // BFS top-down: claim unvisited targets of the out-edges for level+1
  virtual void bfs_expand(Net& n, int32_t* depth, int32_t level, std::vector<uint32_t>& next) = 0;
  // CC: m = min(label_in[v], in-edge labels of buffer b); out-edges get m in 1-b
  virtual int cc_update(Net& n, const uint32_t* in, uint32_t* out, int b) = 0;
  // PR: s = sum of in-edge values of buffer b (in-edge order); r' as in graph.cpp;
  // out-edges get r'/deg in 1-b; returns r'
  virtual float pr_update(Net& n, int b, double base, double d, double DV) = 0;
  uint32_t vid;
};

template <int KIND>
struct VertexK final : ChiVertex {
  explicit VertexK(uint32_t v) : ChiVertex(v) {}
  void bfs_expand(Net& n, int32_t* depth, int32_t level, std::vector<uint32_t>& next) override {
    for (ChiEdge* e : n.out[vid]) {
      const uint32_t u = e->target();  // virtual edge call
      if (depth[u] == -1) {
        depth[u] = level + 1;
        next.push_back(u);
      }
    }
  }
  int cc_update(Net& n, const uint32_t* in, uint32_t* out, int b) override {
    uint32_t m = in[vid];
    for (ChiEdge* e : n.in[vid]) {
      const uint32_t x = e->get_label(b);  // virtual edge call
      if (x < m) m = x;
    }
    out[vid] = m;
    for (ChiEdge* e : n.out[vid]) e->set_label(1 - b, m);  // virtual edge call
    return m != in[vid];
  }
  float pr_update(Net& n, int b, double base, double d, double DV) override {
    double s = 0.0;
    for (ChiEdge* e : n.in[vid]) s += e->get_pr(b);  // virtual edge call
    const float r = (float)(base + d * (s + DV));
    const size_t deg = n.out[vid].size();
    for (ChiEdge* e : n.out[vid]) e->set_pr(1 - b, (double)r / (double)deg);  // virtual edge call
    return r;
  }
};

// Edges in arc order; type HubEdge iff the source vertex is a Hub (type 3).
void build_net(Net& n, uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* vtypes) {
  n.V = V;
  n.in.assign(V, {});
  n.out.assign(V, {});
  n.edges.reserve(offs[V]);
  for (uint64_t u = 0; u < V; ++u) {
    for (uint64_t k = offs[u]; k < offs[u + 1]; ++k) {
      ChiEdge* e = vtypes[u] == 3 ? (ChiEdge*)new EdgeK<1>((uint32_t)u, col[k])
                                  : (ChiEdge*)new EdgeK<0>((uint32_t)u, col[k]);
      n.edges.push_back(e);
      n.out[u].push_back(e);
      n.in[col[k]].push_back(e);  // arcs visited with ascending u
    }
  }
}

std::vector<ChiVertex*> make_vertices(uint64_t V, const uint32_t* types) {
  std::vector<ChiVertex*> vs(V);
  for (uint64_t v = 0; v < V; ++v) {
    switch (types[v]) {
      case 0: vs[v] = new VertexK<0>((uint32_t)v); break;
      case 1: vs[v] = new VertexK<1>((uint32_t)v); break;
      case 2: vs[v] = new VertexK<2>((uint32_t)v); break;
      default: vs[v] = new VertexK<3>((uint32_t)v); break;
    }
  }
  return vs;
}
void free_vertices(std::vector<ChiVertex*>& vs) {
  for (ChiVertex* v : vs) delete v;
}
double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
}  // namespace

extern "C" int oracle_graph_en_edge_types(uint64_t V, const uint64_t* offs, const uint32_t* vtypes,
                                          uint32_t* etypes) {
  for (uint64_t u = 0; u < V; ++u)
    for (uint64_t k = offs[u]; k < offs[u + 1]; ++k) etypes[k] = vtypes[u] == 3 ? 1u : 0u;
  return 0;
}

extern "C" int oracle_graph_en_bfs(uint64_t V, const uint64_t* offs, const uint32_t* col,
                                   const uint32_t* types, uint32_t src, int32_t* depth,
                                   uint32_t* levels, uint64_t* vcalls, uint64_t* ecalls,
                                   double* seconds) {
  if (src >= V) return 1;
  Net n;
  build_net(n, V, offs, col, types);
  std::vector<ChiVertex*> vs = make_vertices(V, types);
  for (uint64_t v = 0; v < V; ++v) depth[v] = -1;
  const double t0 = now();
  depth[src] = 0;
  std::vector<uint32_t> frontier{src}, next;
  int32_t level = 0;
  uint64_t nv = 0, ne = 0;
  while (!frontier.empty()) {
    next.clear();
    for (uint32_t v : frontier) {
      vs[v]->bfs_expand(n, depth, level, next);  // virtual vertex call
      ne += n.out[v].size();
    }
    nv += frontier.size();
    frontier.swap(next);
    ++level;
  }
  if (seconds) *seconds = now() - t0;
  if (levels) *levels = (uint32_t)level;
  if (vcalls) *vcalls = nv;
  if (ecalls) *ecalls = ne;
  free_vertices(vs);
  return 0;
}

extern "C" int oracle_graph_en_cc(uint64_t V, const uint64_t* offs, const uint32_t* col,
                                  const uint32_t* types, uint32_t* label, uint32_t* iters,
                                  uint64_t* vcalls, uint64_t* ecalls, double* seconds) {
  Net n;
  build_net(n, V, offs, col, types);
  std::vector<ChiVertex*> vs = make_vertices(V, types);
  std::vector<uint32_t> a(V), bb(V);
  for (uint64_t v = 0; v < V; ++v) a[v] = (uint32_t)v;
  for (ChiEdge* e : n.edges) e->set_label(0, e->src);  // edge data = the source's label
  const double t0 = now();
  uint32_t it = 0;
  int b = 0;
  while (true) {
    int64_t changed = 0;
    for (uint64_t v = 0; v < V; ++v) changed += vs[v]->cc_update(n, a.data(), bb.data(), b);
    ++it;
    a.swap(bb);
    b = 1 - b;
    if (!changed) break;
  }
  if (seconds) *seconds = now() - t0;
  for (uint64_t v = 0; v < V; ++v) label[v] = a[v];
  if (iters) *iters = it;
  if (vcalls) *vcalls = (uint64_t)it * V;
  if (ecalls) *ecalls = (uint64_t)it * 2 * offs[V];
  free_vertices(vs);
  return 0;
}

extern "C" int oracle_graph_en_pr(uint64_t V, const uint64_t* offs, const uint32_t* col,
                                  const uint32_t* types, double d, uint32_t iters, float* rank,
                                  double* seconds) {
  Net n;
  build_net(n, V, offs, col, types);
  std::vector<ChiVertex*> vs = make_vertices(V, types);
  std::vector<float> r(V, (float)(1.0 / (double)V)), rn(V);
  // initial edge data r0(u)/deg(u) and dangling mass D0 (vertex order)
  double D = 0.0;
  for (uint64_t u = 0; u < V; ++u) {
    const uint64_t deg = offs[u + 1] - offs[u];
    for (ChiEdge* e : n.out[u]) e->set_pr(0, (double)r[u] / (double)deg);
    if (!deg) D += (double)r[u];
  }
  const double t0 = now();
  int b = 0;
  for (uint32_t t = 0; t < iters; ++t) {
    double Dn = 0.0;
    for (uint64_t v = 0; v < V; ++v) {
      rn[v] = vs[v]->pr_update(n, b, (1.0 - d) / (double)V, d, D / (double)V);  // virtual
      if (offs[v + 1] == offs[v]) Dn += (double)rn[v];
    }
    r.swap(rn);
    D = Dn;
    b = 1 - b;
  }
  if (seconds) *seconds = now() - t0;
  for (uint64_t v = 0; v < V; ++v) rank[v] = r[v];
  free_vertices(vs);
  return 0;
}
