// oracle/graph.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 4: BFS / CC / PageRank over polymorphic vertices (Table 2 GraphChi-vE
// P:1538-1564 uses polymorphic edges; BASELINE north_star asks for polymorphic
// vertices: reading G22). Vertex classes by degree bucket — Leaf (deg <= 1),
// Low (2..15), Mid (16..255), Hub (>= 256) — all implement the same method
// semantics; the oracle writes each as the plain loop over the CSR row.
// Readings G20/G21/G23: RMAT input, d = 0.85 with uniform dangling
// redistribution, level-synchronous BFS (depths are unique, so direction does
// not matter), Jacobi (double-buffered) min-label CC.
#include "oracle.h"

#include <chrono>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct G {
  uint64_t V;
  const uint64_t* offs;
  const uint32_t* col;
};

struct Vertex {
  explicit Vertex(uint32_t v) : vid(v) {}
  virtual ~Vertex() {}
  // BFS top-down: claim unvisited neighbours for the next level
  virtual void bfs_expand(const G& g, int32_t* depth, int32_t level, std::vector<uint32_t>& next) = 0;
  // CC (Jacobi): out[v] = min(in[v], min over neighbours in[u]); returns 1 if changed
  virtual int cc_update(const G& g, const uint32_t* in, uint32_t* out) = 0;
  // PageRank pull: s_v = sum over neighbours of contrib[u] (CSR order, fp64)
  virtual double pr_gather(const G& g, const double* contrib) = 0;
  uint32_t vid;
};

template <int KIND>
struct VertexK final : Vertex {
  explicit VertexK(uint32_t v) : Vertex(v) {}
  void bfs_expand(const G& g, int32_t* depth, int32_t level, std::vector<uint32_t>& next) override {
    for (uint64_t e = g.offs[vid]; e < g.offs[vid + 1]; ++e) {
      const uint32_t u = g.col[e];
      if (depth[u] == -1) {
        depth[u] = level + 1;
        next.push_back(u);
      }
    }
  }
  int cc_update(const G& g, const uint32_t* in, uint32_t* out) override {
    uint32_t m = in[vid];
    for (uint64_t e = g.offs[vid]; e < g.offs[vid + 1]; ++e)
      if (in[g.col[e]] < m) m = in[g.col[e]];
    out[vid] = m;
    return m != in[vid];
  }
  double pr_gather(const G& g, const double* contrib) override {
    double s = 0.0;
    for (uint64_t e = g.offs[vid]; e < g.offs[vid + 1]; ++e) s += contrib[g.col[e]];
    return s;
  }
};

std::vector<Vertex*> make_vertices(uint64_t V, const uint32_t* types) {
  std::vector<Vertex*> vs(V);
  for (uint64_t v = 0; v < V; ++v) {  // allocation in index order
    switch (types[v]) {
      case 0: vs[v] = new VertexK<0>((uint32_t)v); break;
      case 1: vs[v] = new VertexK<1>((uint32_t)v); break;
      case 2: vs[v] = new VertexK<2>((uint32_t)v); break;
      default: vs[v] = new VertexK<3>((uint32_t)v); break;
    }
  }
  return vs;
}
void free_vertices(std::vector<Vertex*>& vs) {
  for (Vertex* v : vs) delete v;
}
double now() {
  return std::chrono::duration<double>(std::chrono::steady_clock::now().time_since_epoch()).count();
}
}  // namespace

extern "C" int oracle_graph_bfs(uint64_t V, const uint64_t* offs, const uint32_t* col,
                                const uint32_t* types, uint32_t src, int32_t* depth,
                                uint32_t* levels, uint64_t* calls, double* seconds) {
  if (src >= V) return 1;
  G g{V, offs, col};
  std::vector<Vertex*> vs = make_vertices(V, types);
  for (uint64_t v = 0; v < V; ++v) depth[v] = -1;
  double t0 = now();
  depth[src] = 0;
  std::vector<uint32_t> frontier{src}, next;
  int32_t level = 0;
  uint64_t ncalls = 0;
  while (!frontier.empty()) {
    next.clear();
    for (uint32_t v : frontier) vs[v]->bfs_expand(g, depth, level, next);  // virtual call
    ncalls += frontier.size();
    frontier.swap(next);
    ++level;
  }
  if (seconds) *seconds = now() - t0;
  if (levels) *levels = (uint32_t)level;
  if (calls) *calls = ncalls;
  free_vertices(vs);
  return 0;
}

extern "C" int oracle_graph_cc(uint64_t V, const uint64_t* offs, const uint32_t* col,
                               const uint32_t* types, int threads, uint32_t* label,
                               uint32_t* iters, uint64_t* calls, double* seconds) {
  G g{V, offs, col};
  std::vector<Vertex*> vs = make_vertices(V, types);
  std::vector<uint32_t> a(V), b(V);
  for (uint64_t v = 0; v < V; ++v) a[v] = (uint32_t)v;
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  double t0 = now();
  uint32_t it = 0;
  while (true) {
    int64_t changed = 0;
#pragma omp parallel for schedule(dynamic, 1024) reduction(+ : changed) if (threads != 1)
    for (int64_t v = 0; v < (int64_t)V; ++v) changed += vs[v]->cc_update(g, a.data(), b.data());
    ++it;
    a.swap(b);
    if (!changed) break;
  }
  if (seconds) *seconds = now() - t0;
  for (uint64_t v = 0; v < V; ++v) label[v] = a[v];
  if (iters) *iters = it;
  if (calls) *calls = (uint64_t)it * V;
  free_vertices(vs);
  return 0;
}

extern "C" int oracle_graph_pr(uint64_t V, const uint64_t* offs, const uint32_t* col,
                               const uint32_t* types, double d, uint32_t iters, int threads,
                               float* rank, double* seconds) {
  G g{V, offs, col};
  std::vector<Vertex*> vs = make_vertices(V, types);
  std::vector<float> r(V, (float)(1.0 / (double)V)), rn(V);
  std::vector<double> contrib(V);
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  double t0 = now();
  for (uint32_t t = 0; t < iters; ++t) {
    // contributions and dangling mass D_t (vertex order)
    double D = 0.0;
    for (uint64_t u = 0; u < V; ++u) {
      const uint64_t deg = offs[u + 1] - offs[u];
      contrib[u] = deg ? (double)r[u] / (double)deg : 0.0;
      if (!deg) D += (double)r[u];
    }
#pragma omp parallel for schedule(dynamic, 1024) if (threads != 1)
    for (int64_t v = 0; v < (int64_t)V; ++v) {
      const double s = vs[v]->pr_gather(g, contrib.data());  // virtual call
      rn[v] = (float)((1.0 - d) / (double)V + d * (s + D / (double)V));
    }
    r.swap(rn);
  }
  if (seconds) *seconds = now() - t0;
  for (uint64_t v = 0; v < V; ++v) rank[v] = r[v];
  free_vertices(vs);
  return 0;
}
