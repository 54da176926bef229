// synth/rmat.cpp — seeded synthetic graph INPUT generator (Graph500-style
// RMAT / Kronecker) shared by the oracle tests and the CUDA path. Holds none
// of the method's arithmetic (no BFS / CC / PageRank, no dispatch): it only
// draws edges and lays them out as a symmetric, de-duplicated CSR.
//
// Recipe:
//   edge e, level l (0..scale-1): u = draw(seed, S_GRAPH, e*scale + l),
//   quadrant by (u >> 32) against A, A+B, A+B+C (x 2^32): 0 -> (0,0),
//   1 -> (0,1), 2 -> (1,0), 3 -> (1,1) bits of (src, dst) at level l;
//   vertex ids permuted by perm[v] (random keys draw(seed, S_PERM, v), sorted);
//   self loops dropped, both directions added, duplicates removed, each
//   adjacency list sorted ascending.
#include <stdint.h>

#include <algorithm>
#include <numeric>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#include <parallel/algorithm>
#endif

static inline uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}
static inline uint64_t draw(uint64_t seed, uint64_t stream, uint64_t i) {
  return splitmix64(seed ^ (stream << 56) ^ i);
}

extern "C" {

// Raw directed RMAT edges (before permutation / cleanup).
void synth_rmat_edges(uint32_t scale, uint64_t nedges, double A, double B, double C, uint64_t seed,
                      uint64_t stream, uint32_t* src, uint32_t* dst) {
  const uint64_t tA = (uint64_t)(A * 4294967296.0);
  const uint64_t tAB = (uint64_t)((A + B) * 4294967296.0);
  const uint64_t tABC = (uint64_t)((A + B + C) * 4294967296.0);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < (int64_t)nedges; ++e) {
    uint32_t s = 0, d = 0;
    for (uint32_t l = 0; l < scale; ++l) {
      const uint64_t u = draw(seed, stream, (uint64_t)e * scale + l) >> 32;
      const uint32_t q = u < tA ? 0 : u < tAB ? 1 : u < tABC ? 2 : 3;
      s = (s << 1) | (q >> 1);
      d = (d << 1) | (q & 1);
    }
    src[e] = s;
    dst[e] = d;
  }
}

// Random permutation of [0, n): ranks of random keys (ties by index).
void synth_permutation(uint64_t n, uint64_t seed, uint64_t stream, uint32_t* perm) {
  std::vector<uint64_t> key(n);
  std::vector<uint32_t> idx(n);
#pragma omp parallel for schedule(static)
  for (int64_t v = 0; v < (int64_t)n; ++v) {
    key[v] = draw(seed, stream, (uint64_t)v);
    idx[v] = (uint32_t)v;
  }
  // (key, index) pairs are distinct: any correct sort gives the same order
  auto less = [&](uint32_t a, uint32_t b) { return key[a] < key[b] || (key[a] == key[b] && a < b); };
#ifdef _OPENMP
  __gnu_parallel::sort(idx.begin(), idx.end(), less);
#else
  std::sort(idx.begin(), idx.end(), less);
#endif
  for (uint64_t r = 0; r < n; ++r) perm[idx[r]] = (uint32_t)r;
}

// Symmetric CSR from directed edges (optionally relabelled by perm):
// drop self loops, add both directions, sort + unique each list.
// Fills offs[0..V] and col (capacity >= 2*nedges); returns the arc count.
uint64_t synth_csr(uint64_t V, uint64_t nedges, const uint32_t* src, const uint32_t* dst,
                   const uint32_t* perm, uint64_t* offs, uint32_t* col) {
  // raw degree with duplicates (parallel; counts are order-free)
  std::vector<uint64_t> rawdeg(V + 1, 0);
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < (int64_t)nedges; ++e) {
    uint32_t s = perm ? perm[src[e]] : src[e], d = perm ? perm[dst[e]] : dst[e];
    if (s == d) continue;
    __atomic_fetch_add(&rawdeg[s + 1], 1ull, __ATOMIC_RELAXED);
    __atomic_fetch_add(&rawdeg[d + 1], 1ull, __ATOMIC_RELAXED);
  }
  for (uint64_t v = 0; v < V; ++v) rawdeg[v + 1] += rawdeg[v];
  std::vector<uint32_t> adj(rawdeg[V]);
  std::vector<uint64_t> fill(rawdeg.begin(), rawdeg.end() - 1);
  // scatter in parallel: the order inside a list is arbitrary here, but every
  // list is sorted and de-duplicated below, so the CSR is deterministic
#pragma omp parallel for schedule(static)
  for (int64_t e = 0; e < (int64_t)nedges; ++e) {
    uint32_t s = perm ? perm[src[e]] : src[e], d = perm ? perm[dst[e]] : dst[e];
    if (s == d) continue;
    adj[__atomic_fetch_add(&fill[s], 1ull, __ATOMIC_RELAXED)] = d;
    adj[__atomic_fetch_add(&fill[d], 1ull, __ATOMIC_RELAXED)] = s;
  }
  std::vector<uint64_t> udeg(V, 0);
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < (int64_t)V; ++v) {
    auto b = adj.begin() + rawdeg[v], e = adj.begin() + rawdeg[v + 1];
    std::sort(b, e);
    udeg[v] = (uint64_t)(std::unique(b, e) - b);
  }
  offs[0] = 0;
  for (uint64_t v = 0; v < V; ++v) offs[v + 1] = offs[v] + udeg[v];
#pragma omp parallel for schedule(dynamic, 4096)
  for (int64_t v = 0; v < (int64_t)V; ++v)
    std::copy(adj.begin() + rawdeg[v], adj.begin() + rawdeg[v] + udeg[v], col + offs[v]);
  return offs[V];
}

}  // extern "C"
