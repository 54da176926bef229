// oracle/collide.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 5 "collision" at 16M bodies (DynaSOAr's collision app [46]; not in
// this paper: readings G18 / G19 in DESIGN.md). Bodies Star / Planet / Dust
// (abstract Body) move under a short-range softened gravity with cutoff rc,
// found through a uniform grid of cells of side rc, and merge on contact.
// One step, synchronously from the state at its start:
//   (0) cells: every active body (mass > 0) goes to cell
//       (clamp(floor(x/rc)), clamp(floor(y/rc)), clamp(floor(z/rc))) of a G^3
//       grid; a cell lists its bodies in ascending id.
//   (1) virtual update() per active body i: over the 27 neighbour cells in
//       (z, y, x) order, bodies j != i in ascending id: d = p_j - p_i,
//       d2 = fmaf(dx,dx,fmaf(dy,dy,dz*dz)); if d2 < rc^2:
//       r2 = fmaf(dx,dx,fmaf(dy,dy,fmaf(dz,dz,eps2[type_i]))),
//       a = fmaf(d, m_j / (r2*sqrt(r2)), a)  [exactly the all-pairs N-body
//       formula]; the nearest j with d2 < rm^2 (ties: smaller id) is near[i].
//       Dust: v *= damp; v = fmaf(dt,a,v); x' = fmaf(dt,v,x).
//   (2) virtual merge() per active body i: j = near[i]; if near[j] == i
//       (mutual), the smaller id absorbs the larger: m = m_i + m_j,
//       x = fmaf(m_i, x_i, m_j*x_j) / m, v likewise (post-update values); the
//       larger id becomes inactive (mass 0, velocity 0, position kept).
// fp32, explicit fmaf only, IEEE sqrt / division, no contraction elsewhere.
#include "oracle.h"

#include <chrono>
#include <cmath>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct World {
  uint32_t N, G;
  const float* P;  // start-of-step positions+mass (N x 4)
  const float* V;  // start-of-step velocities (N x 4, w unused)
  float* Pm;       // after update (N x 4)
  float* Vm;
  int32_t* near;
  float* Po;  // after merge
  float* Vo;
  const uint32_t* cell_start;  // G^3 + 1
  const uint32_t* cell_list;   // ids, ascending within a cell
  float rc, rc2, rm2, dt, damp;
  const float* eps2;
};

inline int cell_coord(float x, float rc, uint32_t G) {
  const float f = std::floor(x / rc);
  if (!(f >= 0.0f)) return 0;  // also NaN -> 0
  if (f >= (float)G) return (int)G - 1;
  return (int)f;
}

struct Body {
  uint32_t id;
  explicit Body(uint32_t i) : id(i) {}
  virtual ~Body() {}
  virtual void update(World& w) = 0;
  virtual void merge(World& w) = 0;

 protected:
  void update_with(World& w, float eps2, bool damped) {
    const uint32_t i = id;
    const float xi = w.P[4 * i], yi = w.P[4 * i + 1], zi = w.P[4 * i + 2];
    const int cx = cell_coord(xi, w.rc, w.G), cy = cell_coord(yi, w.rc, w.G), cz = cell_coord(zi, w.rc, w.G);
    float ax = 0.0f, ay = 0.0f, az = 0.0f;
    float best = 0.0f;
    int32_t bestj = -1;
    const int G = (int)w.G;
    for (int z = cz - 1; z <= cz + 1; ++z) {
      if (z < 0 || z >= G) continue;
      for (int y = cy - 1; y <= cy + 1; ++y) {
        if (y < 0 || y >= G) continue;
        for (int x = cx - 1; x <= cx + 1; ++x) {
          if (x < 0 || x >= G) continue;
          const uint64_t c = ((uint64_t)z * G + y) * G + x;
          for (uint32_t e = w.cell_start[c]; e < w.cell_start[c + 1]; ++e) {
            const uint32_t j = w.cell_list[e];
            if (j == i) continue;
            const float dx = w.P[4 * j] - xi, dy = w.P[4 * j + 1] - yi, dz = w.P[4 * j + 2] - zi;
            const float d2 = std::fmaf(dx, dx, std::fmaf(dy, dy, dz * dz));
            if (d2 < w.rc2) {
              const float r2 = std::fmaf(dx, dx, std::fmaf(dy, dy, std::fmaf(dz, dz, eps2)));
              const float inv = 1.0f / (r2 * std::sqrt(r2));
              const float sc = w.P[4 * j + 3] * inv;
              ax = std::fmaf(dx, sc, ax);
              ay = std::fmaf(dy, sc, ay);
              az = std::fmaf(dz, sc, az);
            }
            if (d2 < w.rm2 && (bestj < 0 || d2 < best || (d2 == best && (int32_t)j < bestj))) {
              best = d2;
              bestj = (int32_t)j;
            }
          }
        }
      }
    }
    float vx = w.V[4 * i], vy = w.V[4 * i + 1], vz = w.V[4 * i + 2];
    if (damped) {
      vx = vx * w.damp;
      vy = vy * w.damp;
      vz = vz * w.damp;
    }
    vx = std::fmaf(w.dt, ax, vx);
    vy = std::fmaf(w.dt, ay, vy);
    vz = std::fmaf(w.dt, az, vz);
    w.Vm[4 * i] = vx;
    w.Vm[4 * i + 1] = vy;
    w.Vm[4 * i + 2] = vz;
    w.Vm[4 * i + 3] = 0.0f;
    w.Pm[4 * i] = std::fmaf(w.dt, vx, xi);
    w.Pm[4 * i + 1] = std::fmaf(w.dt, vy, yi);
    w.Pm[4 * i + 2] = std::fmaf(w.dt, vz, zi);
    w.Pm[4 * i + 3] = w.P[4 * i + 3];
    w.near[i] = bestj;
  }

 public:
  void merge_common(World& w) {
    const uint32_t i = id;
    const int32_t j = w.near[i];
    for (int k = 0; k < 4; ++k) {
      w.Po[4 * i + k] = w.Pm[4 * i + k];
      w.Vo[4 * i + k] = w.Vm[4 * i + k];
    }
    if (j < 0 || w.near[j] != (int32_t)i) return;
    if ((uint32_t)j > i) {  // i absorbs j
      const float mi = w.Pm[4 * i + 3], mj = w.Pm[4 * j + 3];
      const float m = mi + mj;
      for (int k = 0; k < 3; ++k) {
        w.Po[4 * i + k] = std::fmaf(mi, w.Pm[4 * i + k], mj * w.Pm[4 * j + k]) / m;
        w.Vo[4 * i + k] = std::fmaf(mi, w.Vm[4 * i + k], mj * w.Vm[4 * j + k]) / m;
      }
      w.Po[4 * i + 3] = m;
    } else {  // absorbed by j < i
      w.Po[4 * i + 3] = 0.0f;
      w.Vo[4 * i] = w.Vo[4 * i + 1] = w.Vo[4 * i + 2] = 0.0f;
    }
  }
};

struct Star final : Body {
  using Body::Body;
  void update(World& w) override { update_with(w, w.eps2[0], false); }
  void merge(World& w) override { merge_common(w); }
};
struct Planet final : Body {
  using Body::Body;
  void update(World& w) override { update_with(w, w.eps2[1], false); }
  void merge(World& w) override { merge_common(w); }
};
struct Dust final : Body {
  using Body::Body;
  void update(World& w) override { update_with(w, w.eps2[2], true); }
  void merge(World& w) override { merge_common(w); }
};
}  // namespace

extern "C" int oracle_collide_run(uint32_t N, const uint32_t* types, const float* pos4, const float* vel4,
                                  uint32_t steps, uint32_t G, float rc, float rm, float dt, const float* eps2,
                                  float damp, int threads, float* pos_out, float* vel_out, uint64_t* calls_out,
                                  double* seconds) {
  if (G == 0 || !(rc > 0.0f)) return 2;
  std::vector<Body*> bodies(N);
  for (uint32_t i = 0; i < N; ++i) {
    switch (types[i]) {
      case 0: bodies[i] = new Star(i); break;
      case 1: bodies[i] = new Planet(i); break;
      case 2: bodies[i] = new Dust(i); break;
      default: return 1;
    }
  }
  const uint64_t ncell = (uint64_t)G * G * G;
  std::vector<float> P(pos4, pos4 + 4ull * N), V(vel4, vel4 + 4ull * N), Pm(4ull * N), Vm(4ull * N),
      Po(4ull * N), Vo(4ull * N);
  std::vector<int32_t> near(N, -1);
  std::vector<uint32_t> start(ncell + 1), list(N), cell(N);
  uint64_t calls = 0;
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t t = 0; t < steps; ++t) {
    // (0) cell lists, ascending id per cell (stable counting sort)
    std::fill(start.begin(), start.end(), 0u);
    for (uint32_t i = 0; i < N; ++i) {
      if (!(P[4 * i + 3] > 0.0f)) {
        cell[i] = 0xFFFFFFFFu;
        continue;
      }
      const int cx = cell_coord(P[4 * i], rc, G), cy = cell_coord(P[4 * i + 1], rc, G),
                cz = cell_coord(P[4 * i + 2], rc, G);
      cell[i] = (uint32_t)(((uint64_t)cz * G + cy) * G + cx);
      ++start[cell[i] + 1];
    }
    for (uint64_t c = 0; c < ncell; ++c) start[c + 1] += start[c];
    {
      std::vector<uint32_t> fill(start.begin(), start.end() - 1);
      for (uint32_t i = 0; i < N; ++i)
        if (cell[i] != 0xFFFFFFFFu) list[fill[cell[i]]++] = i;
    }
    World w{N, G, P.data(), V.data(), Pm.data(), Vm.data(), near.data(), Po.data(), Vo.data(),
            start.data(), list.data(), rc, rc * rc, rm * rm, dt, damp, eps2};
    uint64_t active = 0;
    for (uint32_t i = 0; i < N; ++i) active += P[4 * i + 3] > 0.0f;
    calls += 2 * active;
    // (1) virtual update() per active body
#pragma omp parallel for schedule(dynamic, 256) if (threads != 1)
    for (int64_t i = 0; i < (int64_t)N; ++i) {
      if (P[4 * i + 3] > 0.0f) {
        bodies[i]->update(w);
      } else {
        for (int k = 0; k < 4; ++k) {
          Pm[4 * i + k] = P[4 * i + k];
          Vm[4 * i + k] = V[4 * i + k];
        }
        near[i] = -1;
      }
    }
    // (2) virtual merge() per active body
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t i = 0; i < (int64_t)N; ++i) {
      if (P[4 * i + 3] > 0.0f) {
        bodies[i]->merge(w);
      } else {
        for (int k = 0; k < 4; ++k) {
          Po[4 * i + k] = Pm[4 * i + k];
          Vo[4 * i + k] = Vm[4 * i + k];
        }
      }
    }
    P.swap(Po);
    V.swap(Vo);
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  if (calls_out) *calls_out = calls;
  for (uint64_t k = 0; k < 4ull * N; ++k) {
    pos_out[k] = P[k];
    vel_out[k] = V[k];
  }
  for (auto* b : bodies) delete b;
  return 0;
}
