// oracle/stut.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 5 STUT: a spring-node structure (Table 2 "structure", P:1524-1528:
// nodes and springs, anchored / pulled nodes, springs that break; reading
// G17 fixes the constants, integrator and fracture rule the paper omits).
// Classes: abstract Element; concrete Node, AnchorNode, AnchorPullNode, Spring.
// One step, synchronously:
//   (1) virtual Spring::force() per spring, from the node positions at the
//       start of the step: d = p_b - p_a, len = sqrt(fmaf(dx,dx,dy*dy));
//       a broken spring, or one with len > break_ratio*L0 (which breaks it
//       permanently), exerts 0; else fs = (k*(len - L0))/len, F = (fs*dx, fs*dy)
//       acting on a (and -F on b).
//   (2) virtual move() per node: Node sums its incident springs' forces in
//       ascending spring id (+F at the a end, -F at the b end), adds damping
//       F = fmaf(-c, v, F), then v = fmaf(dt, F/m, v), p = fmaf(dt, v, p)
//       (semi-implicit Euler); AnchorNode stays; AnchorPullNode x = fmaf(dt, v_pull, x).
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
  float* px;  // node positions (updated in place by move())
  float* py;
  float* fx;  // per-spring force of this step
  float* fy;
  const uint32_t* inc_offs;
  const uint32_t* inc;
  float dt, c, v_pull, brk;
};

struct Element {
  virtual ~Element() {}
  virtual void force(World&) {}
  virtual void move(World&) {}
};

struct Spring final : Element {
  uint32_t id, a, b;
  float L0, k;
  uint32_t broken = 0;
  Spring(uint32_t i, uint32_t a_, uint32_t b_, float l, float k_) : id(i), a(a_), b(b_), L0(l), k(k_) {}
  void force(World& w) override {
    float f_x = 0.0f, f_y = 0.0f;
    if (!broken) {
      const float dx = w.px[b] - w.px[a];
      const float dy = w.py[b] - w.py[a];
      const float len = std::sqrt(std::fmaf(dx, dx, dy * dy));
      if (len > w.brk * L0) {
        broken = 1;
      } else {
        const float fs = (k * (len - L0)) / len;
        f_x = fs * dx;
        f_y = fs * dy;
      }
    }
    w.fx[id] = f_x;
    w.fy[id] = f_y;
  }
};

struct NodeBase : Element {
  uint32_t id;
  float vx, vy, m;
  NodeBase(uint32_t i, float a, float b, float mass) : id(i), vx(a), vy(b), m(mass) {}
};

struct Node final : NodeBase {
  using NodeBase::NodeBase;
  void move(World& w) override {
    float Fx = 0.0f, Fy = 0.0f;
    for (uint32_t e = w.inc_offs[id]; e < w.inc_offs[id + 1]; ++e) {
      const uint32_t s = w.inc[e] >> 1;
      if (w.inc[e] & 1u) {
        Fx = Fx - w.fx[s];
        Fy = Fy - w.fy[s];
      } else {
        Fx = Fx + w.fx[s];
        Fy = Fy + w.fy[s];
      }
    }
    Fx = std::fmaf(-w.c, vx, Fx);
    Fy = std::fmaf(-w.c, vy, Fy);
    vx = std::fmaf(w.dt, Fx / m, vx);
    vy = std::fmaf(w.dt, Fy / m, vy);
    w.px[id] = std::fmaf(w.dt, vx, w.px[id]);
    w.py[id] = std::fmaf(w.dt, vy, w.py[id]);
  }
};

struct AnchorNode final : NodeBase {
  using NodeBase::NodeBase;
  void move(World&) override {}
};

struct AnchorPullNode final : NodeBase {
  using NodeBase::NodeBase;
  void move(World& w) override { w.px[id] = std::fmaf(w.dt, w.v_pull, w.px[id]); }
};
}  // namespace

extern "C" int oracle_stut_run(uint32_t n, const uint32_t* types, const float* pos2, const float* vel2,
                               const float* mass, uint32_t S, const uint32_t* sa, const uint32_t* sb,
                               const float* L0, const float* k, const uint32_t* inc_offs, const uint32_t* inc,
                               uint32_t steps, float dt, float c, float v_pull, float brk, int threads,
                               float* pos_out, float* vel_out, uint8_t* broken_out, double* seconds) {
  std::vector<NodeBase*> nodes(n);
  for (uint32_t i = 0; i < n; ++i) {
    const float a = vel2[2 * i], b = vel2[2 * i + 1];
    switch (types[i]) {
      case 0: nodes[i] = new Node(i, a, b, mass[i]); break;
      case 1: nodes[i] = new AnchorNode(i, a, b, mass[i]); break;
      case 2: nodes[i] = new AnchorPullNode(i, a, b, mass[i]); break;
      default: return 1;
    }
  }
  std::vector<Spring*> springs(S);
  for (uint32_t s = 0; s < S; ++s) {
    if (sa[s] >= n || sb[s] >= n) return 2;
    springs[s] = new Spring(s, sa[s], sb[s], L0[s], k[s]);
  }
  std::vector<float> px(n), py(n), fx(S), fy(S);
  for (uint32_t i = 0; i < n; ++i) {
    px[i] = pos2[2 * i];
    py[i] = pos2[2 * i + 1];
  }
  World w{px.data(), py.data(), fx.data(), fy.data(), inc_offs, inc, dt, c, v_pull, brk};
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t t = 0; t < steps; ++t) {
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t s = 0; s < (int64_t)S; ++s) springs[s]->force(w);  // virtual call
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t i = 0; i < (int64_t)n; ++i) nodes[i]->move(w);  // virtual call
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  for (uint32_t i = 0; i < n; ++i) {
    pos_out[2 * i] = px[i];
    pos_out[2 * i + 1] = py[i];
    vel_out[2 * i] = nodes[i]->vx;
    vel_out[2 * i + 1] = nodes[i]->vy;
    delete nodes[i];
  }
  for (uint32_t s = 0; s < S; ++s) {
    broken_out[s] = (uint8_t)springs[s]->broken;
    delete springs[s];
  }
  return 0;
}
