// oracle/nbody.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 5 all-pairs N-body over polymorphic bodies (BASELINE north_star
// "collision/N-body"; the app is from DynaSOAr [46], not this paper: reading
// G18). Classes: abstract Body, concrete Star / Planet / Dust with per-type
// softening eps2[type]; Dust also has a velocity damping factor.
// Per step, synchronously from the positions at the start of the step:
//   body i (virtual update()): a_i = sum over j != i in ascending j of
//     m_j (x_j - x_i) / (r^2 + eps2_i)^(3/2)
//   with r2 = fmaf(dx,dx, fmaf(dy,dy, fmaf(dz,dz, eps2))), inv = 1/(r2*sqrt(r2)),
//   s = m_j*inv, a += fmaf(d, s, a); then (Dust: v *= damp) v = fmaf(dt, a, v),
//   x' = fmaf(dt, v, x) (semi-implicit Euler).
// fp32, explicit fmaf only, IEEE sqrt / division, no contraction elsewhere.
#include "oracle.h"

#include <chrono>
#include <cmath>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct State {
  uint32_t N;
  const float* pin;  // N x 4 (x, y, z, m) at the start of the step
  float* pout;       // N x 4
  float dt;
  const float* eps2;  // per type
  float damp;         // Dust velocity factor per step
};

struct Body {
  uint32_t idx;
  float vx, vy, vz;
  Body(uint32_t i, float a, float b, float c) : idx(i), vx(a), vy(b), vz(c) {}
  virtual ~Body() {}
  virtual void update(const State& s) = 0;

 protected:
  void accel(const State& s, float eps2, float& ax, float& ay, float& az) const {
    const float xi = s.pin[4 * idx], yi = s.pin[4 * idx + 1], zi = s.pin[4 * idx + 2];
    ax = ay = az = 0.0f;
    for (uint32_t j = 0; j < s.N; ++j) {
      if (j == idx) continue;
      const float dx = s.pin[4 * j] - xi, dy = s.pin[4 * j + 1] - yi, dz = s.pin[4 * j + 2] - zi;
      const float r2 = std::fmaf(dx, dx, std::fmaf(dy, dy, std::fmaf(dz, dz, eps2)));
      const float inv = 1.0f / (r2 * std::sqrt(r2));
      const float sc = s.pin[4 * j + 3] * inv;
      ax = std::fmaf(dx, sc, ax);
      ay = std::fmaf(dy, sc, ay);
      az = std::fmaf(dz, sc, az);
    }
  }
  void drift(const State& s, float ax, float ay, float az) {
    vx = std::fmaf(s.dt, ax, vx);
    vy = std::fmaf(s.dt, ay, vy);
    vz = std::fmaf(s.dt, az, vz);
    s.pout[4 * idx] = std::fmaf(s.dt, vx, s.pin[4 * idx]);
    s.pout[4 * idx + 1] = std::fmaf(s.dt, vy, s.pin[4 * idx + 1]);
    s.pout[4 * idx + 2] = std::fmaf(s.dt, vz, s.pin[4 * idx + 2]);
    s.pout[4 * idx + 3] = s.pin[4 * idx + 3];
  }
};

struct Star final : Body {
  using Body::Body;
  void update(const State& s) override {
    float ax, ay, az;
    accel(s, s.eps2[0], ax, ay, az);
    drift(s, ax, ay, az);
  }
};
struct Planet final : Body {
  using Body::Body;
  void update(const State& s) override {
    float ax, ay, az;
    accel(s, s.eps2[1], ax, ay, az);
    drift(s, ax, ay, az);
  }
};
struct Dust final : Body {
  using Body::Body;
  void update(const State& s) override {
    float ax, ay, az;
    accel(s, s.eps2[2], ax, ay, az);
    vx *= s.damp;
    vy *= s.damp;
    vz *= s.damp;
    drift(s, ax, ay, az);
  }
};
}  // namespace

extern "C" int oracle_nbody_run(uint32_t N, const uint32_t* types, const float* pos4, const float* vel3,
                                uint32_t steps, float dt, const float* eps2, float damp, int threads,
                                float* pos_out, float* vel_out, double* seconds) {
  std::vector<Body*> bodies(N);
  for (uint32_t i = 0; i < N; ++i) {
    const float a = vel3[3 * i], b = vel3[3 * i + 1], c = vel3[3 * i + 2];
    switch (types[i]) {
      case 0: bodies[i] = new Star(i, a, b, c); break;
      case 1: bodies[i] = new Planet(i, a, b, c); break;
      case 2: bodies[i] = new Dust(i, a, b, c); break;
      default: return 1;
    }
  }
  std::vector<float> p(pos4, pos4 + 4ull * N), q(4ull * N);
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t t = 0; t < steps; ++t) {
    State s{N, p.data(), q.data(), dt, eps2, damp};
#pragma omp parallel for schedule(dynamic, 64) if (threads != 1)
    for (int64_t i = 0; i < (int64_t)N; ++i) bodies[i]->update(s);  // the virtual call
    p.swap(q);
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  for (uint32_t i = 0; i < N; ++i) {
    for (int k = 0; k < 4; ++k) pos_out[4 * i + k] = p[4 * i + k];
    vel_out[3 * i] = bodies[i]->vx;
    vel_out[3 * i + 1] = bodies[i]->vy;
    vel_out[3 * i + 2] = bodies[i]->vz;
    delete bodies[i];
  }
  return 0;
}
