// oracle/traf.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 5 TRAF: "A Nagel-Schreckenberg model traffic simulation to model
// streets, cars and traffic lights" (Table 2). Reading G16
// (DESIGN.md): R independent single-lane rings of L cells; every cell is an
// object (PlainCell / LightCell), every vehicle an object (Car / Truck / Bus)
// under the abstract Agent base (6 types incl. the abstract one, as in
// Table 2). Per step t, synchronously from the previous state:
//   (1) cell->update(t): blocked[c] = Light ? ((t + phase) mod 20 < 8) : 0
//   (2) vehicle->step(t): v = min(v+1, vmax); gap = free cells ahead (stop
//       before an occupied or blocked cell, scanning at most v cells);
//       v = min(v, gap); with probability p_slow (integer Bernoulli on
//       draw(seed, 9, (id << 24) ^ t)) v = max(v-1, 0); pos = (pos+v) mod L.
//   (3) occupancy rebuilt from the new positions.
// Car vmax 5 p 0.2, Truck vmax 3 p 0.1, Bus vmax 4 p 0.3 (thresholds given by
// the caller as integers < 2^32).
#include "oracle.h"

#include <chrono>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
inline uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

struct World {
  uint32_t L;
  const uint8_t* occ;      // previous occupancy, R*L
  const uint8_t* blocked;  // this step's blocked cells, R*L
  uint8_t* occ_next;
  uint32_t t;
  uint64_t seed;
  const uint32_t* slow_thr;  // per vehicle type (Car, Truck, Bus)
  const uint32_t* vmax;
};

struct Agent {
  virtual ~Agent() {}
  virtual void update(uint8_t* blocked, uint32_t t) = 0;  // cells
  virtual void step(const World& w) = 0;                   // vehicles
};

struct PlainCell final : Agent {
  uint32_t cell;
  explicit PlainCell(uint32_t c) : cell(c) {}
  void update(uint8_t* blocked, uint32_t) override { blocked[cell] = 0; }
  void step(const World&) override {}
};

struct LightCell final : Agent {
  uint32_t cell, phase;
  LightCell(uint32_t c, uint32_t ph) : cell(c), phase(ph) {}
  void update(uint8_t* blocked, uint32_t t) override { blocked[cell] = ((t + phase) % 20u) < 8u ? 1 : 0; }
  void step(const World&) override {}
};

template <int K>  // 0 Car, 1 Truck, 2 Bus
struct Vehicle final : Agent {
  uint32_t id, ring, pos, v;
  Vehicle(uint32_t i, uint32_t r, uint32_t p) : id(i), ring(r), pos(p), v(0) {}
  void update(uint8_t*, uint32_t) override {}
  void step(const World& w) override {
    const uint32_t vm = w.vmax[K];
    uint32_t nv = v + 1 < vm ? v + 1 : vm;
    const uint64_t base = (uint64_t)ring * w.L;
    uint32_t gap = 0;
    while (gap < nv) {
      const uint32_t c = (pos + gap + 1) % w.L;
      if (w.occ[base + c] || w.blocked[base + c]) break;
      ++gap;
    }
    if (gap < nv) nv = gap;
    const uint64_t u = splitmix64(w.seed ^ (9ull << 56) ^ (((uint64_t)id << 24) ^ w.t));
    if ((uint32_t)(u >> 32) < w.slow_thr[K] && nv > 0) --nv;
    v = nv;
    pos = (pos + nv) % w.L;
    w.occ_next[base + pos] = 1;
  }
};
}  // namespace

extern "C" int oracle_traf_run(uint32_t R, uint32_t L, uint32_t nveh, const uint32_t* veh_ring,
                               const uint32_t* veh_pos, const uint32_t* veh_type, const uint8_t* light,
                               const uint32_t* phase, uint32_t steps, uint64_t seed, const uint32_t* vmax,
                               const uint32_t* slow_thr, int threads, uint32_t* pos_out, uint32_t* v_out,
                               double* seconds) {
  const uint64_t N = (uint64_t)R * L;
  std::vector<Agent*> cells(N), vehs(nveh);
  for (uint64_t c = 0; c < N; ++c)
    cells[c] = light[c] ? (Agent*)new LightCell((uint32_t)c, phase[c]) : (Agent*)new PlainCell((uint32_t)c);
  std::vector<uint8_t> occ(N, 0), occ_next(N), blocked(N);
  for (uint32_t i = 0; i < nveh; ++i) {
    if (veh_ring[i] >= R || veh_pos[i] >= L || veh_type[i] > 2) return 1;
    switch (veh_type[i]) {
      case 0: vehs[i] = new Vehicle<0>(i, veh_ring[i], veh_pos[i]); break;
      case 1: vehs[i] = new Vehicle<1>(i, veh_ring[i], veh_pos[i]); break;
      default: vehs[i] = new Vehicle<2>(i, veh_ring[i], veh_pos[i]); break;
    }
    uint8_t& o = occ[(uint64_t)veh_ring[i] * L + veh_pos[i]];
    if (o) return 2;  // two vehicles in one cell
    o = 1;
  }
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t t = 0; t < steps; ++t) {
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t c = 0; c < (int64_t)N; ++c) cells[c]->update(blocked.data(), t);  // virtual
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t c = 0; c < (int64_t)N; ++c) occ_next[c] = 0;
    World w{L, occ.data(), blocked.data(), occ_next.data(), t, seed, slow_thr, vmax};
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t i = 0; i < (int64_t)nveh; ++i) vehs[i]->step(w);  // virtual
    occ.swap(occ_next);
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  for (uint32_t i = 0; i < nveh; ++i) {
    switch (veh_type[i]) {
      case 0: { auto* q = static_cast<Vehicle<0>*>(vehs[i]); pos_out[i] = q->pos; v_out[i] = q->v; } break;
      case 1: { auto* q = static_cast<Vehicle<1>*>(vehs[i]); pos_out[i] = q->pos; v_out[i] = q->v; } break;
      default: { auto* q = static_cast<Vehicle<2>*>(vehs[i]); pos_out[i] = q->pos; v_out[i] = q->v; } break;
    }
    delete vehs[i];
  }
  for (Agent* a : cells) delete a;
  return 0;
}
