// oracle/gen.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 5 "Generation" (Table 2: "Generation is an extension of
// gol benchmark. The cells in Generation have more intermediate states"),
// read as the Generations cellular automaton B/S/C (reading G15): states
// 0 = dead, 1 = alive, 2..C-1 = dying; neighbours count state-1 cells only.
// Classes: abstract Cell, concrete Dead / Alive / Dying (4 types incl. the
// abstract base, as in Table 2). Each cell owns one object of each concrete
// type; a type change is a pointer swap (the new object's counter resets;
// entering Dying sets its stage).
#include "oracle.h"

#include <chrono>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct Rule {
  uint32_t born, survive, C;
};
struct Cell {
  virtual ~Cell() {}
  virtual uint8_t next(uint8_t n, const Rule& r) = 0;  // returns the next state
  uint16_t counter = 0;
};
struct Dead final : Cell {
  uint8_t next(uint8_t n, const Rule& r) override {
    ++counter;
    return ((r.born >> n) & 1u) ? 1 : 0;
  }
};
struct Alive final : Cell {
  uint8_t next(uint8_t n, const Rule& r) override {
    ++counter;
    if ((r.survive >> n) & 1u) return 1;
    return r.C > 2 ? 2 : 0;
  }
};
struct Dying final : Cell {
  uint8_t stage = 2;
  uint8_t next(uint8_t, const Rule& r) override {
    ++counter;
    uint32_t s = stage + 1u;
    if (s >= r.C) return 0;
    stage = (uint8_t)s;
    return (uint8_t)s;
  }
};
inline int kind(uint8_t s) { return s == 0 ? 0 : (s == 1 ? 1 : 2); }
}  // namespace

extern "C" int oracle_gen_run(uint32_t W, uint32_t H, const uint8_t* init_state, uint32_t gens,
                              uint32_t born_mask, uint32_t survive_mask, uint32_t C, int torus,
                              int threads, uint8_t* out_state, uint16_t* out_counter,
                              uint32_t* hist, double* seconds) {
  if (C < 2 || C > 255) return 1;
  const Rule r{born_mask, survive_mask, C};
  const uint64_t N = (uint64_t)W * H;
  std::vector<Dead*> dead(N);
  std::vector<Alive*> alive(N);
  std::vector<Dying*> dying(N);
  std::vector<Cell*> grid(N);
  std::vector<uint8_t> state(N), nstate(N), nb(N);
  for (uint64_t c = 0; c < N; ++c) {
    dead[c] = new Dead();
    alive[c] = new Alive();
    dying[c] = new Dying();
    uint8_t s = init_state[c];
    if (s >= C) return 2;
    state[c] = s;
    if (s >= 2) dying[c]->stage = s;
    grid[c] = s == 0 ? (Cell*)dead[c] : s == 1 ? (Cell*)alive[c] : (Cell*)dying[c];
  }
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t g = 0; g < gens; ++g) {
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t y = 0; y < (int64_t)H; ++y)
      for (uint32_t x = 0; x < W; ++x) {
        int n = 0;
        for (int dy = -1; dy <= 1; ++dy)
          for (int dx = -1; dx <= 1; ++dx) {
            if (dx == 0 && dy == 0) continue;
            int64_t yy = y + dy, xx = (int64_t)x + dx;
            if (torus) {
              yy = (yy + H) % H;
              xx = (xx + W) % W;
            } else if (yy < 0 || yy >= (int64_t)H || xx < 0 || xx >= (int64_t)W) {
              continue;
            }
            n += state[(uint64_t)yy * W + (uint64_t)xx] == 1;
          }
        nb[(uint64_t)y * W + x] = (uint8_t)n;
      }
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t c = 0; c < (int64_t)N; ++c) {
      uint8_t s = grid[c]->next(nb[c], r);  // the virtual call
      if (kind(s) != kind(state[c])) {
        Cell* other = s == 0 ? (Cell*)dead[c] : s == 1 ? (Cell*)alive[c] : (Cell*)dying[c];
        other->counter = 0;
        if (s >= 2) dying[c]->stage = s;
        grid[c] = other;
      }
      nstate[c] = s;
    }
    state.swap(nstate);
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  if (hist)
    for (uint32_t k = 0; k < C; ++k) hist[k] = 0;
  for (uint64_t c = 0; c < N; ++c) {
    out_state[c] = state[c];
    out_counter[c] = grid[c]->counter;
    if (hist) ++hist[state[c]];
    delete dead[c];
    delete alive[c];
    delete dying[c];
  }
  return 0;
}
