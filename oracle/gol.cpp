// oracle/gol.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 1: Game of Life over polymorphic cells (Table 2, P:1518-1522:
// "Game of life is a cellular automaton formulated by John Horton Conway").
// Readings: G12 dead border (torus optional), G13 classes
// Cell (abstract) / Alive / Dead, G14 p = 0.5 soup; each cell owns one object
// per concrete type so a type change is a pointer swap.
#include "oracle.h"

#include <chrono>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct Cell {
  virtual ~Cell() {}
  virtual uint8_t next(uint8_t n) = 0;  // returns the next state (1 alive)
  uint16_t counter = 0;                 // Alive: age, Dead: dead_for
};
struct Alive final : Cell {
  uint8_t next(uint8_t n) override {
    ++counter;
    return (n == 2 || n == 3) ? 1 : 0;  // survival on 2 or 3 neighbours
  }
};
struct Dead final : Cell {
  uint8_t next(uint8_t n) override {
    ++counter;
    return n == 3 ? 1 : 0;  // birth on exactly 3
  }
};
}  // namespace

extern "C" int oracle_gol_run(uint32_t W, uint32_t H, const uint8_t* init_alive,
                              uint32_t gens, int torus, int threads,
                              uint8_t* out_state, uint16_t* out_counter,
                              uint32_t* pop, double* seconds) {
  const uint64_t N = (uint64_t)W * H;
  std::vector<Alive*> alive(N);
  std::vector<Dead*> dead(N);
  std::vector<Cell*> grid(N);
  std::vector<uint8_t> state(N), nstate(N), nb(N);
  for (uint64_t c = 0; c < N; ++c) {  // allocation in index order
    alive[c] = new Alive();
    dead[c] = new Dead();
    state[c] = init_alive[c] ? 1 : 0;
    grid[c] = state[c] ? (Cell*)alive[c] : (Cell*)dead[c];
  }
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t g = 0; g < gens; ++g) {
    // (1) neighbour counts from the previous state (non-virtual)
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
              continue;  // dead border
            }
            n += state[(uint64_t)yy * W + (uint64_t)xx];
          }
        nb[(uint64_t)y * W + x] = (uint8_t)n;
      }
    // (2) one virtual call per cell, (3) pointer swap on a type change
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t c = 0; c < (int64_t)N; ++c) {
      uint8_t s = grid[c]->next(nb[c]);
      if (s != state[c]) {
        Cell* other = s ? (Cell*)alive[c] : (Cell*)dead[c];
        other->counter = 0;
        grid[c] = other;
      }
      nstate[c] = s;
    }
    state.swap(nstate);
    uint32_t p = 0;
    for (uint64_t c = 0; c < N; ++c) p += state[c];
    if (pop) pop[g] = p;
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  for (uint64_t c = 0; c < N; ++c) {
    out_state[c] = state[c];
    out_counter[c] = grid[c]->counter;
    delete alive[c];
    delete dead[c];
  }
  return 0;
}
