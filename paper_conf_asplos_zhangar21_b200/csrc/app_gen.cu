// app_gen.cu — config 5 "Generation" (Table 2: "an extension of
// gol ... more intermediate states"), read as the Generations CA B/S/C
// (reading G15): states 0 dead, 1 alive, 2..C-1 dying; neighbours count
// state-1 cells only. Classes: abstract Cell, concrete Dead / Alive / Dying.
// Each cell owns one object per concrete type (slot = cell id), so a type
// change is a pointer swap (k_gen_swap), exactly as in app_gol.cu.
//
// Object layout (16 B): { vTable* (8 B), u32 cell, u16 counter, u8 stage, u8 pad }.
#include <cstring>

#include "dispatch.cuh"

namespace vf {
namespace gen {

struct Cell {
  __device__ explicit Cell(const void* arg) : cell(arg ? *static_cast<const uint32_t*>(arg) : 0) {}
  __device__ virtual ~Cell() {}
  __device__ virtual void next(vf_gen_next_args a) = 0;
  __device__ virtual void get(vf_gen_get_args a) = 0;
  uint32_t cell;
  uint16_t counter = 0;
  uint8_t stage = 2;  // Dying only: current state 2..C-1
  uint8_t pad = 0;
};

struct Dead final : Cell {
  __device__ explicit Dead(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gen_next_args a) override {
    const uint8_t n = a.nbr_dev[cell];
    ++counter;
    a.state_out_dev[cell] = ((a.born_mask >> n) & 1u) ? 1 : 0;
  }
  __device__ void get(vf_gen_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 0;
  }
};

struct Alive final : Cell {
  __device__ explicit Alive(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gen_next_args a) override {
    const uint8_t n = a.nbr_dev[cell];
    ++counter;
    a.state_out_dev[cell] = ((a.survive_mask >> n) & 1u) ? 1 : (a.C > 2 ? 2 : 0);
  }
  __device__ void get(vf_gen_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 1;
  }
};

struct Dying final : Cell {
  __device__ explicit Dying(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gen_next_args a) override {
    ++counter;
    const uint32_t s = stage + 1u;
    if (s >= a.C) {
      a.state_out_dev[cell] = 0;
    } else {
      stage = (uint8_t)s;
      a.state_out_dev[cell] = (uint8_t)s;
    }
  }
  __device__ void get(vf_gen_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 2;
  }
};

template <int K>
struct TypeOf;
template <>
struct TypeOf<0> { using T = Dead; };
template <>
struct TypeOf<1> { using T = Alive; };
template <>
struct TypeOf<2> { using T = Dying; };

struct App {
  static constexpr int kTypes = 3;  // 0 Dead, 1 Alive, 2 Dying
  static constexpr int kMethods = 2;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  static constexpr bool kLean = true;  // default launch configuration only (knob sweeps: micro)
  using Base = Cell;
  template <int K>
  using Type = typename TypeOf<K>::T;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_GEN_NEXT) o->next(blob_as<vf_gen_next_args>(b));
    else o->get(blob_as<vf_gen_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_GEN_NEXT) o->Type<K>::next(blob_as<vf_gen_next_args>(b));
    else o->Type<K>::get(blob_as<vf_gen_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(Dead) == 16 && sizeof(Alive) == 16 && sizeof(Dying) == 16, "cell layout");

__device__ __forceinline__ int kind(uint8_t s) { return s == 0 ? 0 : (s == 1 ? 1 : 2); }

// Step (3): on a type change point the cell at its object of the new type,
// reset that object's counter, and set the Dying object's stage on entry.
__global__ void k_gen_swap(uint64_t n, const uint8_t* __restrict__ prev, const uint8_t* __restrict__ next,
                           uint64_t* __restrict__ grid, const uint64_t* __restrict__ dead,
                           const uint64_t* __restrict__ alive, const uint64_t* __restrict__ dying) {
  const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  const uint8_t s = next[c];
  const int k = kind(s);
  if (k != kind(prev[c])) {
    const uint64_t p = k == 0 ? dead[c] : k == 1 ? alive[c] : dying[c];
    grid[c] = p;
    Cell* o = reinterpret_cast<Cell*>(strip(p));
    o->counter = 0;
    if (k == 2) o->stage = s;
  }
}

// Fused generation (vf_gen_step / vf_gen_step_rows): neighbours -> virtual
// next() -> swap per cell, over the cells [off, off + n) of a row slab.
struct Step {
  uint32_t W, H;
  int torus;
  uint32_t off;  // first cell of the slab (row0 * W)
  const uint8_t* prev;
  const uint8_t* next;
  uint8_t* nbr;
  uint64_t* grid;
  const uint64_t* dead;
  const uint64_t* alive;
  const uint64_t* dying;
  __device__ __forceinline__ void pre(uint64_t i) const {
    const uint32_t c = off + (uint32_t)i;
    nbr[c] = count_live(W, H, torus, prev, c);
  }
  __device__ __forceinline__ uint64_t ptr(uint64_t i) const { return grid[off + (uint32_t)i]; }
  __device__ __forceinline__ void post(uint64_t i) const {
    const uint32_t c = off + (uint32_t)i;
    const uint8_t s = next[c];
    const int k = kind(s);
    if (k != kind(prev[c])) {
      const uint64_t p = k == 0 ? dead[c] : k == 1 ? alive[c] : dying[c];
      grid[c] = p;
      Cell* o = reinterpret_cast<Cell*>(strip(p));
      o->counter = 0;
      if (k == 2) o->stage = s;
    }
  }
};

}  // namespace gen

cudaError_t gen_step(int variant, uint32_t W, uint32_t H, int torus, uint32_t row0, uint32_t nrows,
                     const uint8_t* prev, uint8_t* next, uint8_t* nbr, uint64_t* grid, const uint64_t* dead,
                     const uint64_t* alive, const uint64_t* dying, uint32_t born, uint32_t survive, uint32_t C,
                     const DevTable& tbl, cudaStream_t s) {
  vf_gen_next_args a{nbr, next, born, survive, C};
  ArgBlob blob{};
  memcpy(blob.b, &a, sizeof a);
  const gen::Step st{W, H, torus, row0 * W, prev, next, nbr, grid, dead, alive, dying};
  return launch_step<gen::App, VF_GEN_NEXT>(variant, (uint64_t)W * nrows, blob, tbl, st, s);
}

static const uint32_t kGenBytes[3] = {16, 16, 16};
static const uint32_t kGenArgs[2] = {sizeof(vf_gen_next_args), sizeof(vf_gen_get_args)};

const AppOps* app_gen() {
  static const AppOps ops = make_ops<gen::App>("gen", kGenBytes, kGenArgs);
  return &ops;
}

}  // namespace vf

extern "C" vf_status vf_gen_swap(vf_ctx*, uint64_t ncells, const uint8_t* prev, const uint8_t* next,
                                 uint64_t* grid, const uint64_t* dead, const uint64_t* alive,
                                 const uint64_t* dying, void* stream) {
  if (!ncells) return VF_OK;
  if (!prev || !next || !grid || !dead || !alive || !dying) return VF_ERR_INVALID;
  vf::gen::k_gen_swap<<<(unsigned)((ncells + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      ncells, prev, next, grid, dead, alive, dying);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
