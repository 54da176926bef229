// app_gol.cu — config 1: Game of Life over polymorphic cells (Table 2,
// P:1518-1522). Readings: G12 dead border (torus optional), G13
// abstract Cell + concrete Alive / Dead, G14 p = 0.5 soup. Every cell owns one
// object in each type's arena (slot = cell id), so a type change is a pointer
// swap and the type-contiguous arenas stay valid for COAL / TypePointer.
//
// Object layout (16 B): { vTable* (8 B), u32 cell, u16 counter, u16 pad }.
// counter = age (Alive) / dead_for (Dead): incremented by next(), reset to 0
// when the cell switches to this object.
#include <cstring>

#include "dispatch.cuh"

namespace vf {
namespace gol {

struct Cell {
  __device__ explicit Cell(const void* arg) : cell(arg ? *static_cast<const uint32_t*>(arg) : 0) {}
  __device__ virtual ~Cell() {}
  __device__ virtual void next(vf_gol_next_args a) = 0;
  __device__ virtual void get(vf_gol_get_args a) = 0;
  uint32_t cell;
  uint16_t counter = 0;
  uint16_t pad = 0;
};

struct Alive final : Cell {
  __device__ explicit Alive(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gol_next_args a) override {
    const uint8_t n = a.nbr_dev[cell];
    ++counter;
    a.state_out_dev[cell] = (n == 2 || n == 3) ? 1 : 0;
  }
  __device__ void get(vf_gol_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 1;
  }
};

struct Dead final : Cell {
  __device__ explicit Dead(const void* arg) : Cell(arg) {}
  __device__ void next(vf_gol_next_args a) override {
    const uint8_t n = a.nbr_dev[cell];
    ++counter;
    a.state_out_dev[cell] = n == 3 ? 1 : 0;
  }
  __device__ void get(vf_gol_get_args a) override {
    a.counter_out_dev[cell] = counter;
    a.type_out_dev[cell] = 0;
  }
};

template <int K>
struct TypeOf;
template <>
struct TypeOf<0> { using T = Dead; };
template <>
struct TypeOf<1> { using T = Alive; };

struct App {
  static constexpr int kTypes = 2;  // 0 = Dead, 1 = Alive
  static constexpr int kMethods = 2;
  static constexpr int kUnroll = 1;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 0;
  using Base = Cell;
  template <int K>
  using Type = typename TypeOf<K>::T;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_GOL_NEXT) o->next(blob_as<vf_gol_next_args>(b));
    else o->get(blob_as<vf_gol_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_GOL_NEXT) o->Type<K>::next(blob_as<vf_gol_next_args>(b));
    else o->Type<K>::get(blob_as<vf_gol_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(Alive) == 16 && sizeof(Dead) == 16, "cell layout");

__global__ void k_neighbors(uint32_t W, uint32_t H, int torus, const uint8_t* __restrict__ st,
                            uint8_t* __restrict__ nb) {
  const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= (uint64_t)W * H) return;
  nb[c] = count_live(W, H, torus, st, c);
}

__global__ void k_swap(uint64_t n, const uint8_t* __restrict__ prev, const uint8_t* __restrict__ next,
                       uint64_t* __restrict__ grid, const uint64_t* __restrict__ alive,
                       const uint64_t* __restrict__ dead) {
  const uint64_t c = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (c >= n) return;
  const uint8_t s = next[c];
  if (s != prev[c]) {
    const uint64_t p = s ? alive[c] : dead[c];
    grid[c] = p;
    reinterpret_cast<Cell*>(strip(p))->counter = 0;
  }
}

// Fused generation (vf_gol_step): neighbours -> virtual next() -> swap per cell.
struct Step {
  uint32_t W, H;
  int torus;
  const uint8_t* prev;
  const uint8_t* next;
  uint8_t* nbr;
  uint64_t* grid;
  const uint64_t* alive;
  const uint64_t* dead;
  __device__ __forceinline__ void pre(uint64_t c) const { nbr[c] = count_live(W, H, torus, prev, c); }
  __device__ __forceinline__ uint64_t ptr(uint64_t c) const { return grid[c]; }
  __device__ __forceinline__ void post(uint64_t c) const {
    const uint8_t s = next[c];
    if (s != prev[c]) {
      const uint64_t p = s ? alive[c] : dead[c];
      grid[c] = p;
      reinterpret_cast<Cell*>(strip(p))->counter = 0;
    }
  }
};

}  // namespace gol

cudaError_t gol_step(int variant, uint32_t W, uint32_t H, int torus, const uint8_t* prev, uint8_t* next, uint8_t* nbr,
                     uint64_t* grid, const uint64_t* alive, const uint64_t* dead, const DevTable& tbl,
                     cudaStream_t s) {
  vf_gol_next_args a{nbr, next};
  ArgBlob blob{};
  memcpy(blob.b, &a, sizeof a);
  const gol::Step st{W, H, torus, prev, next, nbr, grid, alive, dead};
  return launch_step<gol::App, VF_GOL_NEXT>(variant, (uint64_t)W * H, blob, tbl, st, s);
}

static const uint32_t kGolBytes[2] = {16, 16};
static const uint32_t kGolArgs[2] = {sizeof(vf_gol_next_args), sizeof(vf_gol_get_args)};

const AppOps* app_gol() {
  static const AppOps ops = make_ops<gol::App>("gol", kGolBytes, kGolArgs);
  return &ops;
}

}  // namespace vf

extern "C" vf_status vf_gol_neighbors(uint32_t W, uint32_t H, int torus, const uint8_t* state_dev,
                                      uint8_t* nbr_dev, void* stream) {
  const uint64_t n = (uint64_t)W * H;
  if (!n) return VF_OK;
  if (!state_dev || !nbr_dev) return VF_ERR_INVALID;
  vf::gol::k_neighbors<<<(unsigned)((n + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      W, H, torus, state_dev, nbr_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}

extern "C" vf_status vf_gol_swap(vf_ctx*, uint64_t ncells, const uint8_t* prev, const uint8_t* next,
                                 uint64_t* grid, const uint64_t* alive, const uint64_t* dead,
                                 void* stream) {
  if (!ncells) return VF_OK;
  if (!prev || !next || !grid || !alive || !dead) return VF_ERR_INVALID;
  vf::gol::k_swap<<<(unsigned)((ncells + 255) / 256), 256, 0, (cudaStream_t)stream>>>(
      ncells, prev, next, grid, alive, dead);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
