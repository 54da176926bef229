// app_traf.cu — config 5 TRAF: Nagel-Schreckenberg traffic on rings of cells
// with traffic lights (Table 2: "streets, cars and traffic
// lights"; reading G16). Every cell and every vehicle is a polymorphic object
// under the abstract Agent base: PlainCell, LightCell, Car, Truck, Bus.
// Per step t: (1) virtual update(t) on every cell — blocked[c] = light red,
// and the cell clears its slot of the next occupancy; (2) virtual step() on
// every vehicle against the previous occupancy; integer-only, bit-exact.
//
// Layouts: PlainCell / LightCell {vptr, u32 cell, u32 phase} 16 B;
// Car / Truck / Bus {vptr, u32 id, u32 ring, u32 pos, u32 v} 24 B.
#include "dispatch.cuh"

namespace vf {
namespace traf {

__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

struct Agent {
  __device__ Agent() {}
  __device__ virtual ~Agent() {}
  __device__ virtual void update(vf_traf_cell_args a) = 0;
  __device__ virtual void step(vf_traf_step_args a) = 0;
  __device__ virtual void get(vf_traf_get_args a) = 0;
  __device__ virtual void place(vf_traf_get_args a) = 0;
};

struct CellBase : Agent {
  uint32_t cell, phase;
  __device__ explicit CellBase(const void* arg)
      : cell(arg ? static_cast<const uint32_t*>(arg)[0] : 0), phase(arg ? static_cast<const uint32_t*>(arg)[1] : 0) {}
  __device__ void step(vf_traf_step_args) override {}
  __device__ void get(vf_traf_get_args) override {}
  __device__ void place(vf_traf_get_args) override {}
};

struct PlainCell final : CellBase {
  __device__ explicit PlainCell(const void* arg) : CellBase(arg) {}
  __device__ void update(vf_traf_cell_args a) override {
    a.blocked_dev[cell] = 0;
    a.occ_next_dev[cell] = 0;
  }
};

struct LightCell final : CellBase {
  __device__ explicit LightCell(const void* arg) : CellBase(arg) {}
  __device__ void update(vf_traf_cell_args a) override {
    a.blocked_dev[cell] = ((a.t + phase) % 20u) < 8u ? 1 : 0;
    a.occ_next_dev[cell] = 0;
  }
};

template <int K>  // 0 Car, 1 Truck, 2 Bus
struct Vehicle final : Agent {
  uint32_t id, ring, pos, v;
  __device__ explicit Vehicle(const void* arg) : v(0) {
    const uint32_t* q = static_cast<const uint32_t*>(arg);
    id = q ? q[0] : 0;
    ring = q ? q[1] : 0;
    pos = q ? q[2] : 0;
  }
  __device__ void update(vf_traf_cell_args) override {}
  __device__ void step(vf_traf_step_args a) override {
    const uint32_t vm = a.vmax[K];
    uint32_t nv = v + 1 < vm ? v + 1 : vm;
    const uint64_t base = (uint64_t)ring * a.L;
    uint32_t gap = 0;
    while (gap < nv) {
      const uint32_t c = (pos + gap + 1) % a.L;
      if (a.occ_dev[base + c] | a.blocked_dev[base + c]) break;
      ++gap;
    }
    if (gap < nv) nv = gap;
    const uint64_t u = splitmix64(a.seed ^ (9ull << 56) ^ (((uint64_t)id << 24) ^ a.t));
    if ((uint32_t)(u >> 32) < a.slow_thr[K] && nv > 0) --nv;
    v = nv;
    pos = (pos + nv) % a.L;
    a.occ_next_dev[base + pos] = 1;
  }
  __device__ void get(vf_traf_get_args a) override {
    a.pos_out_dev[id - a.id_base] = pos;
    a.v_out_dev[id - a.id_base] = v;
  }
  __device__ void place(vf_traf_get_args a) override { a.occ_dev[(uint64_t)ring * a.L + pos] = 1; }
};

template <int K>
struct TypeOf;
template <>
struct TypeOf<0> { using T = PlainCell; };
template <>
struct TypeOf<1> { using T = LightCell; };
template <>
struct TypeOf<2> { using T = Vehicle<0>; };
template <>
struct TypeOf<3> { using T = Vehicle<1>; };
template <>
struct TypeOf<4> { using T = Vehicle<2>; };

struct App {
  static constexpr int kTypes = 5;
  static constexpr int kMethods = 4;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  static constexpr bool kLean = true;  // default launch configuration only (knob sweeps: micro)
  using Base = Agent;
  template <int K>
  using Type = typename TypeOf<K>::T;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_TRAF_CELL_UPDATE) o->update(blob_as<vf_traf_cell_args>(b));
    else if constexpr (M == VF_TRAF_VEH_STEP) o->step(blob_as<vf_traf_step_args>(b));
    else if constexpr (M == VF_TRAF_GET) o->get(blob_as<vf_traf_get_args>(b));
    else o->place(blob_as<vf_traf_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_TRAF_CELL_UPDATE) o->Type<K>::update(blob_as<vf_traf_cell_args>(b));
    else if constexpr (M == VF_TRAF_VEH_STEP) o->Type<K>::step(blob_as<vf_traf_step_args>(b));
    else if constexpr (M == VF_TRAF_GET) o->Type<K>::get(blob_as<vf_traf_get_args>(b));
    else o->Type<K>::place(blob_as<vf_traf_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(PlainCell) == 16 && sizeof(LightCell) == 16 && sizeof(Vehicle<0>) == 24, "layouts");

}  // namespace traf

static const uint32_t kTrafBytes[5] = {16, 16, 24, 24, 24};
static const uint32_t kTrafArgs[4] = {sizeof(vf_traf_cell_args), sizeof(vf_traf_step_args),
                                      sizeof(vf_traf_get_args), sizeof(vf_traf_get_args)};

const AppOps* app_traf() {
  static const AppOps ops = make_ops<traf::App>("traf", kTrafBytes, kTrafArgs);
  return &ops;
}

}  // namespace vf
