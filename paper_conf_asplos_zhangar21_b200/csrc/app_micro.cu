// app_micro.cu — config 2 dispatch microbenchmark (paper §8.3):
// "threads scale with the number of objects and the compute inside the
// function call is a simple addition operation". Up to 32 concrete classes
// MObjK<k> whose apply() adds k+1 (reading G11), one virtual call per object.
//
// Object layout (16 B): { vTable* (8 B), int32 val, int32 pad }.
#include "dispatch.cuh"

namespace vf {
namespace micro {

struct MObj {
  __device__ explicit MObj(const void* arg) : val(arg ? *static_cast<const int32_t*>(arg) : 0) {}
  __device__ virtual ~MObj() {}
  __device__ virtual void apply() = 0;
  __device__ virtual void get(uint64_t i, vf_micro_get_args a) = 0;
  int32_t val;
  int32_t pad = 0;
};

template <int K>
struct MObjK final : MObj {
  __device__ explicit MObjK(const void* arg) : MObj(arg) {}
  __device__ void apply() override { val += K + 1; }
  __device__ void get(uint64_t i, vf_micro_get_args a) override { a.out_dev[i] = val; }
};

struct App {
  static constexpr int kTypes = 32;
  static constexpr int kMethods = 2;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  using Base = MObj;
  template <int K>
  using Type = MObjK<K>;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_MICRO_APPLY) o->apply();
    else o->get(i, blob_as<vf_micro_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t i, const ArgBlob& b) {
    if constexpr (M == VF_MICRO_APPLY) o->Type<K>::apply();
    else o->Type<K>::get(i, blob_as<vf_micro_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};

static_assert(sizeof(MObjK<0>) == 16, "MObj layout");

}  // namespace micro

static const uint32_t kMicroBytes[32] = {16, 16, 16, 16, 16, 16, 16, 16, 16, 16, 16,
                                         16, 16, 16, 16, 16, 16, 16, 16, 16, 16, 16,
                                         16, 16, 16, 16, 16, 16, 16, 16, 16, 16};
static const uint32_t kMicroArgs[2] = {0, sizeof(vf_micro_get_args)};

const AppOps* app_micro() {
  static const AppOps ops = make_ops<micro::App>("micro", kMicroBytes, kMicroArgs);
  return &ops;
}

}  // namespace vf
