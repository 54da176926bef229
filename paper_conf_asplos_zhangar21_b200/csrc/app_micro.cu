// app_micro.cu — config 2 dispatch microbenchmark (paper §8.3):
// "threads scale with the number of objects and the compute inside the
// function call is a simple addition operation". Up to 32 concrete classes
// MObjK<k> whose apply() adds k+1 (reading G11), one virtual call per object.
//
// Object layout (16 B): { vTable* (8 B), int32 val, u32 tag }. tag = K is the
// embedded type field Concord switches on (VF_CONCORD); the other variants
// never read it.
#include "dispatch.cuh"

namespace vf {
namespace micro {

struct MObj {
  __device__ explicit MObj(const void* arg) : val(arg ? *static_cast<const int32_t*>(arg) : 0) {}
  __device__ virtual ~MObj() {}
  __device__ virtual void apply() = 0;
  __device__ virtual void get(uint64_t i, vf_micro_get_args a) = 0;
  int32_t val;
  uint32_t tag = 0;
};

template <int K>
struct MObjK final : MObj {
  __device__ explicit MObjK(const void* arg) : MObj(arg) { tag = K; }
  __device__ void apply() override { val += K + 1; }
  __device__ void get(uint64_t i, vf_micro_get_args a) override { a.out_dev[i] = val; }
};

struct App {
  static constexpr int kTypes = 32;
  static constexpr int kTagOffset = 12;  // MObj::tag (Concord)
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

// BRANCH ceiling (vf_micro_branch): type from registers, switch, no objects.
__device__ __forceinline__ uint64_t splitmix64(uint64_t x) {
  uint64_t z = x + 0x9E3779B97F4A7C15ull;
  z = (z ^ (z >> 30)) * 0xBF58476D1CE4E5B9ull;
  z = (z ^ (z >> 27)) * 0x94D049BB133111EBull;
  return z ^ (z >> 31);
}

#define VF_BCASE(k) \
  case k:           \
    v += k + 1;     \
    break;
__global__ void __launch_bounds__(kBlock) k_branch(uint64_t n, uint32_t T, int order, uint64_t seed, uint32_t kk,
                                                   int32_t* __restrict__ vals) {
  const uint64_t i = (uint64_t)blockIdx.x * kBlock + threadIdx.x;
  if (i >= n) return;
  uint32_t t;
  if (order == 0) t = (uint32_t)__umul64hi(splitmix64((seed ^ (1ull << 56)) ^ i), (uint64_t)T);
  else if (order == 1) t = (uint32_t)(i * T / n);  // i*T < 2^63 for n < 2^58
  else t = (uint32_t)((i & 31u) % kk);
  int32_t v = vals[i];
  switch (t) {
    VF_BCASE(0) VF_BCASE(1) VF_BCASE(2) VF_BCASE(3) VF_BCASE(4) VF_BCASE(5) VF_BCASE(6) VF_BCASE(7)
    VF_BCASE(8) VF_BCASE(9) VF_BCASE(10) VF_BCASE(11) VF_BCASE(12) VF_BCASE(13) VF_BCASE(14) VF_BCASE(15)
    VF_BCASE(16) VF_BCASE(17) VF_BCASE(18) VF_BCASE(19) VF_BCASE(20) VF_BCASE(21) VF_BCASE(22) VF_BCASE(23)
    VF_BCASE(24) VF_BCASE(25) VF_BCASE(26) VF_BCASE(27) VF_BCASE(28) VF_BCASE(29) VF_BCASE(30) VF_BCASE(31)
    default: break;
  }
  vals[i] = v;
}
#undef VF_BCASE

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

extern "C" vf_status vf_micro_branch(uint64_t n, uint32_t T, int order, uint64_t seed, uint32_t k, int32_t* vals_dev,
                                    void* stream) {
  if (!n) return VF_OK;
  if (!vals_dev || T < 1 || T > 32 || order < 0 || order > 2 || (order == 2 && (k < 1 || k > 32)))
    return VF_ERR_INVALID;
  vf::micro::k_branch<<<(unsigned)((n + vf::kBlock - 1) / vf::kBlock), vf::kBlock, 0, (cudaStream_t)stream>>>(
      n, T, order, seed, k, vals_dev);
  vf::note_launch();
  return cudaGetLastError() == cudaSuccess ? VF_OK : VF_ERR_CUDA;
}
