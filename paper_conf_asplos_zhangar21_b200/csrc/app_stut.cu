// app_stut.cu — config 5 STUT: a spring-node structure (Table 2 "structure",
// P:1524-1528; reading G17). Classes under the abstract Element: Node,
// AnchorNode, AnchorPullNode, Spring. One step = a virtual force() on every
// spring (positions at the start of the step -> per-spring force, permanent
// fracture above break_ratio * L0), then a virtual move() on every node (sum
// of its incident springs' forces in ascending spring id, damping,
// semi-implicit Euler; anchors stay, pull nodes move at v_pull).
//
// Built with -fmad=false -prec-div=true -prec-sqrt=true -ftz=false: every FMA
// is an explicit fmaf of the formula, so results equal the CPU oracle's bit
// for bit, and the fracture threshold flips on exactly the same steps.
//
// Layouts: Node / AnchorNode / AnchorPullNode {vptr, u32 id, f32 vx, vy, m}
// 24 B; Spring {vptr, u32 id, a, b, f32 L0, k, u32 broken} 32 B.
#include "dispatch.cuh"

namespace vf {
namespace stut {

struct Element {
  __device__ Element() {}
  __device__ virtual ~Element() {}
  __device__ virtual void force(const vf_stut_force_args& a) = 0;
  __device__ virtual void move(const vf_stut_move_args& a) = 0;
  __device__ virtual void get(const vf_stut_get_args& a) = 0;
};

struct NodeBase : Element {
  uint32_t id;
  float vx, vy, m;
  __device__ explicit NodeBase(const void* arg) {
    const uint32_t* q = static_cast<const uint32_t*>(arg);
    id = q ? q[0] : 0;
    vx = q ? __uint_as_float(q[1]) : 0.f;
    vy = q ? __uint_as_float(q[2]) : 0.f;
    m = q ? __uint_as_float(q[3]) : 1.f;
  }
  __device__ void force(const vf_stut_force_args&) override {}
  __device__ void get(const vf_stut_get_args& a) override {
    if (a.vel_out_dev) {
      float* o = a.vel_out_dev + 2ull * (id - a.id_base);
      o[0] = vx;
      o[1] = vy;
    }
  }
};

struct Node final : NodeBase {
  __device__ explicit Node(const void* arg) : NodeBase(arg) {}
  __device__ void move(const vf_stut_move_args& a) override {
    float Fx = 0.0f, Fy = 0.0f;
    const uint32_t e1 = __ldg(a.inc_offs_dev + id + 1);
    for (uint32_t e = __ldg(a.inc_offs_dev + id); e < e1; ++e) {
      const uint32_t code = __ldg(a.inc_dev + e);
      const float2 f = __ldg(a.F_dev + (code >> 1));
      if (code & 1u) {
        Fx = Fx - f.x;
        Fy = Fy - f.y;
      } else {
        Fx = Fx + f.x;
        Fy = Fy + f.y;
      }
    }
    Fx = fmaf(-a.c, vx, Fx);
    Fy = fmaf(-a.c, vy, Fy);
    vx = fmaf(a.dt, Fx / m, vx);
    vy = fmaf(a.dt, Fy / m, vy);
    const float2 p = a.pos_dev[id];
    a.pos_dev[id] = make_float2(fmaf(a.dt, vx, p.x), fmaf(a.dt, vy, p.y));
  }
};

struct AnchorNode final : NodeBase {
  __device__ explicit AnchorNode(const void* arg) : NodeBase(arg) {}
  __device__ void move(const vf_stut_move_args&) override {}
};

struct AnchorPullNode final : NodeBase {
  __device__ explicit AnchorPullNode(const void* arg) : NodeBase(arg) {}
  __device__ void move(const vf_stut_move_args& a) override {
    a.pos_dev[id].x = fmaf(a.dt, a.v_pull, a.pos_dev[id].x);
  }
};

struct Spring final : Element {
  uint32_t id, a, b;
  float L0, k;
  uint32_t broken;
  __device__ explicit Spring(const void* arg) : broken(0) {
    const uint32_t* q = static_cast<const uint32_t*>(arg);
    id = q ? q[0] : 0;
    a = q ? q[1] : 0;
    b = q ? q[2] : 0;
    L0 = q ? __uint_as_float(q[3]) : 1.f;
    k = q ? __uint_as_float(q[4]) : 0.f;
  }
  __device__ void force(const vf_stut_force_args& g) override {
    float fx = 0.0f, fy = 0.0f;
    if (!broken) {
      const float2 pa = __ldg(g.pos_dev + a), pb = __ldg(g.pos_dev + b);
      const float dx = pb.x - pa.x;
      const float dy = pb.y - pa.y;
      const float len = sqrtf(fmaf(dx, dx, dy * dy));
      if (len > g.break_ratio * L0) {
        broken = 1;
      } else {
        const float fs = (k * (len - L0)) / len;
        fx = fs * dx;
        fy = fs * dy;
      }
    }
    g.F_dev[id] = make_float2(fx, fy);
  }
  __device__ void move(const vf_stut_move_args&) override {}
  __device__ void get(const vf_stut_get_args& g) override {
    if (g.broken_out_dev) g.broken_out_dev[id - g.spring_base] = (uint8_t)broken;
  }
};

template <int K>
struct TypeOf;
template <>
struct TypeOf<0> { using T = Node; };
template <>
struct TypeOf<1> { using T = AnchorNode; };
template <>
struct TypeOf<2> { using T = AnchorPullNode; };
template <>
struct TypeOf<3> { using T = Spring; };

struct App {
  static constexpr int kTypes = 4;
  static constexpr int kMethods = 3;
  static constexpr int kUnroll = 2;
  static constexpr int kUnrollSorted = 2;
  static constexpr int kPrefetch = 2;
  static constexpr bool kLean = true;  // default launch configuration only (knob sweeps: micro)
  using Base = Element;
  template <int K>
  using Type = typename TypeOf<K>::T;

  template <int M>
  __device__ __forceinline__ static void vcall(Base* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_STUT_FORCE) o->force(blob_as<vf_stut_force_args>(b));
    else if constexpr (M == VF_STUT_MOVE) o->move(blob_as<vf_stut_move_args>(b));
    else o->get(blob_as<vf_stut_get_args>(b));
  }
  template <int M, int K>
  __device__ __forceinline__ static void dcall(Type<K>* o, uint64_t, const ArgBlob& b) {
    if constexpr (M == VF_STUT_FORCE) o->Type<K>::force(blob_as<vf_stut_force_args>(b));
    else if constexpr (M == VF_STUT_MOVE) o->Type<K>::move(blob_as<vf_stut_move_args>(b));
    else o->Type<K>::get(blob_as<vf_stut_get_args>(b));
  }
  __device__ static void construct(uint32_t t, void* mem, const void* arg) {
    construct_switch<App>(t, mem, arg);
  }
  __device__ static Base* make(uint32_t t, const void* arg) { return make_switch<App>(t, arg); }
};
static_assert(sizeof(Node) == 24 && sizeof(AnchorNode) == 24 && sizeof(Spring) == 32, "layouts");

}  // namespace stut

static const uint32_t kStutBytes[4] = {24, 24, 24, 32};
static const uint32_t kStutArgs[3] = {sizeof(vf_stut_force_args), sizeof(vf_stut_move_args),
                                      sizeof(vf_stut_get_args)};

const AppOps* app_stut() {
  static const AppOps ops = make_ops<stut::App>("stut", kStutBytes, kStutArgs);
  return &ops;
}

}  // namespace vf
