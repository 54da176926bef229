// oracle/ray.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 3: ray tracing over polymorphic shapes (Table 2 RAY, P:1592-1600,
// "spheres and planes"; BASELINE adds triangles). Readings G24 / G25
// (DESIGN.md): one deterministic primary ray per pixel through the pixel
// centre, pinhole camera at the origin looking down -z, closest hit over all
// shapes with t > 1e-4 and ties broken by the smaller shape id (strict < in
// ascending id order), Lambert shading with one fixed light + 0.1 ambient.
//
// Float rules (bit-exactness with the GPU): IEEE fp32, explicit fmaf where an
// FMA is written, no contraction elsewhere (-ffp-contract=off), IEEE sqrtf and
// division. Camera constants come from the caller (host-computed fp32).
#include "oracle.h"

#include <chrono>
#include <cmath>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct V3 {
  float x, y, z;
};
inline V3 sub(V3 a, V3 b) { return {a.x - b.x, a.y - b.y, a.z - b.z}; }
inline float dot(V3 a, V3 b) { return std::fmaf(a.x, b.x, std::fmaf(a.y, b.y, a.z * b.z)); }
inline V3 cross(V3 a, V3 b) {
  return {std::fmaf(a.y, b.z, -(a.z * b.y)), std::fmaf(a.z, b.x, -(a.x * b.z)),
          std::fmaf(a.x, b.y, -(a.y * b.x))};
}
inline V3 at(V3 o, V3 d, float t) { return {std::fmaf(t, d.x, o.x), std::fmaf(t, d.y, o.y), std::fmaf(t, d.z, o.z)}; }
inline V3 scale(V3 a, float s) { return {a.x * s, a.y * s, a.z * s}; }
inline float comp(V3 a, int k) { return k == 0 ? a.x : (k == 1 ? a.y : a.z); }
const float kEps = 1e-4f;
const float kInf = INFINITY;

struct Ray {
  V3 o, d;
};

struct Shape {
  virtual ~Shape() {}
  virtual float hit(const Ray& r) const = 0;          // t of the nearest hit > eps, or +inf
  virtual V3 normal(const Ray& r, float t) const = 0;  // unit normal facing the ray
  virtual int kind() const = 0;
};

struct Plane final : Shape {  // y = h, normal +y
  float h;
  explicit Plane(const float* p) : h(p[0]) {}
  float hit(const Ray& r) const override {
    if (r.d.y == 0.0f) return kInf;
    float t = (h - r.o.y) / r.d.y;
    return t > kEps ? t : kInf;
  }
  V3 normal(const Ray& r, float) const override { return {0.0f, r.d.y < 0.0f ? 1.0f : -1.0f, 0.0f}; }
  int kind() const override { return 0; }
};

struct Sphere final : Shape {
  V3 c;
  float rad;
  explicit Sphere(const float* p) : c{p[0], p[1], p[2]}, rad(p[3]) {}
  float hit(const Ray& r) const override {
    V3 oc = sub(r.o, c);
    float b = dot(oc, r.d);
    float cc = std::fmaf(-rad, rad, dot(oc, oc));
    float disc = std::fmaf(b, b, -cc);
    if (disc < 0.0f) return kInf;
    float sq = std::sqrt(disc);
    float t = -b - sq;
    if (t > kEps) return t;
    t = -b + sq;
    return t > kEps ? t : kInf;
  }
  V3 normal(const Ray& r, float t) const override {
    V3 n = scale(sub(at(r.o, r.d, t), c), 1.0f / rad);
    return dot(n, r.d) > 0.0f ? scale(n, -1.0f) : n;
  }
  int kind() const override { return 1; }
};

struct Rect final : Shape {  // axis-aligned: coordinate `axis` == p, extents on the other two
  int axis;
  float p, a0, a1, b0, b1;
  explicit Rect(const float* q) : axis((int)q[0]), p(q[1]), a0(q[2]), a1(q[3]), b0(q[4]), b1(q[5]) {}
  float hit(const Ray& r) const override {
    const float dk = comp(r.d, axis);
    if (dk == 0.0f) return kInf;
    const float t = (p - comp(r.o, axis)) / dk;
    if (!(t > kEps)) return kInf;
    const V3 h = at(r.o, r.d, t);
    const int ia = axis == 0 ? 1 : 0, ib = axis == 2 ? 1 : 2;
    const float ha = comp(h, ia), hb = comp(h, ib);
    return (ha >= a0 && ha <= a1 && hb >= b0 && hb <= b1) ? t : kInf;
  }
  V3 normal(const Ray& r, float) const override {
    const float s = comp(r.d, axis) < 0.0f ? 1.0f : -1.0f;
    return {axis == 0 ? s : 0.0f, axis == 1 ? s : 0.0f, axis == 2 ? s : 0.0f};
  }
  int kind() const override { return 2; }
};

struct Triangle final : Shape {  // Moller-Trumbore
  V3 v0, v1, v2;
  explicit Triangle(const float* q) : v0{q[0], q[1], q[2]}, v1{q[3], q[4], q[5]}, v2{q[6], q[7], q[8]} {}
  float hit(const Ray& r) const override {
    const V3 e1 = sub(v1, v0), e2 = sub(v2, v0);
    const V3 pv = cross(r.d, e2);
    const float det = dot(e1, pv);
    if (det == 0.0f) return kInf;
    const float inv = 1.0f / det;
    const V3 tv = sub(r.o, v0);
    const float u = dot(tv, pv) * inv;
    if (u < 0.0f || u > 1.0f) return kInf;
    const V3 qv = cross(tv, e1);
    const float v = dot(r.d, qv) * inv;
    if (v < 0.0f || u + v > 1.0f) return kInf;
    const float t = dot(e2, qv) * inv;
    return t > kEps ? t : kInf;
  }
  V3 normal(const Ray& r, float) const override {
    V3 n = cross(sub(v1, v0), sub(v2, v0));
    n = scale(n, 1.0f / std::sqrt(dot(n, n)));
    return dot(n, r.d) > 0.0f ? scale(n, -1.0f) : n;
  }
  int kind() const override { return 3; }
};

Shape* make_shape(uint32_t type, const float* p) {
  switch (type) {
    case 0: return new Plane(p);
    case 1: return new Sphere(p);
    case 2: return new Rect(p);
    default: return new Triangle(p);
  }
}
}  // namespace

extern "C" int oracle_ray_render(uint32_t W, uint32_t H, uint32_t row0, uint32_t nrows, uint32_t S,
                                 const uint32_t* types, const float* params, const float* cam,
                                 const float* albedo, int threads, float* rgb, int32_t* hit_id,
                                 uint64_t* calls, double* seconds) {
  // cam: [sx, sy, lx, ly, lz] = (tan(fov/2)*aspect, tan(fov/2), unit light direction)
  std::vector<Shape*> shapes(S);
  for (uint32_t j = 0; j < S; ++j) shapes[j] = make_shape(types[j], params + 12ull * j);  // index order
  const float sx = cam[0], sy = cam[1];
  const V3 L{cam[2], cam[3], cam[4]};
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
#pragma omp parallel for schedule(dynamic, 1) if (threads != 1)
  for (int64_t yy = 0; yy < (int64_t)nrows; ++yy) {
    const uint32_t y = row0 + (uint32_t)yy;
    for (uint32_t x = 0; x < W; ++x) {
      const float u = ((float)x + 0.5f) / (float)W;
      const float v = ((float)y + 0.5f) / (float)H;
      V3 d{(2.0f * u - 1.0f) * sx, (1.0f - 2.0f * v) * sy, -1.0f};
      d = scale(d, 1.0f / std::sqrt(dot(d, d)));
      const Ray ray{{0.0f, 0.0f, 0.0f}, d};
      float best = kInf;
      int32_t id = -1;
      for (uint32_t j = 0; j < S; ++j) {
        const float t = shapes[j]->hit(ray);  // the virtual call
        if (t < best) {
          best = t;
          id = (int32_t)j;
        }
      }
      float* px = rgb + 3ull * ((uint64_t)yy * W + x);
      if (id < 0) {
        px[0] = px[1] = px[2] = 0.0f;
      } else {
        const V3 n = shapes[id]->normal(ray, best);  // virtual
        const float lam = std::fmax(0.0f, dot(n, L));
        const float* al = albedo + 3 * shapes[id]->kind();
        for (int c = 0; c < 3; ++c) px[c] = std::fmaf(al[c], lam, 0.1f);
      }
      hit_id[(uint64_t)yy * W + x] = id;
    }
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  if (calls) *calls = (uint64_t)nrows * W * S;
  for (Shape* s : shapes) delete s;
  return 0;
}
