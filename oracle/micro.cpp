// oracle/micro.cpp — TEST INFRASTRUCTURE (see oracle.h header).
// Config 2 dispatch microbenchmark, paper §8.3: "threads scale
// with the number of objects and the compute inside the function call is a
// simple addition operation". Plain C++ dynamic dispatch: objects from plain
// `new` in index order, `objs[i]->apply()`.
#include "oracle.h"

#include <chrono>
#include <memory>
#include <vector>
#ifdef _OPENMP
#include <omp.h>
#endif

namespace {
struct MObj {
  virtual ~MObj() {}
  virtual void apply() = 0;
  int32_t val = 0;
};
template <int K>
struct MObjK final : MObj {
  void apply() override { val += K + 1; }  // reading G11: type k adds k+1
};

template <int K>
MObj* make_k(int k) {
  if constexpr (K < 32) {
    if (k == K) return new MObjK<K>();
    return make_k<K + 1>(k);
  } else {
    return nullptr;
  }
}
}  // namespace

extern "C" int oracle_max_threads(void) {
#ifdef _OPENMP
  return omp_get_max_threads();
#else
  return 1;
#endif
}

extern "C" int oracle_micro_run(uint64_t n, uint32_t T, const uint32_t* types,
                                const int32_t* init, uint32_t reps, int threads,
                                int32_t* out_vals, double* seconds) {
  if (T == 0 || T > 32) return 1;
  std::vector<MObj*> objs(n);
  for (uint64_t i = 0; i < n; ++i) {  // allocation in index order
    if (types[i] >= T) return 2;
    objs[i] = make_k<0>((int)types[i]);
    objs[i]->val = init[i];
  }
#ifdef _OPENMP
  if (threads > 0) omp_set_num_threads(threads);
#endif
  auto t0 = std::chrono::steady_clock::now();
  for (uint32_t r = 0; r < reps; ++r) {
#pragma omp parallel for schedule(static) if (threads != 1)
    for (int64_t i = 0; i < (int64_t)n; ++i) objs[i]->apply();  // the virtual call
  }
  auto t1 = std::chrono::steady_clock::now();
  if (seconds) *seconds = std::chrono::duration<double>(t1 - t0).count();
  for (uint64_t i = 0; i < n; ++i) {
    out_vals[i] = objs[i]->val;
    delete objs[i];
  }
  return 0;
}
