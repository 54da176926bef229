// dispatch.cuh — generic sm_100a kernels for the four dispatch variants,
// object construction, resolution and verification. Instantiated once per app
// inside that app's translation unit (see vf_internal.h for why).
//
// An App is a struct providing
//   static constexpr int kTypes;                  concrete types (<= 32)
//   using Base;                                   polymorphic base class
//   template <int K> using Type;                  concrete class K
//   static constexpr int kMethods;
//   template <int M> static void vcall(Base*, uint64_t i, const ArgBlob&);
//        -> the ordinary C++ virtual call of method M (vTable* load, vFunc*
//           load, indirect CALL: Fig. 1a)
//   template <int M, int K> static void dcall(Type<K>*, uint64_t i, const ArgBlob&);
//        -> the SAME method body called by qualified name (o->Type<K>::f()),
//           i.e. a direct, inlinable call: what COAL/TypePointer enable once
//           the type is known from the address alone.
//   static void construct(uint32_t t, void* mem, const void* arg);  placement new
//   static Base* make(uint32_t t, const void* arg);                 device new
#pragma once
#include <cuda_runtime.h>
#include <stdint.h>

#include <new>

#include "vf_internal.h"

namespace vf {

static constexpr uint64_t kVaMask = (1ull << VF_VA_BITS) - 1;
static constexpr uint32_t kNF = VF_NOT_FOUND;
static constexpr int kBlock = 256;

__device__ __forceinline__ uint64_t strip(uint64_t p) { return p & kVaMask; }

template <class T>
__device__ __forceinline__ T blob_as(const ArgBlob& b) {
  return *reinterpret_cast<const T*>(b.b);
}

__device__ __forceinline__ uint64_t ldg_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

__device__ __forceinline__ void prefetch_l1(uint64_t a) {
  asm volatile("prefetch.global.L1 [%0];" ::"l"(a));
}

// ---------------------------------------------------------------------------
// Resolvers: pointer value -> (type id or kNF, address to dereference).
// ---------------------------------------------------------------------------

// TypePointer (§6, Fig. 5b): line 1 `SHR Ra, Robj, #57` is one
// SHF.R.U32.HI on the high word; the strip of §6.3 is one LOP3.
// Lines 2-4 (vTable base + index, LDG vFunc*, CALL) are replaced by the warp
// grouping below: the tag selects an inlined body directly.
struct ResolveTP {
  static constexpr bool kNeedsTable = false;
  __device__ static void stage(unsigned char*, const DevTable&) {}
  __device__ __forceinline__ static uint32_t resolve(const unsigned char*, uint32_t,
                                                     uint64_t p, uint64_t& a) {
    a = strip(p);
    const uint32_t tag = (uint32_t)(p >> 32) >> (VF_VA_BITS - 32);
    return tag - 1u;  // tag 0 (untagged) -> 0xFFFFFFFF = not found -> fallback
  }
};

// COAL (§5, Algorithm 1): the virtual range table is staged into
// shared memory once per CTA and searched per lane. The segment tree of
// P:1158-1174 answers "which disjoint [start,end) contains p"; over sorted
// disjoint ranges that is exactly "the last start <= p, then p < end", which
// we do as a branch-free binary search (log2 P dependent LDS + SEL).
struct ResolveCOAL {
  static constexpr bool kNeedsTable = true;
  __device__ static void stage(unsigned char* smem, const DevTable& t) {
    uint64_t* s_start = reinterpret_cast<uint64_t*>(smem);
    uint64_t* s_end = s_start + t.P;
    uint32_t* s_type = reinterpret_cast<uint32_t*>(s_end + t.P);
    for (uint32_t j = threadIdx.x; j < t.P; j += blockDim.x) {
      const bool v = j < t.K;
      s_start[j] = v ? t.start[j] : ~0ull;
      s_end[j] = v ? t.end[j] : 0ull;
      s_type[j] = v ? t.type[j] : kNF;
    }
    __syncthreads();
  }
  __device__ __forceinline__ static uint32_t resolve(const unsigned char* smem, uint32_t P,
                                                     uint64_t p, uint64_t& a) {
    const uint64_t* s_start = reinterpret_cast<const uint64_t*>(smem);
    const uint64_t* s_end = s_start + P;
    const uint32_t* s_type = reinterpret_cast<const uint32_t*>(s_end + P);
    a = p;
    uint32_t j = 0;
    for (uint32_t step = P >> 1; step > 0; step >>= 1) {
      const uint32_t c = j + step;
      j = (s_start[c] <= p) ? c : j;
    }
    const bool hit = (s_start[j] <= p) & (p < s_end[j]);
    return hit ? s_type[j] : kNF;
  }
};

// ---------------------------------------------------------------------------
// Warp grouping + direct call (B200 design): each type present
// in the warp runs its body once, converged and inlined; no CALL, no BRX.
// The warp-uniform set of present types is walked bit by bit; each set bit
// reaches its body through a balanced tree of uniform direct branches
// (log2 kTypes levels), so absent types cost nothing.
// ---------------------------------------------------------------------------
template <class App, int M, int K>
__device__ __forceinline__ void body(uint32_t t, uint64_t a, uint64_t i, const ArgBlob& args) {
  if (t == (uint32_t)K) {
    auto* o = reinterpret_cast<typename App::template Type<K>*>(a);
    __builtin_assume(__isGlobal(o));
    App::template dcall<M, K>(o, i, args);
  }
}

template <class App, int M, int LO, int HI>
__device__ __forceinline__ void select_body(uint32_t k, uint32_t t, uint64_t a, uint64_t i,
                                            const ArgBlob& args) {
  if constexpr (HI - LO == 1) {
    body<App, M, LO>(t, a, i, args);
  } else {
    constexpr int MID = (LO + HI) / 2;
    if (k < (uint32_t)MID) select_body<App, M, LO, MID>(k, t, a, i, args);
    else select_body<App, M, MID, HI>(k, t, a, i, args);
  }
}

template <class App, int M>
__device__ __forceinline__ void group_call(uint32_t t, uint64_t a, uint64_t p, uint64_t i,
                                           const ArgBlob& args) {
  const bool ok = t < (uint32_t)App::kTypes;
  uint32_t present = __reduce_or_sync(0xffffffffu, ok ? (1u << t) : 0u);
  if constexpr (App::kTypes == 1) {
    if (present) body<App, M, 0>(t, a, i, args);
  } else {
    while (present) {  // warp-uniform loop over the types present in this warp
      const uint32_t k = __ffs(present) - 1;
      present &= present - 1;
      select_body<App, M, 0, App::kTypes>(k, t, a, i, args);
    }
  }
  // Fallback: unresolved non-null pointer -> embedded vTable*.
  const bool fb = !ok && p != 0;
  if (__any_sync(0xffffffffu, fb)) {
    if (fb) App::template vcall<M>(reinterpret_cast<typename App::Base*>(a), i, args);
  }
}

// Object-line warm-up before the serialised type groups (PF knob):
//   1 = prefetch.global.L1 (CCTL.E.PF1), 2 = a real L1-allocating load of the
//   object's first word, kept alive through `sink` (consumed once per tile).
template <int PF>
__device__ __forceinline__ void warm_line(uint64_t a, uint32_t& sink) {
  if constexpr (PF == 1) {
    prefetch_l1(a);
  } else if constexpr (PF == 2) {
    sink ^= *reinterpret_cast<const uint32_t*>(a + 8);
  }
}

// Grouped dispatch kernel (COAL / TypePointer). Persistent grid-stride over
// tiles of kBlock*U objects; every lane of every warp runs the same number of
// iterations, so the full-mask warp collectives are legal.
template <class App, int M, class R, int U, int PF>
__global__ void __launch_bounds__(kBlock) k_dispatch_grouped(const uint64_t* __restrict__ objs,
                                                             uint64_t n, ArgBlob args,
                                                             DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  const uint64_t tile = (uint64_t)kBlock * U;
  uint32_t sink = 0;
  for (uint64_t base = (uint64_t)blockIdx.x * tile; base < n; base += (uint64_t)gridDim.x * tile) {
    uint64_t p[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const uint64_t idx = base + (uint64_t)j * kBlock + threadIdx.x;
      p[j] = idx < n ? ldg_u64(objs + idx) : 0ull;
    }
    uint64_t a[U];
    uint32_t t[U];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      t[j] = p[j] ? R::resolve(smem, tbl.P, p[j], a[j]) : kNF;
      if (!p[j]) a[j] = 0;
    }
    // Issue every lane's object line before the (serialised) type groups run,
    // so each group's field loads hit L1 instead of paying a DRAM round trip
    // per type present in the warp.
    if constexpr (PF != 0) {
#pragma unroll
      for (int j = 0; j < U; ++j)
        if (t[j] < (uint32_t)App::kTypes) warm_line<PF>(a[j], sink);
    }
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const uint64_t idx = base + (uint64_t)j * kBlock + threadIdx.x;
      group_call<App, M>(t[j], a[j], p[j], idx, args);
    }
  }
  if constexpr (PF == 2) {
    // never true for a valid launch (n < 2^64-1); keeps the warm-up loads alive
    if (sink == 0x8BADF00Du && n == ~0ull) asm volatile("st.global.u32 [%0], %1;" ::"l"(objs), "r"(sink));
  }
}

// CUDA / SharedOA dispatch: the plain C++ virtual call, one object per thread,
// as the user writes it (`objs[i]->f()`).
template <class App, int M>
__global__ void __launch_bounds__(kBlock) k_dispatch_virtual(const uint64_t* __restrict__ objs,
                                                             uint64_t n, ArgBlob args) {
  const uint64_t i = (uint64_t)blockIdx.x * kBlock + threadIdx.x;
  if (i < n) {
    const uint64_t p = objs[i];
    if (p) App::template vcall<M>(reinterpret_cast<typename App::Base*>(p), i, args);
  }
}

// ---------------------------------------------------------------------------
// Construction / resolution / verification kernels (one-time or test paths).
// ---------------------------------------------------------------------------
template <class App>
__global__ void k_probe_vptrs(uint64_t* out, unsigned char* scratch, uint32_t stride) {
  const uint32_t t = threadIdx.x;
  if (t < (uint32_t)App::kTypes) {
    void* mem = scratch + (uint64_t)t * stride;
    App::construct(t, mem, nullptr);
    out[t] = *reinterpret_cast<const uint64_t*>(mem);
  }
}

template <class App>
__global__ void k_construct(const uint32_t* __restrict__ types, const uint64_t* __restrict__ ptrs,
                            const unsigned char* __restrict__ args, uint32_t arg_bytes, uint64_t n) {
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t p = ptrs[i];
    if (!p) continue;
    App::construct(types[i], reinterpret_cast<void*>(strip(p)),
                   args ? args + i * arg_bytes : nullptr);
  }
}

template <class App>
__global__ void k_new_cuda(const uint32_t* __restrict__ types, const unsigned char* __restrict__ args,
                           uint32_t arg_bytes, uint64_t n, uint64_t* __restrict__ out) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n) {
    typename App::Base* o = App::make(types[i], args ? args + i * arg_bytes : nullptr);
    out[i] = reinterpret_cast<uint64_t>(o);
  }
}

template <class App>
__global__ void k_delete_cuda(const uint64_t* __restrict__ ptrs, uint64_t n) {
  const uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x;
  if (i < n && ptrs[i]) delete reinterpret_cast<typename App::Base*>(strip(ptrs[i]));
}

// type under a variant's rule
template <class App>
__device__ __forceinline__ uint32_t resolve_rule(int variant, const unsigned char* smem,
                                                 const DevTable& tbl, uint64_t p) {
  if (!p) return kNF;
  uint64_t a;
  if (variant == VF_TYPEPTR) return ResolveTP::resolve(smem, tbl.P, p, a);
  if (variant == VF_COAL) return ResolveCOAL::resolve(smem, tbl.P, p, a);
  // CUDA / SharedOA: the embedded vTable* (Fig. 1a load A), mapped to a type id
  const uint64_t vp = *reinterpret_cast<const uint64_t*>(p);
  for (uint32_t k = 0; k < tbl.ntypes; ++k)
    if (tbl.vptr[k] == vp) return k;
  return kNF;
}

template <class App>
__global__ void k_resolve(int variant, const uint64_t* __restrict__ ptrs, uint64_t n,
                          uint32_t* __restrict__ out, DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  if (variant == VF_COAL) ResolveCOAL::stage(smem, tbl);
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x)
    out[i] = resolve_rule<App>(variant, smem, tbl, ptrs[i]);
}

// Brute-force type identity: the variant's resolved type must
// name the vTable* the constructor actually installed in the object.
template <class App>
__global__ void k_verify(int variant, const uint64_t* __restrict__ ptrs, uint64_t n,
                         unsigned long long* mism, DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  if (variant == VF_COAL) ResolveCOAL::stage(smem, tbl);
  unsigned long long bad = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * blockDim.x + threadIdx.x; i < n;
       i += (uint64_t)gridDim.x * blockDim.x) {
    const uint64_t p = ptrs[i];
    if (!p) continue;
    const uint32_t t = resolve_rule<App>(variant, smem, tbl, p);
    const uint64_t embedded = *reinterpret_cast<const uint64_t*>(strip(p));
    if (t >= tbl.ntypes || tbl.vptr[t] != embedded) ++bad;
  }
  for (int o = 16; o > 0; o >>= 1) bad += __shfl_xor_sync(0xffffffffu, bad, o);
  if ((threadIdx.x & 31) == 0 && bad) atomicAdd(mism, bad);
}

// ---------------------------------------------------------------------------
// Host-side launch helpers shared by the app modules.
// ---------------------------------------------------------------------------
inline int num_sms() {
  static int sms = 0;
  if (!sms) {
    int dev = 0;
    cudaGetDevice(&dev);
    cudaDeviceGetAttribute(&sms, cudaDevAttrMultiProcessorCount, dev);
    if (sms <= 0) sms = 148;
  }
  return sms;
}

inline size_t table_smem(const DevTable& t) { return (size_t)t.P * (8 + 8 + 4); }

inline unsigned grid_for(uint64_t n, uint64_t per_block, uint64_t cap) {
  uint64_t g = (n + per_block - 1) / per_block;
  if (g > cap) g = cap;
  if (g == 0) g = 1;
  return (unsigned)g;
}

template <class App, int M, class R, int U, int PF>
cudaError_t launch_grouped(const uint64_t* objs, uint64_t n, const ArgBlob& args,
                           const DevTable& tbl, cudaStream_t s) {
  auto kern = k_dispatch_grouped<App, M, R, U, PF>;
  const size_t sm = R::kNeedsTable ? table_smem(tbl) : 0;
  static int occ = -1;
  static size_t occ_sm = ~(size_t)0;
  if (occ < 0 || occ_sm != sm) {
    if (sm > 48 * 1024)
      cudaFuncSetAttribute(kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, kern, kBlock, sm);
    if (occ < 1) occ = 1;
    occ_sm = sm;
  }
  const unsigned grid = grid_for(n, (uint64_t)kBlock * U, (uint64_t)num_sms() * occ);
  kern<<<grid, kBlock, sm, s>>>(objs, n, args, tbl);
  note_launch();
  return cudaGetLastError();
}

template <class App, int M>
cudaError_t launch_virtual(const uint64_t* objs, uint64_t n, const ArgBlob& args, cudaStream_t s) {
  const unsigned grid = grid_for(n, kBlock, ~0u);
  k_dispatch_virtual<App, M><<<grid, kBlock, 0, s>>>(objs, n, args);
  note_launch();
  return cudaGetLastError();
}

// Benchmark / ablation knobs (vf_set_tuning): objects per thread and the L1
// prefetch of object lines before the type groups.
template <class App, int M, class R, int U>
cudaError_t launch_grouped_pf(int pf, const uint64_t* objs, uint64_t n, const ArgBlob& args,
                              const DevTable& tbl, cudaStream_t s) {
  if (pf == 0) return launch_grouped<App, M, R, U, 0>(objs, n, args, tbl, s);
  if (pf == 1) return launch_grouped<App, M, R, U, 1>(objs, n, args, tbl, s);
  return launch_grouped<App, M, R, U, 2>(objs, n, args, tbl, s);
}

template <class App, int M, class R>
cudaError_t launch_grouped_tuned(const uint64_t* objs, uint64_t n, const ArgBlob& args,
                                 const DevTable& tbl, cudaStream_t s) {
  const Tuning& tu = tuning();
  // Objects per thread trade memory-level parallelism against the number of
  // type groups walked per tile; with >= 24 live types (~20 groups per warp,
  // random order) one object per thread measured best on B200.
  const int u = tu.unroll > 0 ? tu.unroll : (tbl.active_types >= 24 ? 1 : App::kUnroll);
  const int pf = tu.prefetch < 0 ? App::kPrefetch : tu.prefetch;
  if (u >= 4) return launch_grouped_pf<App, M, R, 4>(pf, objs, n, args, tbl, s);
  if (u == 2) return launch_grouped_pf<App, M, R, 2>(pf, objs, n, args, tbl, s);
  return launch_grouped_pf<App, M, R, 1>(pf, objs, n, args, tbl, s);
}

template <class App, int M>
cudaError_t dispatch_method(int variant, const uint64_t* objs, uint64_t n, const ArgBlob& args,
                            const DevTable& tbl, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  switch (variant) {
    case VF_CUDA:
    case VF_SHAREDOA:
      return launch_virtual<App, M>(objs, n, args, s);
    case VF_COAL:
      return launch_grouped_tuned<App, M, ResolveCOAL>(objs, n, args, tbl, s);
    case VF_TYPEPTR:
      return launch_grouped_tuned<App, M, ResolveTP>(objs, n, args, tbl, s);
  }
  return cudaErrorInvalidValue;
}

template <class App, int M = 0>
cudaError_t dispatch_any(int variant, uint32_t method, const uint64_t* objs, uint64_t n,
                         const ArgBlob& args, const DevTable& tbl, cudaStream_t s) {
  if constexpr (M < App::kMethods) {
    if (method == (uint32_t)M) return dispatch_method<App, M>(variant, objs, n, args, tbl, s);
    return dispatch_any<App, M + 1>(variant, method, objs, n, args, tbl, s);
  } else {
    return cudaErrorInvalidValue;
  }
}

template <class App>
cudaError_t probe_vptrs_impl(uint64_t* out_dev, cudaStream_t s) {
  unsigned char* scratch = nullptr;
  const uint32_t stride = 256;
  cudaError_t e = cudaMallocAsync(&scratch, (size_t)stride * App::kTypes, s);
  if (e != cudaSuccess) return e;
  k_probe_vptrs<App><<<1, 32 * ((App::kTypes + 31) / 32), 0, s>>>(out_dev, scratch, stride);
  note_launch();
  e = cudaGetLastError();
  cudaFreeAsync(scratch, s);
  return e;
}

template <class App>
cudaError_t construct_impl(const uint32_t* types, const uint64_t* ptrs, const void* args,
                           uint32_t arg_bytes, uint64_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_construct<App><<<grid_for(n, 256, (uint64_t)num_sms() * 16), 256, 0, s>>>(
      types, ptrs, static_cast<const unsigned char*>(args), arg_bytes, n);
  note_launch();
  return cudaGetLastError();
}

template <class App>
cudaError_t new_cuda_impl(const uint32_t* types, const void* args, uint32_t arg_bytes, uint64_t n,
                          uint64_t* out, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_new_cuda<App><<<grid_for(n, 256, ~0u), 256, 0, s>>>(
      types, static_cast<const unsigned char*>(args), arg_bytes, n, out);
  note_launch();
  return cudaGetLastError();
}

template <class App>
cudaError_t delete_cuda_impl(const uint64_t* ptrs, uint64_t n, cudaStream_t s) {
  if (!n) return cudaSuccess;
  k_delete_cuda<App><<<grid_for(n, 256, ~0u), 256, 0, s>>>(ptrs, n);
  note_launch();
  return cudaGetLastError();
}

template <class App>
cudaError_t resolve_impl(int variant, const uint64_t* ptrs, uint64_t n, uint32_t* out,
                         const DevTable& tbl, cudaStream_t s) {
  if (!n) return cudaSuccess;
  const size_t sm = variant == VF_COAL ? table_smem(tbl) : 0;
  if (sm > 48 * 1024)
    cudaFuncSetAttribute(k_resolve<App>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  k_resolve<App><<<grid_for(n, 256, (uint64_t)num_sms() * 4), 256, sm, s>>>(variant, ptrs, n, out,
                                                                              tbl);
  note_launch();
  return cudaGetLastError();
}

template <class App>
cudaError_t verify_impl(int variant, const uint64_t* ptrs, uint64_t n, unsigned long long* mism,
                        const DevTable& tbl, cudaStream_t s) {
  if (!n) return cudaSuccess;
  const size_t sm = variant == VF_COAL ? table_smem(tbl) : 0;
  if (sm > 48 * 1024)
    cudaFuncSetAttribute(k_verify<App>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)sm);
  k_verify<App><<<grid_for(n, 256, (uint64_t)num_sms() * 4), 256, sm, s>>>(variant, ptrs, n, mism,
                                                                             tbl);
  note_launch();
  return cudaGetLastError();
}

// construct-by-type helpers for apps
template <class App, int K = 0>
__device__ __forceinline__ void construct_switch(uint32_t t, void* mem, const void* arg) {
  if constexpr (K < App::kTypes) {
    if (t == (uint32_t)K) {
      new (mem) typename App::template Type<K>(arg);
      return;
    }
    construct_switch<App, K + 1>(t, mem, arg);
  }
}

template <class App, int K = 0>
__device__ __forceinline__ typename App::Base* make_switch(uint32_t t, const void* arg) {
  if constexpr (K < App::kTypes) {
    if (t == (uint32_t)K) return new typename App::template Type<K>(arg);
    return make_switch<App, K + 1>(t, arg);
  } else {
    return nullptr;
  }
}

template <class App>
AppOps make_ops(const char* name, const uint32_t* obj_bytes, const uint32_t* margs) {
  AppOps o;
  o.name = name;
  o.ntypes = App::kTypes;
  o.obj_bytes = obj_bytes;
  o.nmethods = App::kMethods;
  o.method_args_bytes = margs;
  o.probe_vptrs = probe_vptrs_impl<App>;
  o.construct = construct_impl<App>;
  o.new_cuda = new_cuda_impl<App>;
  o.delete_cuda = delete_cuda_impl<App>;
  o.dispatch = dispatch_any<App, 0>;
  o.resolve = resolve_impl<App>;
  o.verify = verify_impl<App>;
  return o;
}

}  // namespace vf
