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

#include <mutex>
#include <new>
#include <type_traits>
#include <utility>

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

// Minimum resident CTAs per SM the dispatch kernels are compiled for
// (__launch_bounds__ min blocks; caps registers). Apps whose bodies keep many
// values in flight set kMinBlocks so the whole grid stays resident.
template <class A, class = void>
struct MinBlocks {
  static constexpr int value = 1;
};
template <class A>
struct MinBlocks<A, std::void_t<decltype(A::kMinBlocks)>> {
  static constexpr int value = A::kMinBlocks;
};

// CTA size of the grid-sorted list kernel (k_dispatch_list). Apps whose heavy
// grid is only a few CTAs per SM (N-body: 65,536 bodies = 256 CTAs of 256 on
// 148 SMs, so 108 SMs run two and 40 run one) set a smaller block so the CTAs
// spread evenly; the register cap stays that of kBlock x kMinBlocks.
template <class A, class = void>
struct ListBlock {
  static constexpr int value = kBlock;
};
template <class A>
struct ListBlock<A, std::void_t<decltype(A::kListBlock)>> {
  static constexpr int value = A::kListBlock;
};

__device__ __forceinline__ uint64_t ldg_u64(const uint64_t* p) {
  uint64_t v;
  asm volatile("ld.global.nc.L1::no_allocate.u64 %0, [%1];" : "=l"(v) : "l"(p));
  return v;
}

// Methods whose bodies are long and of varying length (App::kHeavyMask bit M).
template <class A, class = void>
struct HeavyMaskOf {
  static constexpr uint32_t value = 0;
};
template <class A>
struct HeavyMaskOf<A, std::void_t<decltype(A::kHeavyMask)>> {
  static constexpr uint32_t value = A::kHeavyMask;
};

__host__ __device__ constexpr size_t table_smem_dev(uint32_t P) { return (size_t)P * (8 + 8 + 4); }

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
  __device__ __forceinline__ static uint32_t resolve(const unsigned char*, const DevTable&, uint64_t p, uint64_t& a,
                                                     uint32_t&) {
    a = strip(p);
    const uint32_t tag = (uint32_t)(p >> 32) >> (VF_VA_BITS - 32);
    return tag - 1u;  // tag 0 (untagged) -> 0xFFFFFFFF = not found -> fallback
  }
};

// COAL (§5, Algorithm 1): the segment tree of P:1158-1174 answers
// "which disjoint [start,end) contains p"; over sorted disjoint ranges that is
// exactly "the last start <= p, then p < end".
//  * K <= kTableInline rows (every app here with its VA windows: K = #types):
//    the table rides in the kernel parameters (constant bank) and each lane
//    tests the K ranges directly against constant operands — no shared-memory
//    staging, no CTA barrier, no dependent load;
//  * larger tables (config 2 at T = 32, fragmented K): staged into shared
//    memory once per CTA and searched per lane branch-free (log2 P dependent
//    LDS + SEL, then the end check).
struct ResolveCOAL {
  static constexpr bool kNeedsTable = true;
  __device__ static void stage(unsigned char* smem, const DevTable& t) {
    if (t.inl) return;  // searched in the parameter bank (CTA-uniform)
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
  // Always the full search (measured on B200 faster than first testing the
  // lane's previous range: with mixed types the test mostly misses and splits
  // the warp). `hint` is unused.
  __device__ __forceinline__ static uint32_t resolve(const unsigned char* smem, const DevTable& tbl, uint64_t p,
                                                     uint64_t& a, uint32_t& hint) {
    a = strip(p);  // a TypePointer-tagged pointer is searched (and dereferenced) by its address
    p = a;
    (void)hint;
    if (tbl.inl) {
      // p in [start, end) <=> (p - start) < (end - start), unsigned: one
      // 64-bit subtract and one 64-bit compare per row
      uint32_t t = kNF;
#pragma unroll
      for (uint32_t j = 0; j < kTableInline; ++j) {
        if (j >= tbl.K) break;  // uniform
        t = (p - tbl.in_start[j] < tbl.in_len[j]) ? tbl.in_type[j] : t;
      }
      return t;
    }
    const uint32_t P = tbl.P;
    const uint64_t* s_start = reinterpret_cast<const uint64_t*>(smem);
    const uint64_t* s_end = s_start + P;
    const uint32_t* s_type = reinterpret_cast<const uint32_t*>(s_end + P);
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

// Fallback ("use COAL or the traditional CUDA vFunc lookup as a
// backup"): a non-null pointer the resolver could not place (COAL miss, tag 0)
// is typed by its embedded vTable*, matched against the app's per-type vTable*
// table, and then joins the same grouped direct call. No CALL instruction is
// emitted anywhere in the grouped kernels, so they are not subject to the
// call ABI (which caps a calling kernel at 32 registers on sm_100a).
template <class App>
__device__ __forceinline__ uint32_t type_from_vptr(uint64_t a, const DevTable& tbl) {
  const uint64_t vp = *reinterpret_cast<const uint64_t*>(a);
  uint32_t t = kNF;
#pragma unroll 1
  for (uint32_t k = 0; k < (uint32_t)App::kTypes; ++k)
    if (tbl.vptr[k] == vp) t = k;
  return t;
}

template <class App, int M>
__device__ __forceinline__ void group_call(uint32_t t, uint64_t a, uint64_t p, uint64_t i,
                                           const ArgBlob& args, const DevTable& tbl) {
  const bool fb = t >= (uint32_t)App::kTypes && p != 0;
  if (__any_sync(0xffffffffu, fb)) {
    if (fb) t = type_from_vptr<App>(a, tbl);
  }
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
__global__ void __launch_bounds__(kBlock, MinBlocks<App>::value) k_dispatch_grouped(const uint64_t* __restrict__ objs,
                                                             uint64_t n, ArgBlob args,
                                                             DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  const uint64_t tile = (uint64_t)kBlock * U;
  uint32_t sink = 0;
  uint32_t hint = 0;  // COAL: last range hit by this lane
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
      t[j] = p[j] ? R::resolve(smem, tbl, p[j], a[j], hint) : kNF;
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
      group_call<App, M>(t[j], a[j], p[j], idx, args, tbl);
    }
  }
  if constexpr (PF == 2) {
    // never true for a valid launch (n < 2^64-1); keeps the warm-up loads alive
    if (sink == 0x8BADF00Du && n == ~0ull) asm volatile("st.global.u32 [%0], %1;" ::"l"(objs), "r"(sink));
  }
}

// ---------------------------------------------------------------------------
// TMA-pipelined grouped dispatch (tuning key "pipeline" = 1; measured slower
// than the type-sorted kernel below, which is the default).
//
// The pointer array is a pure stream: one elected thread per CTA moves each
// tile of kBlock*U pointers global -> shared with cp.async.bulk (TMA, 1-D)
// into an S-stage ring completed on mbarriers, so pointer latency never sits
// on a warp's critical path. The warps run one tile ahead on the objects:
// while tile k's type groups execute, tile k+1's pointers are already resolved
// and its object lines are in flight (warm loads), i.e. one DRAM round trip of
// objects overlaps every group walk.
// ---------------------------------------------------------------------------
__device__ __forceinline__ uint32_t smem_u32(const void* p) {
  return (uint32_t)__cvta_generic_to_shared(p);
}
__device__ __forceinline__ void mbar_init(uint64_t* bar, uint32_t count) {
  asm volatile("mbarrier.init.shared::cta.b64 [%0], %1;" ::"r"(smem_u32(bar)), "r"(count) : "memory");
}
__device__ __forceinline__ void mbar_expect_tx(uint64_t* bar, uint32_t bytes) {
  asm volatile("mbarrier.arrive.expect_tx.shared::cta.b64 _, [%0], %1;" ::"r"(smem_u32(bar)), "r"(bytes)
               : "memory");
}
__device__ __forceinline__ void mbar_wait(uint64_t* bar, uint32_t parity) {
  uint32_t done;
  do {
    asm volatile(
        "{\n .reg .pred p;\n mbarrier.try_wait.parity.shared::cta.b64 p, [%1], %2;\n"
        " selp.u32 %0, 1, 0, p;\n}\n"
        : "=r"(done)
        : "r"(smem_u32(bar)), "r"(parity)
        : "memory");
  } while (!done);
}
__device__ __forceinline__ void tma_load_1d(void* dst, const void* src, uint32_t bytes, uint64_t* bar) {
  asm volatile(
      "cp.async.bulk.shared::cluster.global.mbarrier::complete_tx::bytes [%0], [%1], %2, [%3];" ::"r"(
          smem_u32(dst)),
      "l"(src), "r"(bytes), "r"(smem_u32(bar))
      : "memory");
}

__host__ __device__ constexpr size_t align16(size_t x) { return (x + 15) & ~(size_t)15; }

template <int U, int S>
struct PipeSmem {
  static constexpr int kWarps = kBlock / 32;
  static constexpr int kTile = 32 * U;  // objects per warp tile
  static constexpr size_t kRing = (size_t)kWarps * S * kTile * sizeof(uint64_t);
  static constexpr size_t kBars = (size_t)kWarps * S * sizeof(uint64_t);
  static size_t bytes(size_t table_bytes) { return align16(table_bytes) + kRing + kBars; }
};

// Resolve a tile's pointers and start its object lines. The PF=2 warm-up
// values are returned in w[] and folded into `sink` only when the tile becomes
// current, so the wait for them overlaps the previous tile's group walk.
template <class App, int M, class R, int U, int PF>
__device__ __forceinline__ void resolve_tile(const unsigned char* smem, const DevTable& tbl, const uint64_t (&p)[U],
                                             uint64_t (&a)[U], uint32_t (&t)[U], uint32_t (&w)[U],
                                             uint32_t& hint) {
#pragma unroll
  for (int j = 0; j < U; ++j) {
    t[j] = p[j] ? R::resolve(smem, tbl, p[j], a[j], hint) : kNF;
    if (!p[j]) a[j] = 0;
    w[j] = 0;
  }
  if constexpr (PF == 1) {
#pragma unroll
    for (int j = 0; j < U; ++j)
      if (t[j] < (uint32_t)App::kTypes) prefetch_l1(a[j]);
  } else if constexpr (PF == 2) {
#pragma unroll
    for (int j = 0; j < U; ++j)
      if (t[j] < (uint32_t)App::kTypes) w[j] = *reinterpret_cast<const uint32_t*>(a[j] + 8);
  }
}

template <class App, int M, class R, int U, int PF, int S>
__global__ void __launch_bounds__(kBlock, 4) k_dispatch_pipe(const uint64_t* __restrict__ objs,
                                                          uint64_t n, ArgBlob args, DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  using L = PipeSmem<U, S>;
  constexpr int WT = L::kTile;
  const int warp = threadIdx.x >> 5, lane = threadIdx.x & 31;
  const size_t tbytes = R::kNeedsTable ? align16(table_smem_dev(tbl.P)) : 0;
  uint64_t* ring = reinterpret_cast<uint64_t*>(smem + tbytes) + (size_t)warp * S * WT;
  uint64_t* bars = reinterpret_cast<uint64_t*>(smem + tbytes + L::kRing) + warp * S;
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);

  // each warp streams its own sequence of warp tiles: no CTA-wide barrier, so
  // a warp with many type groups never stalls the others
  const uint64_t full = n / WT;
  const uint64_t gw = (uint64_t)blockIdx.x * L::kWarps + warp;
  const uint64_t nw = (uint64_t)gridDim.x * L::kWarps;
  // warp tile k of this warp is tile gw + k*nw; it exists iff that is < full
  // (a multiply instead of a 64-bit division: no CALL into the u64 divide)
  auto has = [&](uint64_t k) { return gw + k * nw < full; };
  auto tile_base = [&](uint64_t k) { return (gw + k * nw) * WT; };

  if (lane == 0) {
    for (int s = 0; s < S; ++s) mbar_init(&bars[s], 1);
    asm volatile("fence.mbarrier_init.release.cluster;" ::: "memory");
    for (int s = 0; s < S && has((uint64_t)s); ++s) {
      mbar_expect_tx(&bars[s], WT * sizeof(uint64_t));
      tma_load_1d(ring + (size_t)s * WT, objs + tile_base(s), WT * sizeof(uint64_t), &bars[s]);
    }
  }
  __syncwarp();

  uint32_t sink = 0;
  uint32_t hint = 0;  // COAL: last range hit by this lane
  uint64_t pc[U], ac[U];
  uint32_t tc[U], wc[U];
  // fetch warp tile k's pointers from the ring, release the stage, resolve + warm
  auto fetch = [&](uint64_t k, uint64_t (&p)[U], uint64_t (&a)[U], uint32_t (&t)[U], uint32_t (&w)[U]) {
    const int s = (int)(k % S);
    mbar_wait(&bars[s], (uint32_t)((k / S) & 1));
#pragma unroll
    for (int j = 0; j < U; ++j) p[j] = ring[(size_t)s * WT + j * 32 + lane];
    __syncwarp();  // the whole warp holds its pointers: the stage can be refilled
    if (lane == 0 && has(k + S)) {
      asm volatile("fence.proxy.async.shared::cta;" ::: "memory");
      mbar_expect_tx(&bars[s], WT * sizeof(uint64_t));
      tma_load_1d(ring + (size_t)s * WT, objs + tile_base(k + S), WT * sizeof(uint64_t), &bars[s]);
    }
    resolve_tile<App, M, R, U, PF>(smem, tbl, p, a, t, w, hint);
  };

  if (has(0)) fetch(0, pc, ac, tc, wc);
  for (uint64_t k = 0; has(k); ++k) {
#pragma unroll
    for (int j = 0; j < U; ++j) sink ^= wc[j];
    uint64_t pn[U], an[U];
    uint32_t tn[U], wn[U];
    if (has(k + 1)) fetch(k + 1, pn, an, tn, wn);
    const uint64_t base = tile_base(k);
#pragma unroll
    for (int j = 0; j < U; ++j) group_call<App, M>(tc[j], ac[j], pc[j], base + j * 32 + lane, args, tbl);
#pragma unroll
    for (int j = 0; j < U; ++j) {
      pc[j] = pn[j];
      ac[j] = an[j];
      tc[j] = tn[j];
      wc[j] = wn[j];
    }
  }
  // ragged tail (< one warp tile): the last warp of the grid, plain loads
  if (gw == nw - 1 && full * WT < n) {
    const uint64_t base = full * WT;
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const uint64_t idx = base + (uint64_t)j * 32 + lane;
      pc[j] = idx < n ? ldg_u64(objs + idx) : 0ull;
    }
    resolve_tile<App, M, R, U, PF>(smem, tbl, pc, ac, tc, wc, hint);
#pragma unroll
    for (int j = 0; j < U; ++j) {
      sink ^= wc[j];
      group_call<App, M>(tc[j], ac[j], pc[j], base + j * 32 + lane, args, tbl);
    }
  }
  if constexpr (PF == 2) {
    if (sink == 0x8BADF00Du && n == ~0ull) asm volatile("st.global.u32 [%0], %1;" ::"l"(objs), "r"(sink));
  }
}

// ---------------------------------------------------------------------------
// Type-regrouped dispatch (default for COAL / TypePointer with > 1 type).
//
// Warp grouping alone still runs one serialised group per type present in a
// warp (≈T groups of 32/T lanes in random order: the SIMD under-utilisation
// the paper identifies as the residual cost). Because the type is
// known from the pointer alone, a CTA can regroup its tile BEFORE touching
// any object: resolve kBlock*U pointers, counting-sort them by type in shared
// memory (warp match_any + one smem atomic per type per warp; stable within a
// warp so same-type objects stay in arena order), then let every warp walk 32
// consecutive entries of the sorted tile. A warp then sees ~1 type, all 32
// lanes active, touching consecutive slots of one arena (coalesced). Calls on
// distinct objects are independent (reading G8), so the reordering is exact.
// ---------------------------------------------------------------------------
template <int U>
struct SortSmem {
  static constexpr int kTile = kBlock * U;
  static constexpr size_t kA = (size_t)kTile * sizeof(uint64_t);   // sorted addresses
  static constexpr size_t kI = (size_t)kTile * sizeof(uint32_t);   // sorted tile-local index
  static constexpr size_t kT = (size_t)kTile * sizeof(uint8_t);    // sorted type
  static constexpr size_t kH = 132 * sizeof(uint32_t);             // hist[32] + offs[33] (+pad) | hist[2][32] (SB 2)
  static size_t bytes(size_t table_bytes) { return align16(table_bytes) + kA + kI + align16(kT) + kH; }
};

// SB = barriers per tile: 4 (rank, scan by one warp, scatter, calls) or, for
// light methods, 2: the rank atomics go into one of two histograms
// (alternating per tile) BEFORE the CTA-wide mixed test, whose barrier then
// also publishes the histogram; every warp scans the 32 counts itself in
// registers; the other histogram is cleared for the next tile.
template <class App, int M, class R, int U, int PF, int SB = 4>
__global__ void __launch_bounds__(kBlock, MinBlocks<App>::value) k_dispatch_sorted(const uint64_t* __restrict__ objs,
                                                            uint64_t n, ArgBlob args, DevTable tbl) {
  static_assert(App::kTypes <= 32, "one warp scans the histogram");
  static_assert(SB == 4 || (SB == 2 && ((HeavyMaskOf<App>::value >> M) & 1u) == 0), "SB 2: light methods");
  extern __shared__ __align__(16) unsigned char smem[];
  using L = SortSmem<U>;
  constexpr int TILE = L::kTile;
  const size_t tbytes = R::kNeedsTable ? align16(table_smem_dev(tbl.P)) : 0;
  uint64_t* s_a = reinterpret_cast<uint64_t*>(smem + tbytes);
  uint32_t* s_i = reinterpret_cast<uint32_t*>(smem + tbytes + L::kA);
  uint8_t* s_t = reinterpret_cast<uint8_t*>(smem + tbytes + L::kA + L::kI);
  uint32_t* s_hist = reinterpret_cast<uint32_t*>(smem + tbytes + L::kA + L::kI + align16(L::kT));
  uint32_t* s_offs = s_hist + 32;  // 33 entries: exclusive offsets + total
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  if (threadIdx.x < 64) s_hist[threadIdx.x] = 0;  // (SB 2 uses s_hist[0..63] as two histograms)
  __syncthreads();
  const int lane = threadIdx.x & 31;
  const uint32_t lt_mask = (1u << lane) - 1u;
  uint32_t sink = 0;
  uint32_t hint = 0;  // COAL: last range hit by this lane
  uint32_t hb = 0;    // SB 2: this tile's histogram

  // Light methods keep the NEXT tile's pointers in flight (registers) while
  // this tile is resolved, sorted and called: the pointer stream never waits
  // for the tile's barriers. PF = 3 (deep): pointers TWO tiles ahead and the
  // next tile already resolved with its object lines warmed (L1-allocating
  // loads) before this tile's sort and calls, so one tile of object traffic is
  // always in flight behind the current tile's work.
  constexpr bool kAhead = ((HeavyMaskOf<App>::value >> M) & 1u) == 0;
  constexpr bool kDeep = kAhead && PF == 3;
  const uint64_t stride = (uint64_t)gridDim.x * TILE;
  auto load_ptrs = [&](uint64_t b, uint64_t (&q)[U]) {
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const uint64_t idx = b + (uint64_t)j * kBlock + threadIdx.x;
      q[j] = idx < n ? ldg_u64(objs + idx) : 0ull;
    }
  };
  // pointers -> (type, address) incl. the vTable* fallback; warm the object lines
  auto resolve_warm = [&](const uint64_t (&q)[U], uint64_t (&aa)[U], uint32_t (&tt)[U], uint32_t (&ww)[U]) {
#pragma unroll
    for (int j = 0; j < U; ++j) {
      tt[j] = q[j] ? R::resolve(smem, tbl, q[j], aa[j], hint) : kNF;
      if (!q[j]) aa[j] = 0;
      const bool fb = tt[j] >= (uint32_t)App::kTypes && q[j] != 0;
      if (__any_sync(0xffffffffu, fb)) {
        if (fb) tt[j] = type_from_vptr<App>(aa[j], tbl);
      }
      ww[j] = 0;
      if constexpr (PF >= 2) {
        if (tt[j] < (uint32_t)App::kTypes) ww[j] = *reinterpret_cast<const uint32_t*>(aa[j] + 8);
      }
    }
  };
  uint64_t pn[U];
  uint64_t an[U];
  uint32_t tn[U], wn[U];
  if constexpr (kDeep) {
    uint64_t p0[U];
    load_ptrs((uint64_t)blockIdx.x * TILE, p0);
    load_ptrs((uint64_t)blockIdx.x * TILE + stride, pn);
    resolve_warm(p0, an, tn, wn);
  } else if constexpr (kAhead) {
    load_ptrs((uint64_t)blockIdx.x * TILE, pn);
  }
  for (uint64_t base = (uint64_t)blockIdx.x * TILE; base < n; base += stride) {
    // A: pointers -> (type, address); warm the object lines
    uint64_t p[U], a[U];
    uint32_t t[U], w[U], rank[U];
    if constexpr (kDeep) {
#pragma unroll
      for (int j = 0; j < U; ++j) {
        a[j] = an[j];
        t[j] = tn[j];
        w[j] = wn[j];
        p[j] = pn[j];  // tile k+1
      }
      load_ptrs(base + 2 * stride, pn);  // tile k+2
      resolve_warm(p, an, tn, wn);       // tile k+1: resolved, lines in flight
    } else {
      if constexpr (kAhead) {
#pragma unroll
        for (int j = 0; j < U; ++j) p[j] = pn[j];
        load_ptrs(base + stride, pn);
      } else {
        load_ptrs(base, p);
      }
      resolve_warm(p, a, t, w);
    }
    // Tiles whose warps are already type-uniform (sorted input, run interiors)
    // skip the sort: one barrier instead of four. Both cases reach the SAME
    // call site below (one inlined copy of each body per j: heavy bodies are
    // not duplicated into the instruction cache).
    bool mixed = false;
#pragma unroll
    for (int j = 0; j < U; ++j) {
      const uint32_t pres = __reduce_or_sync(0xffffffffu, t[j] < (uint32_t)App::kTypes ? (1u << t[j]) : 0u);
      mixed |= (pres & (pres - 1)) != 0;
    }
    if constexpr (SB == 2) {
      // the other histogram belongs to the previous tile: its atomics ended
      // before that tile's first barrier, its reads (C) before its second (or
      // never, for a type-uniform tile) — clear it for the next tile, whose
      // atomics start after this tile's first barrier
      if (threadIdx.x < 32) s_hist[(hb ^ 1u) * 32 + threadIdx.x] = 0;
      // B (before the CTA-wide test): rank within type into this tile's histogram
      uint32_t* hist = s_hist + hb * 32;
#pragma unroll
      for (int j = 0; j < U; ++j) {
        const bool ok = t[j] < (uint32_t)App::kTypes;
        const uint32_t key = ok ? t[j] : 0xFFFFu;
        const uint32_t peers = __match_any_sync(0xffffffffu, key);
        const int leader = __ffs(peers) - 1;
        uint32_t b = 0;
        if (ok && lane == leader) b = atomicAdd(&hist[t[j]], (uint32_t)__popc(peers));
        b = __shfl_sync(0xffffffffu, b, leader);
        rank[j] = b + __popc(peers & lt_mask);
      }
    }
    const bool sorted = __syncthreads_or(mixed) != 0;  // CTA-uniform
    if constexpr (((HeavyMaskOf<App>::value >> M) & 1u) == 0) {
      // light bodies: a separate call site for type-uniform tiles (no selects
      // on the sorted path, measured faster for config 2)
      if (!sorted) {
#pragma unroll
        for (int j = 0; j < U; ++j) {
          sink ^= w[j];
          group_call<App, M>(t[j], a[j], 0ull, base + (uint64_t)j * kBlock + threadIdx.x, args, tbl);
        }
        hb ^= 1u;
        continue;
      }
    }
    uint32_t total2 = 0;
    if constexpr (SB == 2) {
      // C: every warp scans the 32 counts in registers; D: scatter
      const uint32_t h = s_hist[hb * 32 + lane];
      uint32_t x = h;
#pragma unroll
      for (int o = 1; o < 32; o <<= 1) {
        const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
        if (lane >= o) x += y;
      }
      const uint32_t ex = x - h;
      total2 = __shfl_sync(0xffffffffu, x, 31);
#pragma unroll
      for (int j = 0; j < U; ++j) {
        const bool ok = t[j] < (uint32_t)App::kTypes;
        const uint32_t off = __shfl_sync(0xffffffffu, ex, ok ? t[j] : 0u);
        if (ok) {
          const uint32_t pos = off + rank[j];
          s_a[pos] = a[j];
          s_i[pos] = (uint32_t)(j * kBlock + threadIdx.x);
          s_t[pos] = (uint8_t)t[j];
        }
      }
      __syncthreads();
      hb ^= 1u;
    } else if (sorted) {
      // B: rank within type (warp-aggregated smem atomics)
#pragma unroll
      for (int j = 0; j < U; ++j) {
        const bool ok = t[j] < (uint32_t)App::kTypes;
        const uint32_t key = ok ? t[j] : 0xFFFFu;
        const uint32_t peers = __match_any_sync(0xffffffffu, key);
        const int leader = __ffs(peers) - 1;
        uint32_t b = 0;
        if (ok && lane == leader) b = atomicAdd(&s_hist[t[j]], (uint32_t)__popc(peers));
        b = __shfl_sync(0xffffffffu, b, leader);
        rank[j] = b + __popc(peers & lt_mask);
      }
      __syncthreads();
      // C: exclusive scan of the histogram (one warp), reset it for the next tile
      if (threadIdx.x < 32) {
        const uint32_t h = s_hist[lane];
        uint32_t x = h;
#pragma unroll
        for (int o = 1; o < 32; o <<= 1) {
          const uint32_t y = __shfl_up_sync(0xffffffffu, x, o);
          if (lane >= o) x += y;
        }
        s_offs[lane] = x - h;
        if (lane == 31) s_offs[32] = x;
        s_hist[lane] = 0;
      }
      __syncthreads();
      // D: scatter into the sorted tile
#pragma unroll
      for (int j = 0; j < U; ++j) {
        if (t[j] < (uint32_t)App::kTypes) {
          const uint32_t pos = s_offs[t[j]] + rank[j];
          s_a[pos] = a[j];
          s_i[pos] = (uint32_t)(j * kBlock + threadIdx.x);
          s_t[pos] = (uint8_t)t[j];
        }
      }
      __syncthreads();
    }
    // E: each warp walks 32 consecutive (sorted) entries per j
    const uint32_t total = SB == 2 ? total2 : (sorted ? s_offs[32] : 0u);
#pragma unroll
    for (int j = 0; j < U; ++j) sink ^= w[j];
#pragma unroll
    for (int j = 0; j < U; ++j) {
      uint64_t ae, ie;
      uint32_t te;
      if (sorted) {
        const uint32_t e = (uint32_t)(j * kBlock) + threadIdx.x;
        const bool v = e < total;
        ae = v ? s_a[e] : 0ull;
        te = v ? (uint32_t)s_t[e] : kNF;
        ie = v ? base + s_i[e] : 0ull;
      } else {
        ae = a[j];
        te = t[j];
        ie = base + (uint64_t)j * kBlock + threadIdx.x;
      }
      group_call<App, M>(te, ae, 0ull, ie, args, tbl);
    }
    // (the next tile's __syncthreads_or orders these reads before its scatter)
  }
  if constexpr (PF >= 2) {
    if (sink == 0x8BADF00Du && n == ~0ull) asm volatile("st.global.u32 [%0], %1;" ::"l"(objs), "r"(sink));
  }
}

// ---------------------------------------------------------------------------
// Comparison points of the paper (§7, §8.3, Table 1
// row C): Concord's embedded type tag + switch, and the paper-faithful
// COAL / TypePointer that still CALL the looked-up vFunc* indirectly.
// ---------------------------------------------------------------------------

// Apps with an embedded type tag (Concord) define kTagOffset (byte offset of a
// u32 type id inside every object); others get -1 (VF_ERR_UNSUPPORTED).
template <class A, class = void>
struct TagOffset {
  static constexpr int value = -1;
};
template <class A>
struct TagOffset<A, std::void_t<decltype(A::kTagOffset)>> {
  static constexpr int value = A::kTagOffset;
};

// Concord [6]: "a type field is embedded in each object ... the
// compiler inserts a switch statement, which reads the embedded type tag, then
// jumps to the appropriate function body". One object per thread, a plain
// C++ switch (compiled to a jump table / compare tree), no warp grouping.
#define VF_CASE(k)                                                                     \
  case k:                                                                              \
    if constexpr (k < App::kTypes)                                                     \
      App::template dcall<M, k>(reinterpret_cast<typename App::template Type<k>*>(a), i, args); \
    break;
template <class App, int M>
__device__ __forceinline__ void concord_switch(uint32_t t, uint64_t a, uint64_t i, const ArgBlob& args) {
  static_assert(App::kTypes <= 32, "switch covers 32 cases");
  switch (t) {
    VF_CASE(0) VF_CASE(1) VF_CASE(2) VF_CASE(3) VF_CASE(4) VF_CASE(5) VF_CASE(6) VF_CASE(7)
    VF_CASE(8) VF_CASE(9) VF_CASE(10) VF_CASE(11) VF_CASE(12) VF_CASE(13) VF_CASE(14) VF_CASE(15)
    VF_CASE(16) VF_CASE(17) VF_CASE(18) VF_CASE(19) VF_CASE(20) VF_CASE(21) VF_CASE(22) VF_CASE(23)
    VF_CASE(24) VF_CASE(25) VF_CASE(26) VF_CASE(27) VF_CASE(28) VF_CASE(29) VF_CASE(30) VF_CASE(31)
    default: break;
  }
}
#undef VF_CASE

template <class App, int M>
__global__ void __launch_bounds__(kBlock) k_dispatch_concord(const uint64_t* __restrict__ objs, uint64_t n,
                                                              ArgBlob args) {
  const uint64_t i = (uint64_t)blockIdx.x * kBlock + threadIdx.x;
  if (i >= n) return;
  const uint64_t p = ldg_u64(objs + i);
  if (!p) return;
  const uint64_t a = strip(p);
  const uint32_t t = *reinterpret_cast<const uint32_t*>(a + TagOffset<App>::value);  // the embedded tag
  concord_switch<App, M>(t, a, i, args);
}

// Paper-faithful COAL / TypePointer (vf_set_tuning("call", 1)): after the type
// is resolved from the pointer, the vFunc* is fetched from a per-CTA function
// table (Fig. 5b lines 2-3, staged in shared memory) and CALLed indirectly
// (line 4: "CALL R5"), one object per thread, no grouping.
template <class App, int M, int K>
__device__ __noinline__ void thunk(uint64_t a, uint64_t i, const ArgBlob* args) {
  App::template dcall<M, K>(reinterpret_cast<typename App::template Type<K>*>(a), i, *args);
}
using ThunkFn = void (*)(uint64_t, uint64_t, const ArgBlob*);
template <class App, int M, int K = 0>
__device__ __forceinline__ void fill_thunks(ThunkFn* tab) {
  if constexpr (K < App::kTypes) {
    tab[K] = &thunk<App, M, K>;
    fill_thunks<App, M, K + 1>(tab);
  }
}

template <class App, int M, class R>
__global__ void __launch_bounds__(kBlock, MinBlocks<App>::value) k_dispatch_indirect(const uint64_t* __restrict__ objs, uint64_t n,
                                                               ArgBlob args, DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ ThunkFn s_fn[App::kTypes];
  __shared__ ArgBlob s_args;
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  if (threadIdx.x == 0) {
    fill_thunks<App, M>(s_fn);
    s_args = args;
  }
  __syncthreads();
  uint32_t hint = 0;
  for (uint64_t i = (uint64_t)blockIdx.x * kBlock + threadIdx.x; i < n; i += (uint64_t)gridDim.x * kBlock) {
    const uint64_t p = ldg_u64(objs + i);
    if (!p) continue;
    uint64_t a;
    const uint32_t t = R::resolve(smem, tbl, p, a, hint);
    if (t < (uint32_t)App::kTypes) {
      const ThunkFn f = s_fn[t];  // vFunc* = table[type]
      f(a, i, &s_args);           // indirect CALL
    } else {
      App::template vcall<M>(reinterpret_cast<typename App::Base*>(a), i, args);  // fallback
    }
  }
}

// CUDA / SharedOA dispatch: the plain C++ virtual call, one object per thread,
// as the user writes it (`objs[i]->f()`).
template <class App, int M>
__global__ void __launch_bounds__(kBlock, MinBlocks<App>::value) k_dispatch_virtual(const uint64_t* __restrict__ objs,
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
  uint32_t hint = 0;
  if (variant == VF_TYPEPTR) return ResolveTP::resolve(smem, tbl, p, a, hint);
  if (variant == VF_COAL) return ResolveCOAL::resolve(smem, tbl, p, a, hint);
  if (variant == VF_CONCORD) {
    if constexpr (TagOffset<App>::value >= 0) {
      const uint32_t t = *reinterpret_cast<const uint32_t*>(strip(p) + TagOffset<App>::value);
      return t < tbl.ntypes ? t : kNF;
    }
    return kNF;
  }
  // CUDA / SharedOA: the embedded vTable* (Fig. 1a load A), mapped to a type id
  const uint64_t vp = *reinterpret_cast<const uint64_t*>(strip(p));
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
// Launch-configuration caches are per device (a second ctx on another GPU
// gets its own attribute set-up and SM count) and guarded by a mutex (two
// ctxs may launch from two host threads).
constexpr int kMaxDevices = 64;
inline int current_device() {
  int dev = 0;
  cudaGetDevice(&dev);
  return dev & (kMaxDevices - 1);
}
inline std::mutex& launch_cache_mutex() {
  static std::mutex m;
  return m;
}

inline int num_sms() {
  static int sms[kMaxDevices] = {0};
  const int dev = current_device();
  if (!sms[dev]) {
    std::lock_guard<std::mutex> lk(launch_cache_mutex());
    int v = 0;
    int d = 0;
    cudaGetDevice(&d);
    cudaDeviceGetAttribute(&v, cudaDevAttrMultiProcessorCount, d);
    sms[dev] = v > 0 ? v : 148;
  }
  return sms[dev];
}

// Resident CTAs per SM of kernel `Kern` at `smem` dynamic shared memory on the
// current device (sets the opt-in dynamic smem attribute above 48 KB once per
// device and size).
template <auto Kern>
inline int occupancy(size_t smem, int block = kBlock) {
  struct Slot {
    int occ = -1;
    size_t sm = ~(size_t)0;
  };
  static Slot slots[kMaxDevices];
  Slot& sl = slots[current_device()];
  std::lock_guard<std::mutex> lk(launch_cache_mutex());
  if (sl.occ < 0 || sl.sm != smem) {
    if (smem > 32 * 1024) cudaFuncSetAttribute(Kern, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)smem);
    int occ = 0;
    cudaOccupancyMaxActiveBlocksPerMultiprocessor(&occ, Kern, block, smem);
    sl.occ = occ < 1 ? 1 : occ;
    sl.sm = smem;
  }
  return sl.occ;
}

inline size_t table_smem(const DevTable& t) { return table_smem_dev(t.P); }

inline unsigned grid_for(uint64_t n, uint64_t per_block, uint64_t cap) {
  uint64_t g = (n + per_block - 1) / per_block;
  if (g > cap) g = cap;
  if (g == 0) g = 1;
  return (unsigned)g;
}

// Persistent grid (occupancy x SMs, CTAs loop over tiles) or one tile per CTA.
// Apps may mark methods whose bodies are long and of varying length
// (kHeavyMask bit M): there a persistent CTA would wait at every tile's
// barrier for its slowest warp, while one tile per CTA lets finished warps
// leave and other CTAs take their place. Tuning key "persistent" overrides.
template <class A, class = void>
struct HeavyMask {
  static constexpr uint32_t value = 0;
};
template <class A>
struct HeavyMask<A, std::void_t<decltype(A::kHeavyMask)>> {
  static constexpr uint32_t value = A::kHeavyMask;
};
template <class App, int M>
inline uint64_t grid_cap(int occ) {
  const int p = tuning().persistent;
  const bool pers = p >= 0 ? p != 0 : ((HeavyMask<App>::value >> M) & 1u) == 0;
  return pers ? (uint64_t)num_sms() * occ : ~0ull;
}

template <class App, int M, class R, int U, int PF>
cudaError_t launch_grouped(const uint64_t* objs, uint64_t n, const ArgBlob& args,
                           const DevTable& tbl, cudaStream_t s) {
  constexpr auto kern = k_dispatch_grouped<App, M, R, U, PF>;
  const size_t sm = R::kNeedsTable ? table_smem(tbl) : 0;
  const int occ = occupancy<kern>(sm);
  const unsigned grid = grid_for(n, (uint64_t)kBlock * U, grid_cap<App, M>(occ));
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
template <class App, int M, class R, int U, int PF, int S>
cudaError_t launch_pipe(const uint64_t* objs, uint64_t n, const ArgBlob& args, const DevTable& tbl,
                        cudaStream_t s) {
  constexpr auto kern = k_dispatch_pipe<App, M, R, U, PF, S>;
  const size_t sm = PipeSmem<U, S>::bytes(R::kNeedsTable ? table_smem(tbl) : 0);
  const int occ = occupancy<kern>(sm);
  const uint64_t tiles = n / ((uint64_t)kBlock * U);  // CTA-sized tiles of warp tiles
  const unsigned grid = grid_for(tiles, 1, (uint64_t)num_sms() * occ);
  kern<<<grid, kBlock, sm, s>>>(objs, n, args, tbl);
  note_launch();
  return cudaGetLastError();
}

template <class App, int M, class R, int U, int PF, int SB = 4>
cudaError_t launch_sorted(const uint64_t* objs, uint64_t n, const ArgBlob& args, const DevTable& tbl,
                          cudaStream_t s) {
  constexpr auto kern = k_dispatch_sorted<App, M, R, U, PF, SB>;
  const size_t sm = SortSmem<U>::bytes(R::kNeedsTable ? table_smem(tbl) : 0);
  const int occ = occupancy<kern>(sm);
  const unsigned grid = grid_for(n, (uint64_t)kBlock * U, grid_cap<App, M>(occ));
  kern<<<grid, kBlock, sm, s>>>(objs, n, args, tbl);
  note_launch();
  return cudaGetLastError();
}

template <class App, int M, class R, int U>
cudaError_t launch_grouped_pf(int pf, const uint64_t* objs, uint64_t n, const ArgBlob& args,
                              const DevTable& tbl, cudaStream_t s) {
  if constexpr (App::kTypes > 1) {
    if (tuning().regroup != 0) {
      if constexpr (((HeavyMaskOf<App>::value >> M) & 1u) == 0) {
        if (tuning().regroup == 2 && pf == 2) return launch_sorted<App, M, R, U, 2, 2>(objs, n, args, tbl, s);
      }
      if (pf == 3) return launch_sorted<App, M, R, U, 3>(objs, n, args, tbl, s);
      if (pf == 2) return launch_sorted<App, M, R, U, 2>(objs, n, args, tbl, s);
      return launch_sorted<App, M, R, U, 0>(objs, n, args, tbl, s);
    }
  }
  // TMA needs a 16-byte aligned source; the pipeline is the default when it applies
  if (pf == 3) pf = 2;  // the deep pipeline is the sorted kernel's
  if (tuning().pipeline != 0 && (reinterpret_cast<uintptr_t>(objs) & 15) == 0) {
    if (pf == 0) return launch_pipe<App, M, R, U, 0, 4>(objs, n, args, tbl, s);
    if (pf == 1) return launch_pipe<App, M, R, U, 1, 4>(objs, n, args, tbl, s);
    return launch_pipe<App, M, R, U, 2, 4>(objs, n, args, tbl, s);
  }
  if (pf == 0) return launch_grouped<App, M, R, U, 0>(objs, n, args, tbl, s);
  if (pf == 1) return launch_grouped<App, M, R, U, 1>(objs, n, args, tbl, s);
  return launch_grouped<App, M, R, U, 2>(objs, n, args, tbl, s);
}

// Apps with long bodies may set kLean: only the app's default grouped
// configuration is instantiated (sorted tiles or, with regroup = 0, the plain
// grouped kernel, each at kUnrollSorted / kUnroll and kPrefetch); the
// unroll / prefetch / pipeline knobs do not apply. Keeps compile time bounded.
template <class A, class = void>
struct Lean {
  static constexpr bool value = false;
};
template <class A>
struct Lean<A, std::void_t<decltype(A::kLean)>> {
  static constexpr bool value = A::kLean;
};

constexpr uint32_t kGsChunk = 4096;  // entries per histogram chunk of the grid-level type sort
// Apps whose heavy methods default to the grid-level type sort (App::kGridSort)
template <class A, class = void>
struct GridSortDefault {
  static constexpr bool value = false;
};
template <class A>
struct GridSortDefault<A, std::void_t<decltype(A::kGridSort)>> {
  static constexpr bool value = A::kGridSort;
};
template <class App, int M, class R>
cudaError_t launch_gsorted(const uint64_t* objs, uint64_t n, const ArgBlob& args, const DevTable& tbl,
                           cudaStream_t s);

template <class App, int M, class R>
cudaError_t launch_grouped_tuned(const uint64_t* objs, uint64_t n, const ArgBlob& args,
                                 const DevTable& tbl, cudaStream_t s) {
  const Tuning& tu = tuning();
  if constexpr (App::kTypes > 1 && ((HeavyMaskOf<App>::value >> M) & 1u) != 0) {
    // heavy methods: the whole dispatch list sorted by type (tuning "gsort")
    const bool gs = tu.gsort >= 0 ? tu.gsort != 0 : GridSortDefault<App>::value;
    if (gs && tu.regroup != 0 && n >= 2 * kGsChunk) return launch_gsorted<App, M, R>(objs, n, args, tbl, s);
  }
  if constexpr (Lean<App>::value) {
    if constexpr (((HeavyMaskOf<App>::value >> M) & 1u) != 0 && App::kUnrollSorted > 1) {
      // a small dispatch of a long body (graph: the top-down expansion of the
      // BFS source's chunks, a few thousand entries) is a grid of a few CTAs:
      // one entry per thread doubles its parallelism (measured at RMAT-24:
      // level-0 expansion 1.75 -> 1.0 ms, the CUDA kernel's one-per-thread)
      if (App::kTypes > 1 && tu.regroup != 0 && n < (uint64_t)num_sms() * kBlock * 4)
        return launch_sorted<App, M, R, 1, App::kPrefetch>(objs, n, args, tbl, s);
    }
    if (App::kTypes > 1 && tu.regroup != 0)
      return launch_sorted<App, M, R, App::kUnrollSorted, App::kPrefetch>(objs, n, args, tbl, s);
    return launch_grouped<App, M, R, App::kUnroll, App::kPrefetch>(objs, n, args, tbl, s);
  } else {
  // Measured on B200 (config 2, 2^26 objects, profiles/sweep_knobs_r1.md):
  // with the per-tile type sort and the next tile's pointers in flight, the
  // L1 warm-up (prefetch 2; config 2's app default) wins at every type
  // count, also at >= 24 live types where it used to lose; 2 objects per thread up
  // to ~16 live types; with >= 24 live types (the sort leaves ~half-warp
  // groups) TypePointer prefers 4 objects per thread, COAL (whose smem search
  // adds registers) stays at 2. Without the sort, >= 24 types prefer 1.
  const bool rg = tu.regroup != 0 && App::kTypes > 1;
  const bool many = tbl.active_types >= 24;
  const int u = tu.unroll > 0 ? tu.unroll
                : rg ? (many ? (R::kNeedsTable ? 2 : 4) : App::kUnrollSorted)
                     : (many ? 1 : App::kUnroll);
  const int pf = tu.prefetch >= 0 ? tu.prefetch : (rg && many) ? 2 : App::kPrefetch;
  if (u >= 4) return launch_grouped_pf<App, M, R, 4>(pf, objs, n, args, tbl, s);
  if (u == 2) return launch_grouped_pf<App, M, R, 2>(pf, objs, n, args, tbl, s);
  return launch_grouped_pf<App, M, R, 1>(pf, objs, n, args, tbl, s);
  }
}

// ---------------------------------------------------------------------------
// Grid-level type sort for heavy methods (tuning key "gsort"; App::kHeavyMask).
//
// A CTA-level sort still leaves the warps that straddle two type runs of its
// tile running a long body twice (once per type, half the lanes each), and
// heavy bodies make every CTA wait for those warps. Because the type comes
// from the pointer alone (COAL / TypePointer), the whole dispatch list can be
// counting-sorted by type first — (pointer, index) pairs, index order kept
// within a type — so only the warps at the <= T-1 run boundaries of the whole
// list are mixed. Three small passes (per-chunk type histogram, per-type scan,
// placement) move 8 B in and 12 B out per entry; then one thread per sorted
// entry resolves its pointer again and runs the grouped direct call with the
// entry's ORIGINAL index (bodies that use it, e.g. graph work-entry chunks,
// see the same index). Calls are order-independent (reading G8).
// ---------------------------------------------------------------------------

template <class App, class R>
__device__ __forceinline__ uint32_t gs_type(const unsigned char* smem, const DevTable& tbl, uint64_t p) {
  if (!p) return 0xFFFFu;
  uint64_t a;
  uint32_t hint = 0;
  uint32_t t = R::resolve(smem, tbl, p, a, hint);
  if (t >= (uint32_t)App::kTypes) t = type_from_vptr<App>(a, tbl);  // fallback
  return t < (uint32_t)App::kTypes ? t : 0xFFFFu;                 // unresolvable: dropped (as the dispatch would)
}

template <class App, class R>
__global__ void __launch_bounds__(256) k_gs_hist(const uint64_t* __restrict__ objs, uint64_t n, DevTable tbl,
                                                 uint32_t* __restrict__ hist) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ uint32_t h[32];
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  if (threadIdx.x < 32) h[threadIdx.x] = 0;
  __syncthreads();
  const uint64_t base = (uint64_t)blockIdx.x * kGsChunk;
  const uint32_t lane = threadIdx.x & 31u;
  for (uint32_t r = 0; r < kGsChunk / 256; ++r) {
    const uint64_t i = base + (uint64_t)r * 256 + threadIdx.x;
    const uint32_t t = i < n ? gs_type<App, R>(smem, tbl, ldg_u64(objs + i)) : 0xFFFFu;
    const uint32_t peers = __match_any_sync(0xffffffffu, t);
    if (t < 32u && lane == (uint32_t)(__ffs(peers) - 1)) atomicAdd(&h[t], (uint32_t)__popc(peers));
  }
  __syncthreads();
  if (threadIdx.x < 32) hist[(uint64_t)blockIdx.x * 32 + threadIdx.x] = h[threadIdx.x];
}

template <class App, class R>
__global__ void __launch_bounds__(256) k_gs_place(const uint64_t* __restrict__ objs, uint64_t n, DevTable tbl,
                                                  const uint32_t* __restrict__ hist,
                                                  const unsigned long long* __restrict__ totals,
                                                  uint64_t* __restrict__ sp, uint32_t* __restrict__ si) {
  extern __shared__ __align__(16) unsigned char smem[];
  constexpr int kWarps = 256 / 32;
  __shared__ uint32_t run[32];
  __shared__ uint32_t wcnt[kWarps][32];
  __shared__ unsigned long long boff[32];
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  const uint32_t lane = threadIdx.x & 31u, warp = threadIdx.x >> 5;
  if (threadIdx.x < 32) {
    // this chunk's first slot of type t = (objects of types < t) + (type t in earlier chunks)
    const unsigned long long tot = lane < (uint32_t)App::kTypes ? totals[lane] : 0ull;
    unsigned long long x = tot;
#pragma unroll
    for (int o = 1; o < 32; o <<= 1) {
      const unsigned long long y = __shfl_up_sync(0xffffffffu, x, o);
      if (lane >= (uint32_t)o) x += y;
    }
    run[lane] = 0;
    boff[lane] = x - tot + hist[(uint64_t)blockIdx.x * 32 + lane];
  }
  const uint64_t base = (uint64_t)blockIdx.x * kGsChunk;
  for (uint32_t r = 0; r < kGsChunk / 256; ++r) {
    const uint64_t i = base + (uint64_t)r * 256 + threadIdx.x;
    const uint64_t p = i < n ? ldg_u64(objs + i) : 0ull;
    const uint32_t t = i < n ? gs_type<App, R>(smem, tbl, p) : 0xFFFFu;
    wcnt[warp][lane] = 0;
    __syncwarp();
    const uint32_t peers = __match_any_sync(0xffffffffu, t);
    const uint32_t within = __popc(peers & ((1u << lane) - 1u));
    if (t < 32u && lane == (uint32_t)(__ffs(peers) - 1)) wcnt[warp][t] = __popc(peers);
    __syncthreads();
    if (t < 32u) {
      uint32_t before = run[t];
      for (uint32_t w = 0; w < warp; ++w) before += wcnt[w][t];
      const unsigned long long pos = boff[t] + before + within;
      sp[pos] = p;
      si[pos] = (uint32_t)i;
    }
    __syncthreads();
    if (threadIdx.x < 32) {
      uint32_t c = 0;
      for (int w = 0; w < kWarps; ++w) c += wcnt[w][threadIdx.x];
      run[threadIdx.x] += c;
    }
    __syncthreads();
  }
}

// one thread per type-sorted entry; warps are type-uniform except at run boundaries
template <class App, int M, class R, int B = ListBlock<App>::value>
__global__ void __launch_bounds__(B, MinBlocks<App>::value * (kBlock / B)) k_dispatch_list(
    const uint64_t* __restrict__ sp, const uint32_t* __restrict__ si, const unsigned long long* __restrict__ totals,
    ArgBlob args, DevTable tbl) {
  extern __shared__ __align__(16) unsigned char smem[];
  __shared__ unsigned long long s_m;
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  if (threadIdx.x < 32) {
    // sorted entries = typed objects (nulls and untypable pointers were dropped)
    unsigned long long x = threadIdx.x < (uint32_t)App::kTypes ? totals[threadIdx.x] : 0ull;
#pragma unroll
    for (int o = 16; o > 0; o >>= 1) x += __shfl_xor_sync(0xffffffffu, x, o);
    if (threadIdx.x == 0) s_m = x;
  }
  __syncthreads();
  const uint64_t m = s_m;
  const uint64_t k = (uint64_t)blockIdx.x * B + threadIdx.x;
  uint64_t p = 0, a = 0, i = 0;
  uint32_t t = kNF, hint = 0;
  if (k < m) {
    p = ldg_u64(sp + k);
    i = __ldg(si + k);
    t = R::resolve(smem, tbl, p, a, hint);
  }
  group_call<App, M>(t, a, p, i, args, tbl);
}

uint64_t rank_chunks(uint64_t n);
cudaError_t scan_type_hist(uint32_t* hist, uint64_t nchunks, uint32_t ntypes, unsigned long long* totals,
                           cudaStream_t s);

template <class App, int M, class R>
cudaError_t launch_gsorted(const uint64_t* objs, uint64_t n, const ArgBlob& args, const DevTable& tbl,
                           cudaStream_t s) {
  static_assert(App::kTypes <= 32, "one warp scans the type totals");
  const uint64_t nch = (n + kGsChunk - 1) / kGsChunk;
  if (nch > 0x7FFFFFFFull || n > 0xFFFFFFFFull) return cudaErrorInvalidValue;
  const size_t hist_b = 128ull * nch, tot_b = 8ull * 32;
  const size_t sp_b = 8ull * n, si_b = 4ull * n;
  unsigned char* scratch = nullptr;
  cudaError_t e = cudaMallocAsync(reinterpret_cast<void**>(&scratch), hist_b + tot_b + sp_b + si_b + 64, s);
  if (e != cudaSuccess) return e;
  uint32_t* hist = reinterpret_cast<uint32_t*>(scratch);
  unsigned long long* totals = reinterpret_cast<unsigned long long*>(scratch + hist_b);
  uint64_t* sp = reinterpret_cast<uint64_t*>(scratch + align16(hist_b + tot_b));
  uint32_t* si = reinterpret_cast<uint32_t*>(reinterpret_cast<unsigned char*>(sp) + sp_b);
  const size_t tsm = R::kNeedsTable ? table_smem(tbl) : 0;
  if (tsm > 32 * 1024) {
    cudaFuncSetAttribute(k_gs_hist<App, R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tsm);
    cudaFuncSetAttribute(k_gs_place<App, R>, cudaFuncAttributeMaxDynamicSharedMemorySize, (int)tsm);
  }
  k_gs_hist<App, R><<<(unsigned)nch, 256, tsm, s>>>(objs, n, tbl, hist);
  e = scan_type_hist(hist, nch, App::kTypes, totals, s);
  if (e == cudaSuccess) {
    k_gs_place<App, R><<<(unsigned)nch, 256, tsm, s>>>(objs, n, tbl, hist, totals, sp, si);
    note_launch(2);
    // one thread per entry: n threads cover the (<= n) sorted entries
    constexpr auto kern = k_dispatch_list<App, M, R>;
    (void)occupancy<kern>(tsm);  // sets the dynamic smem attribute when needed
    constexpr int B = ListBlock<App>::value;
    kern<<<grid_for(n, B, ~0ull), B, tsm, s>>>(sp, si, totals, args, tbl);
    note_launch();
    e = cudaGetLastError();
  }
  cudaFreeAsync(scratch, s);
  return e;
}

template <class App, int M, class R>
cudaError_t launch_indirect(const uint64_t* objs, uint64_t n, const ArgBlob& args, const DevTable& tbl,
                            cudaStream_t s) {
  constexpr auto kern = k_dispatch_indirect<App, M, R>;
  const size_t sm = R::kNeedsTable ? table_smem(tbl) : 0;
  const int occ = occupancy<kern>(sm);
  kern<<<grid_for(n, kBlock, (uint64_t)num_sms() * occ), kBlock, sm, s>>>(objs, n, args, tbl);
  note_launch();
  return cudaGetLastError();
}

template <class App, int M>
cudaError_t dispatch_method(int variant, const uint64_t* objs, uint64_t n, const ArgBlob& args,
                            const DevTable& tbl, cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  const bool indirect = tuning().call != 0;
  switch (variant) {
    case VF_CUDA:
    case VF_SHAREDOA:
      return launch_virtual<App, M>(objs, n, args, s);
    case VF_COAL:
      if (indirect) return launch_indirect<App, M, ResolveCOAL>(objs, n, args, tbl, s);
      return launch_grouped_tuned<App, M, ResolveCOAL>(objs, n, args, tbl, s);
    case VF_TYPEPTR:
      if (indirect) return launch_indirect<App, M, ResolveTP>(objs, n, args, tbl, s);
      return launch_grouped_tuned<App, M, ResolveTP>(objs, n, args, tbl, s);
    case VF_CONCORD:
      if constexpr (TagOffset<App>::value >= 0) {
        k_dispatch_concord<App, M><<<grid_for(n, kBlock, ~0u), kBlock, 0, s>>>(objs, n, args);
        note_launch();
        return cudaGetLastError();
      } else {
        return cudaErrorNotSupported;
      }
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

// ---------------------------------------------------------------------------
// Fused per-index step (B200 design for apps whose step is a non-virtual
// pre-phase, the virtual call and a non-virtual post-phase on the same index,
// e.g. the cellular automata): one thread per index runs all three, so a
// whole step is ONE launch and the pre-phase's result reaches the method
// through L1 instead of a separate kernel round trip. The call itself is the
// variant's: a plain virtual call (CUDA / SharedOA) or resolve + warp-grouped
// direct call (COAL / TypePointer). Step provides
//   __device__ void pre(uint64_t c) const; uint64_t ptr(uint64_t c) const;
//   void post(uint64_t c) const;
// ---------------------------------------------------------------------------
// Optional Step hook `uint32_t warm(uint64_t c, uint64_t addr) const`: touch
// (L1-allocating loads) what the method will read before the type groups run
// one after another, so the second group's loads hit L1 (cf. warm_line).
template <class S, class = void>
struct HasWarm {
  static constexpr bool value = false;
};
template <class S>
struct HasWarm<S, std::void_t<decltype(std::declval<const S&>().warm(0ull, 0ull))>> {
  static constexpr bool value = true;
};

template <class App, int M, class R, class Step>
__global__ void __launch_bounds__(kBlock) k_step_grouped(uint64_t n, ArgBlob args, DevTable tbl, Step st) {
  extern __shared__ __align__(16) unsigned char smem[];
  if constexpr (R::kNeedsTable) R::stage(smem, tbl);
  uint32_t hint = 0;
  // CTA-uniform loop: every lane of every warp iterates together (full-mask collectives)
  for (uint64_t base = (uint64_t)blockIdx.x * kBlock; base < n; base += (uint64_t)gridDim.x * kBlock) {
    const uint64_t c = base + threadIdx.x;
    const bool valid = c < n;
    uint64_t p = 0, a = 0;
    uint32_t t = kNF;
    if (valid) {
      st.pre(c);
      p = st.ptr(c);
    }
    if (p) t = R::resolve(smem, tbl, p, a, hint);
    if constexpr (HasWarm<Step>::value) {
      uint32_t sink = 0;
      if (valid && t < (uint32_t)App::kTypes) sink = st.warm(c, a);
      group_call<App, M>(t, a, p, c, args, tbl);
      if (sink == 0x8BADF00Du && n == ~0ull) asm volatile("st.global.u32 [%0], %1;" ::"l"(st.ptr_base()), "r"(sink));
    } else {
      group_call<App, M>(t, a, p, c, args, tbl);
    }
    if (valid) st.post(c);
  }
}

template <class App, int M, class Step>
__global__ void __launch_bounds__(kBlock) k_step_virtual(uint64_t n, ArgBlob args, Step st) {
  const uint64_t c = (uint64_t)blockIdx.x * kBlock + threadIdx.x;
  if (c >= n) return;
  st.pre(c);
  const uint64_t p = st.ptr(c);
  if (p) App::template vcall<M>(reinterpret_cast<typename App::Base*>(p), c, args);
  st.post(c);
}

template <class App, int M, class R, class Step>
cudaError_t launch_step_grouped(uint64_t n, const ArgBlob& args, const DevTable& tbl, const Step& st,
                                cudaStream_t s) {
  constexpr auto kern = k_step_grouped<App, M, R, Step>;
  const size_t sm = R::kNeedsTable ? table_smem(tbl) : 0;
  const int occ = occupancy<kern>(sm);
  kern<<<grid_for(n, kBlock, (uint64_t)num_sms() * occ), kBlock, sm, s>>>(n, args, tbl, st);
  note_launch();
  return cudaGetLastError();
}

template <class App, int M, class Step>
cudaError_t launch_step(int variant, uint64_t n, const ArgBlob& args, const DevTable& tbl, const Step& st,
                        cudaStream_t s) {
  if (n == 0) return cudaSuccess;
  switch (variant) {
    case VF_CUDA:
    case VF_SHAREDOA:
      k_step_virtual<App, M, Step><<<grid_for(n, kBlock, ~0u), kBlock, 0, s>>>(n, args, st);
      note_launch();
      return cudaGetLastError();
    case VF_COAL:
      return launch_step_grouped<App, M, ResolveCOAL, Step>(n, args, tbl, st, s);
    case VF_TYPEPTR:
      return launch_step_grouped<App, M, ResolveTP, Step>(n, args, tbl, st, s);
  }
  return cudaErrorInvalidValue;
}

// live (state == 1) neighbours of cell c of a W x H grid (dead border, or
// torus). 32-bit index arithmetic (W*H < 2^32, checked at the ABI): a 64-bit
// `c / W` compiles to a CALL into the u64 division subroutine.
__device__ __forceinline__ uint8_t count_live(uint32_t W, uint32_t H, int torus, const uint8_t* __restrict__ st,
                                              uint32_t c) {
  const uint32_t yq = c / W;
  const int y = (int)yq, x = (int)(c - yq * W);
  int n = 0;
#pragma unroll
  for (int dy = -1; dy <= 1; ++dy)
#pragma unroll
    for (int dx = -1; dx <= 1; ++dx) {
      if (dx == 0 && dy == 0) continue;
      int yy = y + dy, xx = x + dx;
      if (torus) {
        yy = (yy + (int)H) % (int)H;
        xx = (xx + (int)W) % (int)W;
      } else if (yy < 0 || yy >= (int)H || xx < 0 || xx >= (int)W) {
        continue;
      }
      n += st[(uint32_t)yy * W + (uint32_t)xx] == 1;
    }
  return (uint8_t)n;
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
