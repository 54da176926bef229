/*
 * vf.h — C ABI of libvf.so: B200-native GPU virtual-function dispatch after
 * "Judging a Type by Its Pointer: Optimizing GPU Virtual Functions"
 * (Zhang, Alawneh, Rogers, ASPLOS'21). Citations are P:<line> of the paper
 * text with the section / figure / algorithm they fall in.
 *
 * The paper's user-visible operations are
 *   - `Obj* = sharedNew TYPE()`                 (Fig. 4, §4)
 *       -> vf_alloc_typed / vf_alloc_typed_batch (type-based arenas + the
 *          virtual range table of Fig. 3)
 *   - device `new TYPE()` of the CUDA baseline
 *       -> vf_alloc_cuda
 *   - TypePointer `new` returning a tagged pointer (Fig. 5a P:1178-1180,
 *       §6.1) -> `tag` = 1 on any allocation call
 *   - `obj->vFun()` (Fig. 4) resolved four ways:
 *       vf_dispatch_cuda      embedded vTable* -> vFunc* -> indirect CALL
 *                             (Fig. 1a, §2)
 *       vf_dispatch_sharedoa  the same call on SharedOA-allocated objects (§4)
 *       vf_dispatch_coal      ObjectRangeLookup on the object address alone
 *                             (§5, Algorithm 1)
 *       vf_dispatch_typeptr   type from the pointer's upper bits (§6, Fig. 5b)
 *
 * Conventions (all functions):
 *   - extern "C", never throw; return vf_status (VF_OK == 0). On failure a
 *     human-readable detail is available from vf_last_error(ctx).
 *   - Pointer arguments named *_dev are DEVICE pointers (caller-owned, e.g.
 *     torch tensors' data_ptr()); all others are host pointers.
 *   - All device work is enqueued on `stream` (a cudaStream_t passed as
 *     void*; NULL = legacy default stream) and is asynchronous; CUDA faults
 *     surface on a later call as VF_ERR_CUDA.
 *   - A ctx is bound to one device and must not be used from two host
 *     threads at once. Type ids are app-local (0 .. ntypes-1) and global
 *     across ranks; addresses and range tables are per device.
 *   - Ownership: the ctx owns every object, arena, range table and the
 *     device heap objects it created; the caller owns pointer arrays,
 *     argument blobs and output buffers.
 */
#ifndef VF_H
#define VF_H
#include <stddef.h>
#include <stdint.h>

#ifdef __cplusplus
extern "C" {
#endif

/* float4 in the ABI: CUDA's float4 inside the library, a plain 16-B-aligned
 * struct for C callers (same layout). */
#if defined(__CUDACC__)
typedef float4 float4_t;
typedef float2 float2_t;
#else
typedef struct { float x, y, z, w; } __attribute__((aligned(16))) float4_t;
typedef struct { float x, y; } __attribute__((aligned(8))) float2_t;
#endif

typedef enum {
  VF_OK = 0,
  VF_ERR_INVALID = 1,         /* bad argument (null ctx, unknown app/method/type, ...) */
  VF_ERR_OOM = 2,             /* device memory / device heap / VA exhausted            */
  VF_ERR_CUDA = 3,            /* a CUDA runtime/driver call failed                     */
  VF_ERR_TAG_BITS = 4,        /* an object address has bits 63:57 != 0  */
  VF_ERR_TOO_MANY_TYPES = 5,  /* more types than a 7-bit tag / 32-lane group can hold  */
  VF_ERR_TABLE_FULL = 6,      /* range table larger than VF_MAX_RANGES                 */
  VF_ERR_UNSUPPORTED = 7      /* valid but not implemented for this app/variant        */
} vf_status;

/* VF_CONCORD is the paper's comparison point (§7): a type tag
 * embedded in every object, read per call and switched on (apps with an
 * embedded tag only: VF_APP_MICRO; others return VF_ERR_UNSUPPORTED). */
typedef enum { VF_CUDA = 0, VF_SHAREDOA = 1, VF_COAL = 2, VF_TYPEPTR = 3, VF_CONCORD = 4 } vf_variant;

/* Workload apps compiled into libvf.so (GPUs cannot load code at run time,
 * so every class whose virtual methods a kernel may call is compiled into
 * that kernel's module: P:607-615). */
enum {
  VF_APP_MICRO = 0, /* config 2: MObj<k>::apply(){ val += k+1; }  (§8.3)      */
  VF_APP_GOL = 1,   /* config 1: Cell / Alive / Dead               (Table 2)  */
  VF_APP_GEN = 2,   /* config 5: Cell / Dead / Alive / Dying       (Table 2)  */
  VF_APP_GRAPH = 3, /* config 4: Vertex / Leaf / Low / Mid / Hub   (Table 2)  */
  VF_APP_RAY = 4,   /* config 3: Shape / Plane / Sphere / Rect / Triangle   */
  VF_APP_TRAF = 5,  /* config 5: Agent / PlainCell / LightCell / Car / Truck / Bus        */
  VF_APP_NBODY = 6, /* config 5: Body / Star / Planet / Dust (all-pairs N-body, G18)      */
  VF_APP_STUT = 7,  /* config 5: Element / Node / AnchorNode / AnchorPullNode / Spring   */
  VF_APP_COLLIDE = 8, /* config 5: Body / Star / Planet / Dust (cutoff grid + merging, G19) */
  VF_APP_GRAPH_EN = 9,/* GraphChi-vEN vertices: ChiVertex / Leaf / Low / Mid / Hub */
  VF_APP_EDGE = 10,   /* GraphChi-vEN edges: ChiEdge / Edge / HubEdge  (G32)     */
  VF_APP_COUNT = 11
};

/* Methods of VF_APP_STUT (Table 2 "structure" P:1524-1528, reading G17). Type
 * ids 0 Node, 1 AnchorNode, 2 AnchorPullNode (ctor {u32 id, f32 vx, vy, m}),
 * 3 Spring (ctor {u32 id, a, b, f32 L0, k, u32 pad}). One step = FORCE on
 * every spring, then MOVE on every node:
 *   force(): broken -> 0; d = pos[b]-pos[a], len = sqrt(fmaf(dx,dx,dy*dy));
 *            len > break_ratio*L0 -> broken = 1 (permanent), 0; else
 *            fs = (k*(len-L0))/len, F[id] = (fs*dx, fs*dy) (acts on a, -F on b)
 *   move():  Node: sum F of incident springs (inc_offs/inc CSR, code =
 *            spring<<1 | is_b, ascending), F = fmaf(-c, v, F),
 *            v = fmaf(dt, F/m, v), pos = fmaf(dt, v, pos); AnchorNode: none;
 *            AnchorPullNode: pos.x = fmaf(dt, v_pull, pos.x).
 * Methods a class does not define are no-ops on it. */
enum { VF_STUT_FORCE = 0, VF_STUT_MOVE = 1, VF_STUT_GET = 2 };
typedef struct {
  const float2_t* pos_dev;  /* node positions (n)                 */
  float2_t* F_dev;          /* per-spring force of this step (S)  */
  float break_ratio;
} vf_stut_force_args;
typedef struct {
  float2_t* pos_dev;
  const float2_t* F_dev;
  const uint32_t* inc_offs_dev;  /* n+1 */
  const uint32_t* inc_dev;       /* 2S  */
  float dt, c, v_pull;
} vf_stut_move_args;
typedef struct {
  float* vel_out_dev;       /* nodes: 2 floats at (id - id_base), may be NULL      */
  uint8_t* broken_out_dev;  /* springs: flag at (id - spring_base), may be NULL    */
  uint32_t id_base, spring_base;
} vf_stut_get_args;

/* Methods of VF_APP_NBODY (reading G18; DynaSOAr's N-body, BASELINE north_star).
 * Type ids 0 Star, 1 Planet, 2 Dust; constructor argument {u32 idx, f32 vx,
 * vy, vz}. Positions+masses are float4 (x, y, z, m) arrays indexed by idx.
 * update(): a = sum_{j != idx, ascending j} m_j d / (r^2+eps2[type])^{3/2}
 * with r2 = fmaf(dx,dx,fmaf(dy,dy,fmaf(dz,dz,eps2))), 1/(r2*sqrt(r2)),
 * a = fmaf(d, m_j*inv, a); Dust: v *= damp; v = fmaf(dt,a,v);
 * pout[idx] = (fmaf(dt,v,x), ..., m). Reads pin[0..N), writes pout[idx].
 * Precondition (IEEE-exact results): eps2[t] >= 1e-20 and |coordinates| < 1e11. */
enum { VF_NBODY_UPDATE = 0, VF_NBODY_GET = 1 };
typedef struct {
  const float4_t* pin_dev;  /* N float4, positions at the start of the step (all bodies) */
  float4_t* pout_dev;       /* N float4, this call writes pout[idx] of its bodies only   */
  uint32_t N;
  float dt;
  float eps2[3];            /* per type softening^2                                      */
  float damp;               /* Dust velocity factor per step                             */
} vf_nbody_update_args;
typedef struct {
  float* vel_out_dev;       /* 3 floats per body at (idx - idx_base)                     */
  uint32_t idx_base;
} vf_nbody_get_args;

/* Methods of VF_APP_COLLIDE (config 5 "collision" at 16M bodies; DynaSOAr's
 * collision app [46], readings G18 / G19 in DESIGN.md). Type ids 0 Star,
 * 1 Planet, 2 Dust; constructor argument {u32 idx, f32 vx, vy, vz} (the body
 * keeps its velocity; positions+masses are float4 (x, y, z, m) arrays indexed
 * by idx, m <= 0 = absorbed / inactive). One step, from the state P at its
 * start: vf_collide_grid (non-virtual: uniform grid of cells of side rc, ids
 * ascending per cell), then one virtual update() and one virtual merge() per
 * active body:
 *   update(): over the 27 neighbour cells in (z, y, x) order, bodies j != idx
 *     in ascending id: d = p_j - p_i, d2 = fmaf(dx,dx,fmaf(dy,dy,dz*dz)); if
 *     d2 < rc2: r2 = fmaf(dx,dx,fmaf(dy,dy,fmaf(dz,dz,eps2[type]))),
 *     a = fmaf(d, m_j * (1/(r2*sqrt(r2))), a); the nearest j with d2 < rm2
 *     (ties: smaller id) is near[idx] (-1 if none). Dust: v *= damp;
 *     v = fmaf(dt,a,v); Pm[idx] = (fmaf(dt,v,x), m); Vm[idx] = v if near >= 0.
 *   merge(): j = near[idx]; if near[j] == idx the smaller id absorbs:
 *     m = m_i + m_j, x = fmaf(m_i,x_i,m_j*x_j)/m, v likewise (post-update
 *     values); the larger id gets mass 0, velocity 0, position kept.
 *     P[idx] = the result (Pm[idx] when there is no mutual partner).
 * Same arithmetic as VF_APP_NBODY (IEEE-exact, no contraction). Preconditions:
 * eps2[t] >= 1e-20, rc2 + eps2 <= 1e24, |coordinates| < 1e11. */
enum { VF_COLLIDE_UPDATE = 0, VF_COLLIDE_MERGE = 1, VF_COLLIDE_GET = 2 };
typedef struct {
  const float4_t* P_dev;           /* N, start of step, by id (all bodies)            */
  const float4_t* Ps_dev;          /* N, cell-sorted copy: Ps[e] = P[list[e]]          */
  const uint32_t* list_dev;        /* ids in cell order, ascending within a cell       */
  const uint32_t* cell_start_dev;  /* G^3 + 1 offsets into list                         */
  const uint32_t* slot_dev;        /* N, slot[id] = e with list[e] = id (active bodies) */
  float4_t* Pm_dev;                /* N, post-update position + mass, by id             */
  float4_t* Vm_dev;                /* N, post-update velocity (written when near >= 0)  */
  int32_t* near_dev;               /* N, nearest body within rm or -1                   */
  uint32_t G;
  float rc, rc2, rm2, dt;          /* rc2 = rc*rc, rm2 = rm*rm (fp32, host-rounded)     */
  float eps2[3];
  float damp;
} vf_collide_update_args;
typedef struct {
  const float4_t* Pm_dev;
  const float4_t* Vm_dev;
  const int32_t* near_dev;
  float4_t* P_dev;                 /* N, end of step, by id: this call writes P[idx]    */
} vf_collide_merge_args;
typedef struct {
  float* vel_out_dev;              /* 3 floats per body at (idx - idx_base)              */
  uint32_t idx_base;
} vf_collide_get_args;

/* Methods of VF_APP_TRAF (Table 2, reading G16). Type ids: 0
 * PlainCell, 1 LightCell (ctor arg {u32 cell, u32 phase}); 2 Car, 3 Truck,
 * 4 Bus (ctor arg {u32 id, u32 ring, u32 pos, u32 pad}). Cells are indexed
 * globally (ring * L + pos). */
enum {
  VF_TRAF_CELL_UPDATE = 0, /* blocked[c] = LightCell red ((t+phase) mod 20 < 8); occ_next[c] = 0 */
  VF_TRAF_VEH_STEP = 1,    /* Nagel-Schreckenberg step against occ / blocked; sets occ_next  */
  VF_TRAF_GET = 2,         /* pos_out[id], v_out[id]                                          */
  VF_TRAF_PLACE = 3        /* occ[ring*L + pos] = 1 (initial occupancy)                        */
};
typedef struct {
  uint8_t* blocked_dev;
  uint8_t* occ_next_dev;
  uint32_t t;
} vf_traf_cell_args;
typedef struct {
  const uint8_t* occ_dev;
  const uint8_t* blocked_dev;
  uint8_t* occ_next_dev;
  uint32_t L, t;
  uint64_t seed;
  uint32_t vmax[3];
  uint32_t slow_thr[3];
} vf_traf_step_args;
typedef struct {
  uint32_t* pos_out_dev;  /* indexed by id - id_base (vehicle ids are global, ring-major) */
  uint32_t* v_out_dev;
  uint8_t* occ_dev;
  uint32_t L;
  uint32_t id_base;
} vf_traf_get_args;

/* Methods of VF_APP_MICRO (args structs are passed by value, see dispatch).
 * Layout {vptr, i32 val, u32 tag}: tag = the class id, Concord's embedded
 * type field (VF_CONCORD reads it; the other variants ignore it). */
enum { VF_MICRO_APPLY = 0, /* args: none                                       */
       VF_MICRO_GET = 1 }; /* args: vf_micro_get_args — out_dev[i] = objs[i].val */
typedef struct { int32_t* out_dev; } vf_micro_get_args;

/* Methods of VF_APP_GOL. */
enum { VF_GOL_NEXT = 0, /* args: vf_gol_next_args (one generation, step 2 of W1) */
       VF_GOL_GET = 1 };/* args: vf_gol_get_args                                  */
typedef struct {
  const uint8_t* nbr_dev;   /* live-neighbour count per cell (cell id = object's own index) */
  uint8_t* state_out_dev;   /* next state per cell                                          */
} vf_gol_next_args;
typedef struct { uint16_t* counter_out_dev; uint8_t* type_out_dev; } vf_gol_get_args;

/* Methods of VF_APP_GEN (Generations CA B/S/C, reading G15; type ids 0 Dead,
 * 1 Alive, 2 Dying). born/survive: bit n set = rule holds with n live
 * (state-1) neighbours; C = number of states (2..255). */
enum { VF_GEN_NEXT = 0, VF_GEN_GET = 1 };
typedef struct {
  const uint8_t* nbr_dev;   /* live (state-1) neighbours per cell                  */
  uint8_t* state_out_dev;   /* next state per cell                                 */
  uint32_t born_mask, survive_mask, C;
} vf_gen_next_args;
typedef struct { uint16_t* counter_out_dev; uint8_t* type_out_dev; } vf_gen_get_args;

/* Methods of VF_APP_GRAPH (readings G20-G23). Type ids by degree: 0 Leaf
 * (<= 1), 1 Low (2..15), 2 Mid (16..255), 3 Hub (>= 256). Constructor
 * argument per object: { u32 vid, u32 deg }. CSR: offs[V+1] (u64), col (u32),
 * symmetric. vobj_dev[v] = the object pointer of vertex v.
 *
 * Work entries (load balance): a dispatch list holds one entry
 * per (vertex, edge chunk): a vertex of degree deg > C appears
 * nch = ceil(deg / C) times, consecutively, with chunk_dev[i] = 0 .. nch-1
 * (chunk_dev is read only for such vertices); every other vertex appears once.
 * Entry i of vertex v covers edges [offs[v] + c*C, min(offs[v] + (c+1)*C,
 * offs[v+1])). Each entry is one virtual call on v's object. */
enum {
  VF_GRAPH_BFS_EXPAND = 0, /* top-down: claim depth[u] = level+1 for unvisited neighbours
                              (atomicCAS) and append u's entries to next_queue /
                              next_chunk; *next_count counts appended entries           */
  VF_GRAPH_BFS_PROBE = 1,  /* bottom-up: an unvisited vertex with a neighbour at `level`
                              takes depth level+1 (atomicCAS); *next_count = 1 if any   */
  VF_GRAPH_CC_UPDATE = 2,  /* label_out[v] = min(label_in over v and N(v)) (Jacobi; a
                              multi-chunk vertex combines with atomicMin: label_out must
                              hold a label >= label_in[v], e.g. the previous-but-one
                              iterate); *changed = 1 if it is below label_in[v]          */
  VF_GRAPH_PR_CONTRIB = 3, /* chunk 0 only: contrib[v] = deg ? rank_in[v]/deg : 0, the
                              fp64 quotient rounded once to fp32 (DESIGN §2 R-PR32);
                              deg-0 vertices add rank_in[v] to *dangling                 */
  VF_GRAPH_PR_UPDATE = 4,  /* rank_out[v] = (float)(base + d*(sum_{N(v)} contrib +
                              *dangling / Vd)); a multi-chunk vertex writes its chunk sum
                              to partial[i]; the last chunk to finish (counter[v]) sums
                              the partials in chunk order and resets counter[v] to 0    */
  VF_GRAPH_BFS_PROBE_BITS = 5 /* bottom-up over a frontier BITMAP (multi-GPU, SURVEY §8e:
                              the per-level exchange is an all-gather of bitmap slices):
                              an unvisited vertex v with a neighbour u whose bit is set in
                              frontier_bits takes depth level+1 (atomicCAS), sets bit v of
                              next_bits (atomicOr) and *next_count = 1. Args:
                              vf_graph_bfs_bits_args                                     */
};
typedef struct {
  const uint64_t* offs_dev;
  const uint32_t* col_dev;
  int32_t* depth_dev;
  const uint64_t* vobj_dev;
  const uint32_t* chunk_dev;   /* chunk index of each entry of this dispatch       */
  uint64_t* next_queue_dev;    /* top-down: next frontier entries (objects)        */
  uint32_t* next_chunk_dev;    /* top-down: their chunk indices                    */
  uint32_t* next_count_dev;
  int32_t level;
  uint32_t C;                  /* edges per chunk (>= 1)                           */
} vf_graph_bfs_args;
/* VF_GRAPH_BFS_PROBE_BITS: bit v of a bitmap is word v >> 5, bit v & 31 (u32 words). */
typedef struct {
  const uint64_t* offs_dev;
  const uint32_t* col_dev;
  int32_t* depth_dev;          /* read + written for the dispatched (owned) vertices only */
  const uint32_t* frontier_dev;/* ceil(V/32) words: vertices at depth `level`            */
  uint32_t* next_dev;          /* ceil(V/32) words: owned vertices that joined level+1;
                                  the caller zeroes the owned words before the call     */
  const uint32_t* chunk_dev;
  uint32_t* next_count_dev;
  int32_t level;
  uint32_t C;
} vf_graph_bfs_bits_args;
typedef struct {
  const uint64_t* offs_dev;
  const uint32_t* col_dev;
  const uint32_t* label_in_dev;
  uint32_t* label_out_dev;
  uint32_t* changed_dev;
  const uint32_t* chunk_dev;
  uint32_t C;
} vf_graph_cc_args;
typedef struct {
  const uint64_t* offs_dev;
  const uint32_t* col_dev;
  const float* rank_in_dev;
  float* rank_out_dev;
  float* contrib_dev;          /* V floats (gathered; summed in fp64 by pr_update) */
  double* dangling_dev;
  double base, d, Vd;
  const uint32_t* chunk_dev;
  double* partial_dev;         /* one slot per entry of this dispatch              */
  uint32_t* counter_dev;       /* per vertex, zero between iterations              */
  uint32_t C;
} vf_graph_pr_args;

/* GraphChi-vEN: virtual edges AND virtual vertices (Table 2 P:1566-1588:
 * "GraphChi-vEN CC has both virtual edges and nodes"; readings
 * G32/G33 in DESIGN.md). Same CSR, degree-bucket vertex types, constructor
 * argument { u32 vid, u32 deg } and work entries as VF_APP_GRAPH.
 *
 * VF_APP_EDGE objects: one per arc k = (u -> v) of the symmetric CSR, type 0
 * Edge, or 1 HubEdge when the source u is a Hub (deg >= 256); constructor
 * argument { u32 src, u32 dst }. Layout (32 B): { vTable*, u32 src, u32 dst,
 * union { double f[2]; u32 u[2]; } val } — a double-buffered edge value
 * (Jacobi: iteration with buffer b reads val[b], the next reads val[1-b]).
 * out_edges_dev[k] = pointer of arc k (the vertex's own arcs, CSR order);
 * in_edges_dev[k] = pointer of the reverse arc (col[k] -> v) of arc k, so the
 * in-edges of v are visited in ascending source order, the oracle's order.
 *
 * Inside a vertex method every edge access is a virtual call on the edge
 * object (ChiEdge::target / get_pr / get_label). Under VF_CUDA / VF_SHAREDOA
 * it is the compiler's virtual call (vTable* load, vFunc* load, indirect
 * CALL); under VF_COAL / VF_TYPEPTR the vertex body is devirtualised and so
 * are its edge calls: the edge type comes from the edge pointer by `er.rule`
 * (VF_COAL: the edge app's range table; VF_TYPEPTR: the pointer's tag),
 * unresolvable pointers fall back to the embedded vTable* (matched against
 * er.vptr_dev), and the lanes of a warp are grouped by edge type for a
 * direct, inlined call. Pointers in the edge arrays must be tagged under
 * VF_TYPEPTR (vf_alloc_typed_batch(tag = 1)). */
typedef struct {
  const uint64_t* start_dev;   /* VF_APP_EDGE range table rows (vf_range_table), device copies */
  const uint64_t* end_dev;
  const uint32_t* type_dev;
  const uint64_t* vptr_dev;    /* vf_type_vptrs(VF_APP_EDGE): 2 entries                          */
  uint32_t K;                  /* rows                                                           */
  uint32_t P;                  /* smallest power of two >= K                                     */
  uint32_t rule;               /* VF_COAL or VF_TYPEPTR (used only by the COAL/TP kernels)        */
} vf_edge_resolver;

enum {
  VF_GRAPH_EN_BFS_EXPAND = 0, /* top-down: for each out-edge e of the entry's chunk, u =
                                 e->target(); claim depth[u] = level+1 (atomicCAS) and
                                 append u's entries to next_queue / next_chunk           */
  VF_GRAPH_EN_CC_UPDATE = 1,  /* m = min(label_in[v], e->get_label(b) over the chunk's
                                 in-edges); label_out[v] = m (multi-chunk: atomicMin, as
                                 VF_GRAPH_CC_UPDATE); *changed = 1 if m < label_in[v]     */
  VF_GRAPH_EN_PR_INIT = 2,    /* chunk 0 only: contrib[v] = deg ? rank_in[v]/deg : 0;
                                 deg-0 vertices add rank_in[v] to *dangling_out           */
  VF_GRAPH_EN_PR_GATHER = 3   /* s = sum of e->get_pr(b) over the chunk's in-edges (fp64);
                                 multi-chunk combine as VF_GRAPH_PR_UPDATE; r =
                                 (float)(base + d*(s + *dangling_in/Vd)); rank_out[v] = r,
                                 contrib[v] = deg ? r/deg : 0, deg-0: *dangling_out += r */
};
enum {
  VF_EDGE_PULL_PR = 0,    /* val.f[slot] = contrib[src]  (the edge stores its source's share) */
  VF_EDGE_PULL_LABEL = 1, /* val.u[slot] = label[src]                                         */
  VF_EDGE_GET = 2         /* out[k] = (u64)src << 32 | dst, k = the entry index (verification) */
};
typedef struct {
  const uint64_t* offs_dev;
  const uint64_t* out_edges_dev;
  int32_t* depth_dev;
  const uint64_t* vobj_dev;
  const uint32_t* chunk_dev;
  uint64_t* next_queue_dev;
  uint32_t* next_chunk_dev;
  uint32_t* next_count_dev;
  int32_t level;
  uint32_t C;
  vf_edge_resolver er;
} vf_graph_en_bfs_args;
typedef struct {
  const uint64_t* offs_dev;
  const uint64_t* in_edges_dev;
  const uint32_t* label_in_dev;
  uint32_t* label_out_dev;
  uint32_t* changed_dev;
  const uint32_t* chunk_dev;
  uint32_t C;
  uint32_t b;                  /* edge buffer read this iteration (0 / 1)                        */
  vf_edge_resolver er;
} vf_graph_en_cc_args;
typedef struct {
  const uint64_t* offs_dev;
  const uint64_t* in_edges_dev;
  const float* rank_in_dev;
  float* rank_out_dev;
  double* contrib_dev;
  const double* dangling_in_dev;  /* D_t (read)                                                 */
  double* dangling_out_dev;       /* D_{t+1} (accumulated; zeroed by the caller)                 */
  double base, d, Vd;
  const uint32_t* chunk_dev;
  double* partial_dev;
  uint32_t* counter_dev;
  uint32_t C;
  uint32_t b;
  vf_edge_resolver er;
} vf_graph_en_pr_args;
typedef struct {
  const double* contrib_dev;
  const uint32_t* label_dev;
  uint64_t* out_dev;           /* VF_EDGE_GET                                                    */
  uint32_t slot;
} vf_edge_args;

#define VF_MAX_RANGES 4096u     /* COAL range-table capacity (staged in shared memory)   */
#define VF_MAX_ARGS_BYTES 256u  /* method argument blob, copied into kernel parameters   */
#define VF_VA_BITS 57u          /* TypePointer: tag in bits 63:57 (reading G6)           */
#define VF_NOT_FOUND 0xFFFFFFFFu

typedef struct vf_ctx vf_ctx;

typedef struct {
  int device;                /* CUDA device ordinal                                        */
  uint64_t init_chunk_objs;  /* first region size in objects (4K)               */
  int reserve_va;            /* 1: reserve one VA window per type so consecutive regions   */
                             /*    are contiguous and merge (K = #types); 0: one           */
                             /*    cudaMalloc per region (K grows as log2)      */
  uint64_t va_window_bytes;  /* VA reserved per (app,type) when reserve_va (default 64 GiB)*/
  uint64_t cuda_heap_bytes;  /* device malloc heap for vf_alloc_cuda; must   */
                             /* be set before any device-malloc kernel in the process      */
} vf_config;

/* One row of the virtual range table (Fig. 3): [start, end) holds objects of
 * (app, type_id) whose embedded device vTable* equals vptr. Reading G1:
 * "Range" is the end address, half-open. */
typedef struct {
  uint64_t start, end;
  uint32_t type_id, app;
  uint64_t vptr;
} vf_range;

/* One raw allocator region before merging. */
typedef struct {
  uint64_t start;
  uint64_t cap_objs;   /* capacity in objects (4096, 8192, ... per type)  */
  uint64_t used_objs;
  uint32_t obj_bytes;  /* stride = sizeof(class)                          */
  uint32_t type_id, app, pad;
} vf_region;

/* Fills *cfg with defaults: device 0, 4096, reserve_va 1, 64 GiB, 8 GiB heap. */
void vf_config_default(vf_config* cfg);
vf_status vf_create(const vf_config* cfg, vf_ctx** out);
/* Frees all arenas and device-heap objects; every object pointer becomes invalid. */
void vf_destroy(vf_ctx* ctx);
const char* vf_status_str(vf_status s);
const char* vf_last_error(const vf_ctx* ctx);

/* App metadata: number of concrete types, sizeof each type (bytes, ntypes
 * entries written to obj_bytes if non-null), number of methods. */
vf_status vf_app_info(uint32_t app, uint32_t* ntypes, uint32_t* obj_bytes, uint32_t* nmethods);

/* ---- allocation (one-time; not timed) --------- */
/* `count` objects of class (app, type_id), placed at the next slots of that
 * type's arena (regions of 4K, 8K, ... objects) and constructed on
 * the device (vTable* installed). ctor_args_dev: optional
 * per-object constructor argument blob (ctor_arg_bytes each, app-defined,
 * may be NULL). Writes `count` u64 pointers to out_ptrs_dev. tag = 1 returns
 * TypePointer pointers: (type_id+1) << 57 | address (Fig. 5a). Objects live
 * until vf_reset / vf_destroy. */
vf_status vf_alloc_typed(vf_ctx* ctx, uint32_t app, uint32_t type_id, uint64_t count,
                         const void* ctor_args_dev, uint32_t ctor_arg_bytes,
                         uint64_t* out_ptrs_dev, int tag, void* stream);
/* Batched: object i is of class (app, type_ids_dev[i]) and takes the next
 * slot of its type's arena in index order (allocation order = index order).
 * The slot of object i is its rank among the objects of its type with a
 * smaller index: a device prefix count (per-chunk type histograms, a per-type
 * scan, then a placement pass); only the per-type totals (ntypes x 8 B) come
 * back to the host, which maps the regions. The app must have <= 32 types
 * (VF_ERR_TOO_MANY_TYPES); a type id >= ntypes -> VF_ERR_INVALID. Synchronises
 * `stream`; the range table is republished as a NEW device version (kernels
 * still running on other streams keep reading the old one, which is freed at
 * vf_reset / vf_destroy). */
vf_status vf_alloc_typed_batch(vf_ctx* ctx, uint32_t app, const uint32_t* type_ids_dev,
                               uint64_t count, const void* ctor_args_dev,
                               uint32_t ctor_arg_bytes, uint64_t* out_ptrs_dev, int tag,
                               void* stream);
/* cuda_packed (SURVEY §7 "A fair CUDA baseline", a sensitivity point for the
 * CUDA baseline): object i of class (app, type_ids_dev[i]) is placement-new'd
 * at slab + i * stride of ONE cudaMalloc'd index-ordered slab (stride = the
 * app's largest object rounded to 16 B): embedded vTable*, no type grouping,
 * no heap scatter. Dispatch it with VF_CUDA. Not in the range table. Freed at
 * vf_reset / vf_destroy. */
vf_status vf_alloc_packed(vf_ctx* ctx, uint32_t app, const uint32_t* type_ids_dev, uint64_t count,
                          const void* ctor_args_dev, uint32_t ctor_arg_bytes, uint64_t* out_ptrs_dev,
                          void* stream);
/* CUDA baseline: device-heap `new` of class (app, type_ids_dev[i]) per object
 * in a kernel. tag = 1 additionally tags the
 * returned pointers (TypePointer on the default CUDA allocator, §8.2
 * P:2749-2757); such objects are NOT in the range table. */
vf_status vf_alloc_cuda(vf_ctx* ctx, uint32_t app, const uint32_t* type_ids_dev, uint64_t count,
                        const void* ctor_args_dev, uint32_t ctor_arg_bytes,
                        uint64_t* out_ptrs_dev, int tag, void* stream);
/* Drop every object (arenas unmapped, device-heap objects deleted); VA
 * reservations are kept. Synchronises the device. */
vf_status vf_reset(vf_ctx* ctx);

/* Sorted, disjoint, merged range table of `app` (app = 0xFFFFFFFF: all
 * apps). Host view owned by ctx, valid until the next alloc / reset. */
vf_status vf_range_table(const vf_ctx* ctx, uint32_t app, const vf_range** out, uint32_t* n);
/* Raw regions in creation order (owned by ctx, same lifetime). */
vf_status vf_regions(const vf_ctx* ctx, const vf_region** out, uint32_t* n);
/* Device vTable* of each concrete type of `app` (ntypes entries, host array). */
vf_status vf_type_vptrs(vf_ctx* ctx, uint32_t app, uint64_t* vptrs_out);

/* ---- resolution / verification ---------------------------------------- */
/* types_out_dev[i] = type id of ptrs_dev[i] under the variant's rule
 * (CUDA/SHAREDOA: embedded vTable* -> type; COAL: range lookup; TYPEPTR:
 * tag); VF_NOT_FOUND if unresolved (the dispatch kernels fall back to the
 * embedded vTable* for those) or if the pointer is null. */
vf_status vf_resolve(vf_ctx* ctx, uint32_t app, vf_variant v, const uint64_t* ptrs_dev,
                     uint64_t n, uint32_t* types_out_dev, void* stream);
/* Brute-force type identity: counts pointers whose variant-resolved type's
 * vTable* differs from the vTable* embedded in the object (or that fail to
 * resolve). Adds the count to *mismatches_dev (u64, device). */
vf_status vf_verify_types(vf_ctx* ctx, uint32_t app, vf_variant v, const uint64_t* ptrs_dev,
                          uint64_t n, unsigned long long* mismatches_dev, void* stream);

/* ---- dispatch: one call of virtual method `method` on every objs_dev[i],
 * i in [0, n); null entries are skipped. `args` is a host pointer to the
 * method's argument struct (args_bytes <= VF_MAX_ARGS_BYTES), copied into
 * the kernel parameters. Pointers must be unique for mutating methods.
 * CUDA / SHAREDOA: plain C++ virtual call (vTable* load, vFunc* load,
 * indirect CALL) on the pointer as given — it must be untagged (a tagged
 * pointer faults there, as any invalid pointer does in C++). COAL: range
 * lookup (the kernel-parameter table for K <= 8 rows, else shared memory) of
 * the pointer's address (a tag, if present, is stripped first). TYPEPTR:
 * tag shift + strip. COAL and TYPEPTR then group the lanes of a warp by type
 * and run each type's body once per warp as a direct, inlined call; a
 * pointer neither rule types (COAL miss, tag 0) falls back to its embedded
 * vTable*. vf_resolve / vf_verify_types strip tags before any dereference. */
vf_status vf_dispatch_cuda(vf_ctx* ctx, uint32_t app, uint32_t method, const uint64_t* objs_dev,
                           uint64_t n, const void* args, size_t args_bytes, void* stream);
vf_status vf_dispatch_sharedoa(vf_ctx* ctx, uint32_t app, uint32_t method,
                               const uint64_t* objs_dev, uint64_t n, const void* args,
                               size_t args_bytes, void* stream);
vf_status vf_dispatch_coal(vf_ctx* ctx, uint32_t app, uint32_t method, const uint64_t* objs_dev,
                           uint64_t n, const void* args, size_t args_bytes, void* stream);
vf_status vf_dispatch_typeptr(vf_ctx* ctx, uint32_t app, uint32_t method,
                              const uint64_t* objs_dev, uint64_t n, const void* args,
                              size_t args_bytes, void* stream);
/* Concord (embedded type tag + switch, one object per thread). */
vf_status vf_dispatch_concord(vf_ctx* ctx, uint32_t app, uint32_t method, const uint64_t* objs_dev,
                              uint64_t n, const void* args, size_t args_bytes, void* stream);
/* Same, variant as a parameter. */
vf_status vf_dispatch(vf_ctx* ctx, vf_variant v, uint32_t app, uint32_t method,
                      const uint64_t* objs_dev, uint64_t n, const void* args, size_t args_bytes,
                      void* stream);
/* Dispatch from a HOST pointer array (the end-to-end path): objs_host (n
 * pointers; pinned memory for full PCIe bandwidth) is copied in chunks of
 * `chunk` pointers (0 = 2^22) into staging_dev (caller-owned device buffer of
 * n u64) on a ctx-internal copy stream, and every chunk is dispatched on
 * `stream` as soon as its copy has landed, so the transfer overlaps the
 * calls. Same semantics as vf_dispatch over the copied array. Asynchronous:
 * objs_host must stay valid and unchanged until `stream` has passed this
 * call; staging_dev is overwritten only after earlier work on `stream`. */
vf_status vf_dispatch_host(vf_ctx* ctx, vf_variant v, uint32_t app, uint32_t method, const uint64_t* objs_host,
                           uint64_t n, const void* args, size_t args_bytes, uint64_t* staging_dev, uint64_t chunk,
                           void* stream);

/* ---- app helpers (non-virtual phases) ---------------------------------- */
/* GOL / GEN step (1): nbr_dev[c] = neighbours of cell c whose state is 1
 * (alive) in state_dev (W x H, dead border, or torus if torus != 0). */
vf_status vf_gol_neighbors(uint32_t W, uint32_t H, int torus, const uint8_t* state_dev,
                           uint8_t* nbr_dev, void* stream);
/* GOL step (3): where state_next != state_prev, swap grid_dev[c] between
 * alive_dev[c] and dead_dev[c] and reset the new object's counter. */
vf_status vf_gol_swap(vf_ctx* ctx, uint64_t ncells, const uint8_t* state_prev_dev,
                      const uint8_t* state_next_dev, uint64_t* grid_dev,
                      const uint64_t* alive_dev, const uint64_t* dead_dev, void* stream);
/* GEN step (3): where the type of state_next differs from state_prev's, point
 * grid_dev[c] at the cell's Dead / Alive / Dying object, reset its counter and
 * (Dying) set its stage to the new state. */
vf_status vf_gen_swap(vf_ctx* ctx, uint64_t ncells, const uint8_t* state_prev_dev,
                      const uint8_t* state_next_dev, uint64_t* grid_dev, const uint64_t* dead_dev,
                      const uint64_t* alive_dev, const uint64_t* dying_dev, void* stream);

/* Fused generation (B200 design): steps (1) neighbours, (2) one
 * virtual next() per cell under variant v, (3) swap, done per cell by ONE
 * thread in ONE launch — identical results to vf_gol_neighbors + vf_dispatch
 * (VF_GOL_NEXT, args {nbr_dev, next_dev}) + vf_gol_swap. grid_dev[c] must be
 * cell c's current object (its own cell field = c). */
vf_status vf_gol_step(vf_ctx* ctx, vf_variant v, uint32_t W, uint32_t H, int torus, const uint8_t* state_prev_dev,
                      uint8_t* state_next_dev, uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* alive_dev,
                      const uint64_t* dead_dev, void* stream);
/* `gens` generations of vf_gol_step in ONE cooperative launch (config 1 is
 * launch-latency bound: a 256 x 256 generation is a few microseconds of
 * work). Generation g reads state[g & 1] and writes state[(g + 1) & 1]
 * (state0 = the current state; after the call the current state is
 * state[gens & 1]); generations are separated by a grid barrier on
 * *barrier_dev (caller-owned u32, zeroed by the call on `stream`), or, for
 * grids of <= 2^17 cells, the launch is ONE thread-block cluster of up to 16
 * CTAs that keeps the state rows in distributed shared memory and separates
 * generations with the hardware cluster barrier (tuning key "cluster", off
 * by default). Every
 * variant runs the same structure; results are identical to `gens` calls of
 * vf_gol_step. VF_ERR_CUDA if the grid cannot be co-resident. */
vf_status vf_gol_run(vf_ctx* ctx, vf_variant v, uint32_t W, uint32_t H, int torus, uint8_t* state0_dev,
                     uint8_t* state1_dev, uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* alive_dev,
                     const uint64_t* dead_dev, uint32_t gens, uint32_t* barrier_dev, void* stream);
/* Same for GEN (VF_GEN_NEXT with {nbr, next, born_mask, survive_mask, C}, then vf_gen_swap). */
vf_status vf_gen_step(vf_ctx* ctx, vf_variant v, uint32_t W, uint32_t H, int torus, const uint8_t* state_prev_dev,
                      uint8_t* state_next_dev, uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* dead_dev,
                      const uint64_t* alive_dev, const uint64_t* dying_dev, uint32_t born_mask,
                      uint32_t survive_mask, uint32_t C, void* stream);
/* The same generation restricted to the row slab [row0, row0 + nrows) (multi-GPU
 * row slabs): neighbours of the slab's cells are read from
 * state_prev rows row0-1 and row0+nrows (the halo rows, torus-wrapped when
 * torus != 0), which the caller keeps current; only the slab's cells (and their
 * grid_dev / nbr_dev / state_next_dev entries and objects) are touched. W*H <
 * 2^32. VF_ERR_INVALID if the slab leaves [0, H). vf_gen_step = rows [0, H). */
vf_status vf_gen_step_rows(vf_ctx* ctx, vf_variant v, uint32_t W, uint32_t H, int torus, uint32_t row0,
                           uint32_t nrows, const uint8_t* state_prev_dev, uint8_t* state_next_dev,
                           uint8_t* nbr_dev, uint64_t* grid_dev, const uint64_t* dead_dev, const uint64_t* alive_dev,
                           const uint64_t* dying_dev, uint32_t born_mask, uint32_t survive_mask, uint32_t C,
                           void* stream);

/* Config 3 ray tracer (readings G24, G25): render rows [row0, row0+nrows) of
 * a W x H image over S shapes of VF_APP_RAY (type ids 0 Plane, 1 Sphere,
 * 2 Rect, 3 Triangle; constructor argument = 12 fp32 params, see
 * synth.ray_scene). Per pixel: one primary ray through the pixel centre, one
 * virtual hit() per shape in ascending id (CUDA / SHAREDOA: virtual call;
 * COAL / TYPEPTR: type from the pointer, direct inlined call), closest
 * t > 1e-4 with ties to the smaller id, Lambert shading with 0.1 ambient.
 * cam (host, 5 floats) = {tan(fov/2)*W/H, tan(fov/2), unit light xyz};
 * albedo (host, 12 floats) = rgb per type. Writes rgb_dev[nrows*W*3] (fp32)
 * and hit_dev[nrows*W] (shape id or -1). Bit-identical to the CPU oracle. */
vf_status vf_ray_render(vf_ctx* ctx, vf_variant v, const uint64_t* shapes_dev, uint32_t S, uint32_t W,
                        uint32_t H, uint32_t row0, uint32_t nrows, const float* cam, const float* albedo,
                        float* rgb_dev, int32_t* hit_dev, void* stream);

/* Collision step (0), non-virtual: the uniform grid and the dispatch order.
 * For every body i with P[i].w > 0: cell (clamp(floor(x/rc)), clamp(floor(y/rc)),
 * clamp(floor(z/rc))) of a G^3 grid, c = (z*G + y)*G + x; cell_start = the
 * exclusive prefix sum of the cell counts; list[cell_start[c] ..) = the ids of
 * cell c ascending; Ps[e] = P[list[e]]; slot[list[e]] = e. Then order[k] = the objects of the
 * owned ids [id_lo, id_hi) that are active, in cell order (spatially
 * neighbouring bodies share a warp), null-padded to id_hi - id_lo entries
 * (null pointers are skipped by every dispatch variant). *active_dev (if not
 * NULL) += the number of owned active bodies (call accounting).
 * Buffers are device memory owned by the caller; cell_count_dev must be all
 * zero on entry and is left all zero; tmp_dev holds vf_collide_tmp_words(N, G)
 * u32. 1 <= G <= 1024; VF_ERR_INVALID otherwise. */
typedef struct {
  uint32_t N, G;
  float rc;
  const float4_t* P_dev;          /* N                                          */
  uint32_t* cell_of_dev;          /* N (0xFFFFFFFF = inactive)                  */
  uint32_t* cell_count_dev;       /* G^3, zero on entry and on return           */
  uint32_t* cell_start_dev;       /* G^3 + 1                                    */
  uint32_t* list_dev;             /* N                                          */
  float4_t* Ps_dev;               /* N                                          */
  uint32_t* slot_dev;             /* N (entries of inactive bodies untouched)   */
  uint32_t* tmp_dev;              /* vf_collide_tmp_words(N, G)                 */
  const uint64_t* objs_dev;       /* id_hi - id_lo: object of body id_lo + k     */
  uint32_t id_lo, id_hi;
  uint64_t* order_dev;            /* id_hi - id_lo                              */
  unsigned long long* active_dev; /* may be NULL                                */
} vf_collide_grid_args;
uint64_t vf_collide_tmp_words(uint32_t N, uint32_t G);
vf_status vf_collide_grid(const vf_collide_grid_args* args, void* stream);
/* Multi-GPU exchange after update. merge() of body i reads near,
 * Pm, Vm of j = near[i] only when near[j] >= 0, so a rank owning bodies
 * [lo, hi) packs just those with near >= 0 (vf_collide_pack_near: appends
 * entries to out_dev at *count_dev, order unspecified), the packed lists are
 * all-gathered (rank r's segment of `seg` entries holds counts_dev[r] valid
 * ones), and vf_collide_unpack_near resets near[] of every body outside
 * [lo, hi) to -1 and then writes the received entries (own ones skipped). */
typedef struct {
  uint32_t id;
  int32_t near;
  uint32_t pad[2];
  float Pm[4]; /* post-update position + mass */
  float Vm[4]; /* post-update velocity        */
} vf_collide_near_entry;
vf_status vf_collide_pack_near(uint32_t lo, uint32_t hi, const int32_t* near_dev, const float* Pm_dev,
                               const float* Vm_dev, vf_collide_near_entry* out_dev, uint32_t* count_dev,
                               void* stream);
vf_status vf_collide_unpack_near(const vf_collide_near_entry* in_dev, uint32_t nseg, uint32_t seg,
                                 const int64_t* counts_dev, uint32_t N, uint32_t lo, uint32_t hi,
                                 int32_t* near_dev, float* Pm_dev, float* Vm_dev, void* stream);

/* Graph helpers: BFS start state (depth = -1 except depth[src] = 0, queue =
 * src's nch work entries (vobj[src], chunks 0..nch-1), *count = nch), iota
 * (x[i] = i), fill (x[i] = value). */
vf_status vf_graph_bfs_init(uint64_t V, int32_t* depth_dev, uint32_t src, const uint64_t* vobj_dev,
                            const uint64_t* offs_dev, uint32_t C, uint64_t* queue_dev,
                            uint32_t* queue_chunk_dev, uint32_t* count_dev, void* stream);
vf_status vf_iota_u32(uint64_t n, uint32_t* x_dev, void* stream);
vf_status vf_fill_f32(uint64_t n, float* x_dev, float value, void* stream);

/* BRANCH ceiling of the microbenchmark (§8.3: "decides which
 * function to call based on register values and does not access memory for
 * the function call"): no objects; for i in [0, n): t = the type config 2
 * gives object i, computed in registers from (seed, order, T, k) with the
 * synth recipe (order 0 random: t = floor(splitmix64(seed ^ 1<<56 ^ i) * T /
 * 2^64); 1 sorted: floor(i*T/n); 2 k-per-warp: (i mod 32) mod k); then a
 * switch on t adds t+1 to vals_dev[i] (int32). */
vf_status vf_micro_branch(uint64_t n, uint32_t T, int order, uint64_t seed, uint32_t k, int32_t* vals_dev,
                          void* stream);

/* ---- utilities ---------------------------------------------------------- */
/* sum over i of vals_dev[i] (int32, widened) into *out_dev (i64, device). */
vf_status vf_checksum_i32(const int32_t* vals_dev, uint64_t n, long long* out_dev, void* stream);
/* Benchmark / ablation knobs of the COAL / TYPEPTR kernels (process-wide):
 * "unroll" = objects per thread (1, 2, 4; -1 = app default); "prefetch" =
 * object-line warm-up before the type groups (0 none, 1 prefetch.global.L1,
 * 2 L1-allocating load, 3 = 2 issued one tile ahead with the pointers two
 * tiles ahead (sorted kernel); -1 = app default); "regroup" = 1 (default) sorts
 * each CTA tile by type in shared memory before the calls (4 barriers per
 * tile), 2 the same sort with 2 barriers per tile (double-buffered histogram
 * that every warp scans; light methods, prefetch 2), 0 groups within warps
 * only; "pipeline" = 1 streams the pointer array through a TMA /
 * mbarrier ring in shared memory (regroup 0 only), 0 (default) uses plain
 * per-thread loads; "call" = 1 makes COAL / TYPEPTR CALL the resolved type's
 * vFunc* indirectly (the paper's design, Table 1 row C, Fig. 5b line 4), 0
 * (default) groups lanes by type and calls each body directly;
 * "persistent" = 1 runs the grouped kernels on a persistent grid (CTAs loop
 * over tiles), 0 gives every CTA one tile, -1 (default) = persistent except
 * for the app methods marked heavy (long bodies of varying length: collision
 * and N-body update, graph methods); "cluster" = 1 lets vf_gol_run run
 * grids of <= 2^17 cells in ONE thread-block cluster (state in distributed
 * shared memory, hardware cluster barrier), 0 (default; measured faster on
 * B200: a 16-SM cluster serialises 4 cells per thread) always uses the
 * cooperative grid-barrier kernel; "ray_rays" = 4 (default) or 2: pixels
 * (rays) per thread in both ray-tracer kernels; "gsort" = 1 sorts the whole
 * dispatch list of a heavy method (long bodies: N-body / collision update,
 * graph methods) by type before the calls under COAL / TYPEPTR (type from
 * the pointer; (pointer, index) pairs, index order kept within a type; the
 * body still receives the entry's original index), 0 sorts per CTA tile
 * only, -1 (default) = the app's choice (N-body and collision sort the list;
 * the graph methods, measured no faster, do not); "coal_inline" = the largest
 * COAL table (rows, 0..8, default 8) tested from the kernel parameters rather
 * than searched in shared memory.
 * The unroll / prefetch / pipeline knobs apply to config 2's app (micro);
 * the other apps run their default launch configuration.
 * VF_ERR_INVALID for unknown keys / values. */
vf_status vf_set_tuning(const char* key, int value);
/* Number of libvf kernel launches issued since load (for bench accounting). */
uint64_t vf_launch_count(void);

/* Strip a TypePointer tag (restore the upper bits before any
 * field access). Host-side helper; the kernels do the same with one LOP3. */
static inline uint64_t vf_strip(uint64_t p) { return p & ((1ull << VF_VA_BITS) - 1); }

#ifdef __cplusplus
}
#endif
#endif
