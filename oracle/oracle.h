/*
 * oracle.h — C ABI of the CPU ORACLE for "Judging a Type by Its Pointer:
 * Optimizing GPU Virtual Functions" (Zhang, Alawneh, Rogers, ASPLOS'21).
 *
 * TEST INFRASTRUCTURE ONLY. Only tests/, __graft_entry__.smoke() and
 * bench.py's cpu_baseline / --impl reference leg may load liboracle.so.
 * It shares no code, header, table or constant generator with the CUDA path
 * (paper_conf_asplos_zhangar21_b200/csrc, include/vf.h), and neither side
 * includes the other.
 *
 * Citations are P:<line> of /root/reference/PAPER.md (section / figure /
 * algorithm given alongside). Readings of silent or garbled passages are the
 * G-numbers listed in DESIGN.md §"Readings".
 *
 * Plain, slow, obviously-correct: ordinary C++ classes with `virtual`
 * methods, objects from plain `new`, one per object, in index order; loops in
 * the paper's order. OpenMP (threads>1) only splits independent per-object
 * loops; results are identical for any thread count (tested).
 */
#ifndef VF_ORACLE_H
#define VF_ORACLE_H
#include <stdint.h>
#ifdef __cplusplus
extern "C" {
#endif

#define ORACLE_NOT_FOUND 0xFFFFFFFFu

/* ---- Allocator region policy (§4; §5) ------------
 * Capacities (in objects) of the regions SharedOA creates for one type when
 * `count` objects are allocated: r0 = init_chunk, r_{j+1} = 2 r_j, until the
 * sum reaches count. Returns the number of regions (0 if count == 0), writes
 * at most max_out capacities. */
uint32_t oracle_region_plan(uint64_t count, uint64_t init_chunk,
                            uint64_t* caps_out, uint32_t max_out);

/* ---- Virtual range table (Fig. 3) --------------
 * Build the table from raw regions [start_i, start_i + bytes_i) of type
 * type_i: sort by start, merge a region into its predecessor when it is of
 * the same type and exactly adjacent. Writes K <= n rows
 * (start, end, type); returns K. */
uint32_t oracle_build_table(const uint64_t* start, const uint64_t* bytes,
                            const uint32_t* type, uint32_t n,
                            uint64_t* t_start, uint64_t* t_end, uint32_t* t_type);

/* ---- COAL ObjectRangeLookup (Algorithm 1) ----
 * Balanced segment tree over the K sorted disjoint ranges (leaves = ranges,
 * internal nodes = [min start, max end) of their children), descended from
 * the root; returns the type of the leaf whose [start,end) contains addr,
 * else ORACLE_NOT_FOUND (Alg. 1 "return NULL"). Reading G5. */
void oracle_coal_lookup(const uint64_t* t_start, const uint64_t* t_end,
                        const uint32_t* t_type, uint32_t K,
                        const uint64_t* addrs, uint64_t n, uint32_t* out_type);

/* ---- TypePointer (Fig. 5; §6.1; §6.3)
 * B200 format (reading G6): 7-bit tag in bits 63:57 above the 57-bit VA;
 * tag = type+1 (0 = untagged). Pattern of the upper bits = 0 (reading G7). */
uint64_t oracle_tp_tag(uint64_t addr, uint32_t type);
uint32_t oracle_tp_type(uint64_t tagged);     /* ORACLE_NOT_FOUND if untagged */
uint64_t oracle_tp_strip(uint64_t tagged);
/* Fig. 5b with the padded-index form:
 * vFunc = vtables[type(q) * vtable_slots + func_index]. */
uint64_t oracle_tp_vfunc(uint64_t tagged, const uint64_t* vtables,
                         uint32_t vtable_slots, uint32_t func_index);

/* ---- Config 2 microbenchmark (§8.3) ------------------------
 * n objects; object i is of class MObj<types[i]> (types[i] < T <= 32) with
 * val = init[i]; `reps` passes of `for i: objs[i]->apply()` where
 * MObj<k>::apply() { val += k + 1; } ("simple addition").
 * out_vals[i] = final val. *seconds = wall time of the dispatch passes only.
 * threads = OpenMP threads over i (1 = the reference semantics). */
int oracle_micro_run(uint64_t n, uint32_t T, const uint32_t* types,
                     const int32_t* init, uint32_t reps, int threads,
                     int32_t* out_vals, double* seconds);

/* ---- Config 1 Game of Life (Table 2; readings G12-G14) -----
 * Grid W x H, cell c = y*W + x. Each cell owns one Alive and one Dead
 * object; grid[c] points at the one matching its state. Per generation:
 *  (1) n[c] = live neighbours among 8 in the previous state (dead border,
 *      or torus if torus != 0);
 *  (2) s' = grid[c]->next(n[c])  (virtual; Alive: n==2||n==3, Dead: n==3;
 *      both increment their own counter: age / dead_for);
 *  (3) if s' != s: grid[c] = the other object, whose counter is reset to 0.
 * Outputs: final state (uint8), final counter of each cell's current object,
 * population after every generation pop[g], g = 0..gens-1.
 * *seconds = wall time of the generation loop. */
int oracle_gol_run(uint32_t W, uint32_t H, const uint8_t* init_alive,
                   uint32_t gens, int torus, int threads,
                   uint8_t* out_state, uint16_t* out_counter, uint32_t* pop,
                   double* seconds);

/* ---- Config 5 Generation (Table 2; reading G15) ------------
 * Generations CA B/S/C: states 0 dead, 1 alive, 2..C-1 dying. born_mask /
 * survive_mask bit n = rule holds with n live (state-1) neighbours. Per
 * generation: n[c] from the previous state (dead border / torus), one virtual
 * next() per cell (Dead: born? 1 : 0; Alive: survive? 1 : (C>2 ? 2 : 0);
 * Dying(s): s+1 < C ? s+1 : 0), pointer swap on a type change. hist[k] =
 * cells in state k at the end (C entries). */
int oracle_gen_run(uint32_t W, uint32_t H, const uint8_t* init_state, uint32_t gens,
                   uint32_t born_mask, uint32_t survive_mask, uint32_t C, int torus,
                   int threads, uint8_t* out_state, uint16_t* out_counter, uint32_t* hist,
                   double* seconds);

/* ---- Config 4 graph apps over polymorphic vertices (Table 2 P:1538-1588;
 * readings G20-G23). CSR offs[V+1] / col[arcs] (symmetric), types[v] in
 * {0 Leaf, 1 Low, 2 Mid, 3 Hub}; one object per vertex from plain `new`.
 * BFS: level-synchronous from src, one virtual bfs_expand() per frontier
 *   vertex; depth[v] = level or -1; *levels = levels visited (incl. the
 *   empty last), *calls = sum of frontier sizes.
 * CC: Jacobi min-label propagation from label = id until no change, one
 *   virtual cc_update() per vertex per iteration (*iters incl. the final
 *   no-change pass).
 * PR: r0 = 1/V; per iteration c_u = deg ? r_u/deg : 0 (fp64), D = sum of r
 *   over deg-0 vertices (fp64, vertex order), s_v = virtual pr_gather() =
 *   sum over N(v) of c_u in CSR order (fp64), r_v' = (float)((1-d)/V +
 *   d*(s_v + D/V)). */
int oracle_graph_bfs(uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* types,
                     uint32_t src, int32_t* depth, uint32_t* levels, uint64_t* calls,
                     double* seconds);
int oracle_graph_cc(uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* types,
                    int threads, uint32_t* label, uint32_t* iters, uint64_t* calls, double* seconds);
int oracle_graph_pr(uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* types,
                    double d, uint32_t iters, int threads, float* rank, double* seconds);

/* ---- GraphChi-vEN: virtual edges AND virtual vertices (Table 2
 * P:1566-1588; readings G32/G33). One edge object per arc
 * (u -> v) from plain `new` in arc order (ChiEdge / Edge / HubEdge: HubEdge
 * iff the source is a Hub, etypes[k] = 1), double-buffered value; per vertex
 * in-edge list (arcs (u -> v), ascending u) and out-edge list (own arcs).
 * BFS: as oracle_graph_bfs, each vertex visits its out-edges through the
 *   virtual target(); *vcalls = vertex calls, *ecalls = edge calls.
 * CC: edges start with their source's label; update(v): m = min(label_in[v],
 *   virtual get_label(b) over in-edges), label_out[v] = m, virtual
 *   set_label(1-b, m) on out-edges; until no change. Same labels as
 *   oracle_graph_cc.
 * PR: edges start with r0(u)/deg(u); update(v): s = sum of virtual get_pr(b)
 *   over in-edges (ascending u), r' = (float)((1-d)/V + d*(s + D/V)), virtual
 *   set_pr(1-b, r'/deg) on out-edges; D of the next iteration = sum of r'
 *   over deg-0 vertices in vertex order. Bit-identical to oracle_graph_pr. */
int oracle_graph_en_edge_types(uint64_t V, const uint64_t* offs, const uint32_t* vtypes, uint32_t* etypes);
int oracle_graph_en_bfs(uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* types,
                        uint32_t src, int32_t* depth, uint32_t* levels, uint64_t* vcalls,
                        uint64_t* ecalls, double* seconds);
int oracle_graph_en_cc(uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* types,
                       uint32_t* label, uint32_t* iters, uint64_t* vcalls, uint64_t* ecalls,
                       double* seconds);
int oracle_graph_en_pr(uint64_t V, const uint64_t* offs, const uint32_t* col, const uint32_t* types,
                       double d, uint32_t iters, float* rank, double* seconds);

/* ---- Config 3 ray tracer over polymorphic shapes (Table 2 RAY P:1592-1600;
 * readings G24, G25). Shapes j = 0..S-1 of type types[j] (0 Plane y=h,
 * 1 Sphere, 2 axis-aligned Rect, 3 Triangle) with 12 fp32 params each
 * (params + 12 j). Rows [row0, row0+nrows) of a W x H image; per pixel one
 * primary ray, one virtual hit() per shape in ascending id, closest t > 1e-4
 * with strict '<' (ties -> smaller id), then one virtual normal() on the
 * winner; rgb = fmaf(albedo[kind], max(0, n.l), 0.1), black and id -1 on a
 * miss. cam = {tan(fov/2)*W/H, tan(fov/2), lx, ly, lz}. *calls = nrows*W*S. */
int oracle_ray_render(uint32_t W, uint32_t H, uint32_t row0, uint32_t nrows, uint32_t S,
                      const uint32_t* types, const float* params, const float* cam,
                      const float* albedo, int threads, float* rgb, int32_t* hit_id,
                      uint64_t* calls, double* seconds);

/* ---- Config 5 TRAF: Nagel-Schreckenberg rings (Table 2 P:1513-1516;
 * reading G16). R rings x L cells; cell c (global ring*L + pos) is a
 * LightCell if light[c] (phase[c]) else a PlainCell; vehicle i of type
 * veh_type[i] (0 Car, 1 Truck, 2 Bus; vmax[], slow_thr[] per type) starts at
 * (veh_ring[i], veh_pos[i]) with v = 0. Per step t: virtual update(t) per
 * cell (blocked = light red: (t+phase) mod 20 < 8), then virtual step() per
 * vehicle against the previous occupancy (see traf.cpp), occupancy rebuilt.
 * Writes final pos_out / v_out per vehicle. Returns 2 if two vehicles share
 * a starting cell. */
int oracle_traf_run(uint32_t R, uint32_t L, uint32_t nveh, const uint32_t* veh_ring,
                    const uint32_t* veh_pos, const uint32_t* veh_type, const uint8_t* light,
                    const uint32_t* phase, uint32_t steps, uint64_t seed, const uint32_t* vmax,
                    const uint32_t* slow_thr, int threads, uint32_t* pos_out, uint32_t* v_out,
                    double* seconds);

/* ---- Config 5 all-pairs N-body (reading G18; see nbody.cpp) -------------
 * N bodies, types[i] in {0 Star, 1 Planet, 2 Dust}, pos4 = N x (x,y,z,m),
 * vel3 = N x (vx,vy,vz); per step one virtual update() per body (softening
 * eps2[type], Dust damped by `damp`), semi-implicit Euler with dt; outputs
 * final positions (N x 4) and velocities (N x 3). */
int oracle_nbody_run(uint32_t N, const uint32_t* types, const float* pos4, const float* vel3,
                     uint32_t steps, float dt, const float* eps2, float damp, int threads,
                     float* pos_out, float* vel_out, double* seconds);

/* ---- Config 5 STUT spring-node structure (reading G17; see stut.cpp) ----
 * n nodes (types 0 Node, 1 AnchorNode, 2 AnchorPullNode; pos2 / vel2 = n x 2,
 * mass), S springs (sa, sb, rest L0, stiffness k), incidence CSR (inc_offs[n+1],
 * inc = (spring << 1) | is_b_end, ascending spring id per node). Per step: a
 * virtual force() per spring, then a virtual move() per node. Outputs final
 * positions / velocities (n x 2) and the broken flag per spring. */
int oracle_stut_run(uint32_t n, const uint32_t* types, const float* pos2, const float* vel2,
                    const float* mass, uint32_t S, const uint32_t* sa, const uint32_t* sb,
                    const float* L0, const float* k, const uint32_t* inc_offs, const uint32_t* inc,
                    uint32_t steps, float dt, float c, float v_pull, float brk, int threads,
                    float* pos_out, float* vel_out, uint8_t* broken_out, double* seconds);

/* ---- Config 5 collision (readings G18/G19; see collide.cpp) --------------
 * N bodies (types 0 Star, 1 Planet, 2 Dust; pos4 = x,y,z,m with m = 0 meaning
 * inactive; vel4 = vx,vy,vz,unused) on a G^3 grid of cells of side rc:
 * per step one virtual update() (cutoff rc softened gravity, nearest body
 * within rm) and one virtual merge() (mutual nearest pairs: the smaller id
 * absorbs the larger) per active body. calls_out = virtual calls issued. */
int oracle_collide_run(uint32_t N, const uint32_t* types, const float* pos4, const float* vel4,
                       uint32_t steps, uint32_t G, float rc, float rm, float dt, const float* eps2,
                       float damp, int threads, float* pos_out, float* vel_out, uint64_t* calls_out,
                       double* seconds);

/* number of OpenMP threads actually available */
int oracle_max_threads(void);

#ifdef __cplusplus
}
#endif
#endif
