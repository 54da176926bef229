"""Parity at the BASELINE.json config sizes, in the launch configuration bench.py times.

Every app of configs 4 and 5 runs here at its full size against the CPU oracle
run on the same full input (no sampling: the oracle finishes each in seconds to
a minute on the box's cores):
  graph  RMAT-24 (V = 16.8M, 520.8M arcs): BFS depths and CC labels exact on
         every vertex, PageRank (10 iterations) 1e-5 relative on every vertex
  TRAF   3,277 rings x 4,096 cells, 100 steps: every vehicle's position and
         speed exact
  STUT   2048 x 2048 nodes + 12.6M springs, 100 steps: positions bit-exact,
         broken set exact
  GEN    4096 x 4096, 100 generations: state and per-cell counters exact
  N-body 65,536 bodies, 2 steps: positions and velocities bit-exact (the
         oracle's all-pairs step is ~1 min of host time at this size; longer
         trajectories are covered at 4,429 bodies in test_gpu_nbody.py)
(config 2 at 2^26 objects: test_gpu_micro.py; collision at 16M bodies:
test_gpu_collide.py; the ray tracer's full frame: test_gpu_ray.py.)
The persistent grouped kernels cover each of these inputs in many waves
(asserted: > 2 x 148 SMs x 16 CTAs x 1024 objects), so their grid-stride wrap
and the next-tile pointer prefetch run.
"""
import numpy as np
import pytest
import torch

import oracle
import synth
from paper_conf_asplos_zhangar21_b200 import apps, vf

pytestmark = [pytest.mark.gpu, pytest.mark.slow]
WAVE = 148 * 16 * 1024  # SMs x max resident CTAs x max objects per CTA tile
VARIANTS = ["cuda", "cuda_packed", "sharedoa", "coal", "typeptr"]


@pytest.fixture(scope="module")
def ctx():
    c = vf.Ctx(0, cuda_heap_bytes=16 << 30)
    yield c
    c.close()


def _free(ctx):
    torch.cuda.synchronize()
    ctx.reset()
    torch.cuda.empty_cache()


@pytest.fixture(scope="module")
def rmat24():
    offs, col = synth.rmat_graph(24, seed=1)
    types = synth.vertex_types(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    thr = oracle.max_threads()
    depth, levels, _, _ = oracle.graph_bfs(offs, col, types, src)
    label, iters, _, _ = oracle.graph_cc(offs, col, types, threads=thr)
    rank, _ = oracle.graph_pr(offs, col, types, iters=10, threads=thr)
    return dict(offs=offs, col=col, src=src, depth=depth, levels=levels, label=label, iters=iters, rank=rank)


@pytest.mark.parametrize("variant", VARIANTS)
def test_graph_rmat24(ctx, rmat24, variant):
    from paper_conf_asplos_zhangar21_b200.graph import Graph
    g = Graph(ctx, rmat24["offs"], rmat24["col"], variant)
    for mode in ("hybrid", "topdown", "bits"):
        depth, levels, _ = g.bfs(rmat24["src"], mode=mode)
        assert np.array_equal(depth.cpu().numpy(), rmat24["depth"]), mode
        assert levels == rmat24["levels"]
    lab, iters, _ = g.cc()
    assert np.array_equal(lab.cpu().numpy().view(np.uint32), rmat24["label"]) and iters == rmat24["iters"]
    r, _ = g.pagerank(10)
    np.testing.assert_allclose(r.cpu().numpy(), rmat24["rank"], rtol=1e-5, atol=0)
    if variant != "cuda_packed":
        assert ctx.verify(vf.APP_GRAPH, g.v, g.owned) == 0
    del g
    _free(ctx)


@pytest.fixture(scope="module")
def traf_full():
    w = synth.traf_world(3277, 4096, seed=11)
    pos, v, _ = oracle.traf_run(w, 100, threads=oracle.max_threads())
    return w, pos, v


@pytest.mark.parametrize("variant", VARIANTS)
def test_traf_full(ctx, traf_full, variant):
    from paper_conf_asplos_zhangar21_b200.traf import Traf
    w, pos_ref, v_ref = traf_full
    t = Traf(ctx, w, variant)
    assert t.calls_per_step > 2 * WAVE
    for _ in range(100):
        t.step()
    pos, v = t.state()
    assert np.array_equal(pos, pos_ref) and np.array_equal(v, v_ref)
    del t
    _free(ctx)


@pytest.fixture(scope="module")
def stut_full():
    w = synth.stut_lattice(2048, 2048, seed=12, v_pull=4.0)
    pos, vel, br, _ = oracle.stut_run(w, 100, threads=oracle.max_threads())
    return w, pos, vel, br


@pytest.mark.parametrize("variant", VARIANTS)
def test_stut_full(ctx, stut_full, variant):
    from paper_conf_asplos_zhangar21_b200.stut import Stut
    w, pos_ref, vel_ref, br_ref = stut_full
    st = Stut(ctx, w, variant)
    assert st.calls_per_step > 2 * WAVE
    for _ in range(100):
        st.step()
    assert np.array_equal(st.positions().view(np.uint32), pos_ref.view(np.uint32))
    assert np.array_equal(st.velocities().view(np.uint32), vel_ref.view(np.uint32))
    assert np.array_equal(st.broken(), br_ref)
    del st
    _free(ctx)


@pytest.fixture(scope="module")
def gen_full():
    W = 4096
    s0 = synth.soup(W, W, seed=42)
    st, ctr, hist, _ = oracle.gen_run(W, W, s0, 100, threads=oracle.max_threads())
    return W, s0, st, ctr, hist


@pytest.mark.parametrize("variant", ["cuda_packed", "sharedoa", "coal", "typeptr"])
def test_gen_full(ctx, gen_full, variant):
    """(the device-heap arm runs GEN at 2048^2 in bench.py: test_gen_2048_heap)"""
    W, s0, st_ref, ctr_ref, hist_ref = gen_full
    g = apps.Gen(ctx, W, W, s0, variant)
    assert W * W > 2 * WAVE
    for _ in range(100):
        g.gen()
    st = g.current.cpu().numpy()
    assert np.array_equal(st, st_ref)
    ctr, _ = g.counters()
    assert np.array_equal(ctr.cpu().numpy().view(np.uint16), ctr_ref)
    assert list(np.bincount(st, minlength=4)) == list(hist_ref)
    del g
    _free(ctx)


def test_gen_2048_heap(ctx):
    W = 2048
    s0 = synth.soup(W, W, seed=42)
    st_ref, ctr_ref, _, _ = oracle.gen_run(W, W, s0, 50, threads=oracle.max_threads())
    g = apps.Gen(ctx, W, W, s0, "cuda")
    for _ in range(50):
        g.gen()
    assert np.array_equal(g.current.cpu().numpy(), st_ref)
    ctr, _ = g.counters()
    assert np.array_equal(ctr.cpu().numpy().view(np.uint16), ctr_ref)
    del g
    _free(ctx)


@pytest.fixture(scope="module")
def nbody_full():
    s = synth.nbody_system(65536, seed=10)
    p, v, _ = oracle.nbody_run(s, 2, threads=oracle.max_threads())
    return s, p, v


@pytest.mark.parametrize("variant", VARIANTS)
def test_nbody_full(ctx, nbody_full, variant):
    from paper_conf_asplos_zhangar21_b200.nbody import Nbody
    s, p_ref, v_ref = nbody_full
    nb = Nbody(ctx, s, variant)
    for _ in range(2):
        nb.step()
    assert np.array_equal(nb.positions().view(np.uint32), p_ref.view(np.uint32))
    assert np.array_equal(nb.velocities().view(np.uint32), v_ref.view(np.uint32))
    del nb
    _free(ctx)
