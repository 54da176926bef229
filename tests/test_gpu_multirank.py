"""The multi-GPU data plane run through a REAL process
group with libvf's kernels on the GPU, against the unsharded CPU oracle.

Two processes, world_size 2, `gloo` over 127.0.0.1, both ranks on cuda:0
(this box has one GPU; NCCL refuses two ranks on one device, so the exchange
module stages the owned blocks through pinned host memory — the same
exchange code, BlockArray / HaloRows / allreduce_, that runs over NCCL on a
multi-GPU node). Every app that exchanges state runs its sharded step loop
with exchange on:
  graph    BFS over frontier bitmaps (bottom-up probes + all-gather of the
           bitmap slices), CC (label slices), PageRank (contribution slices +
           dangling all-reduce): depth / labels exact, ranks 1e-5
  N-body   id blocks, all-gather of the new positions: bit-exact
  STUT     node row slabs + ghost springs, all-gather of positions: bit-exact
  GEN      row slabs with halo rows (batch_isend_irecv), dead border and torus:
           state and counters bit-exact
  collide  id blocks, all-gather of Pm / Vm / near and P: bit-exact
  ray      8-row strips round-robin + gather_image: bit-exact frame
"""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch.multiprocessing as mp

import oracle
import synth

pytestmark = pytest.mark.gpu
WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, outdir, app, variant):
    import torch
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    from paper_conf_asplos_zhangar21_b200 import apps, vf
    ctx = vf.Ctx(0, cuda_heap_bytes=1 << 30)
    out = {}
    if app == "graph":
        from paper_conf_asplos_zhangar21_b200.graph import Graph
        offs, col = synth.rmat_graph(12, seed=4)
        src = int(np.argmax(np.diff(offs.astype(np.int64))))
        for C in (256, 7):
            g = Graph(ctx, offs, col, variant, rank=rank, world=world, chunk=C)
            depth, levels, _ = g.bfs(src)
            out[f"depth{C}"] = depth.cpu().numpy()
            out[f"levels{C}"] = np.array([levels])
            lab, it, _ = g.cc()
            out[f"label{C}"] = lab.cpu().numpy().view(np.uint32)
            out[f"iters{C}"] = np.array([it])
            r, _ = g.pagerank(20)
            out[f"rank{C}"] = r.cpu().numpy()
            out[f"lohi{C}"] = np.array([g.lo, g.hi])
    elif app == "nbody":
        from paper_conf_asplos_zhangar21_b200.nbody import Nbody
        s = synth.nbody_system(1111, seed=9)
        nb = Nbody(ctx, s, variant, rank, world)
        for _ in range(4):
            nb.step()
        out["pos"] = nb.positions()
        out["vel"] = nb.velocities()
        out["lohi"] = np.array([nb.lo, nb.hi])
    elif app == "stut":
        from paper_conf_asplos_zhangar21_b200.stut import Stut
        w = synth.stut_lattice(40, 23, seed=3, v_pull=5.0)
        st = Stut(ctx, w, variant, rank, world)
        for _ in range(30):
            st.step()
        out["pos"] = st.positions()
        out["vel"] = st.velocities()
        out["lohi"] = np.array([st.lo, st.hi])
        br = st.broken()
        own = st.spring_ids[(w["a"][st.spring_ids] >= st.lo) & (w["a"][st.spring_ids] < st.hi)]
        mask = np.zeros(len(w["a"]), np.uint8)
        mask[own] = 1
        out["broken"], out["own"] = br, mask
    elif app.startswith("gen"):
        torus = app == "gen_torus"
        W, H = 61, 37
        s0 = synth.soup(W, H, seed=42)
        g = apps.Gen(ctx, W, H, s0, variant, "2", "345", 4, torus, rank=rank, world=world)
        for _ in range(25):
            g.gen()
        out["state"] = g.current.cpu().numpy()
        ctr, typ = g.counters()
        out["ctr"] = ctr.cpu().numpy().view(np.uint16)
        out["lohi"] = np.array([g.lo, g.hi])
    elif app == "collide":
        from paper_conf_asplos_zhangar21_b200.collide import Collide
        s = synth.collide_system(3000, seed=11, rm=0.2)
        c = Collide(ctx, s, variant, rank, world)
        for _ in range(3):
            c.step()
        out["pos"] = c.positions()
        out["vel"] = c.velocities()
        out["lohi"] = np.array([c.lo, c.hi])
        out["calls"] = np.array([c.calls()])
    elif app == "ray":
        from paper_conf_asplos_zhangar21_b200.ray import Ray
        types, P = synth.ray_scene(40, seed=7)
        W, H = 48, 27
        cam = synth.ray_camera(W, H)
        r = Ray(ctx, types, P, variant)
        rgb, hid = r.render_frame(W, H, cam, rank, world)
        rgb, hid = Ray.gather_image(rgb, hid, world)
        out["rgb"], out["hid"] = rgb.cpu().numpy(), hid.cpu().numpy()
    torch.cuda.synchronize()
    np.savez(os.path.join(outdir, f"r{rank}.npz"), **out)
    ctx.close()
    dist.barrier()
    dist.destroy_process_group()


def _run(app, variant):
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_worker, args=(WORLD, _free_port(), td, app, variant), nprocs=WORLD, join=True)
        return [dict(np.load(os.path.join(td, f"r{r}.npz"))) for r in range(WORLD)]


@pytest.mark.parametrize("variant", ["cuda", "coal", "typeptr"])
def test_graph_world2(variant):
    res = _run("graph", variant)
    offs, col = synth.rmat_graph(12, seed=4)
    t = synth.vertex_types(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    depth, levels, _, _ = oracle.graph_bfs(offs, col, t, src)
    label, iters, _, _ = oracle.graph_cc(offs, col, t)
    rank, _ = oracle.graph_pr(offs, col, t, iters=20)
    for C in (256, 7):
        for r in res:  # every rank ends with the full state after the final gathers
            assert np.array_equal(r[f"depth{C}"], depth)
            assert int(r[f"levels{C}"][0]) == levels
            assert np.array_equal(r[f"label{C}"], label)
            assert int(r[f"iters{C}"][0]) == iters
            np.testing.assert_allclose(r[f"rank{C}"], rank, rtol=1e-5, atol=0)
        lo0, hi0 = res[0][f"lohi{C}"]
        lo1, hi1 = res[1][f"lohi{C}"]
        assert lo0 == 0 and hi0 == lo1 and hi1 == len(offs) - 1 and hi0 % 32 == 0


@pytest.mark.parametrize("variant", ["cuda", "sharedoa", "coal", "typeptr"])
def test_nbody_world2(variant):
    res = _run("nbody", variant)
    s = synth.nbody_system(1111, seed=9)
    p_ref, v_ref, _ = oracle.nbody_run(s, 4)
    for r in res:
        assert np.array_equal(r["pos"].view(np.uint32), p_ref.view(np.uint32))
    v = np.concatenate([r["vel"] for r in res])
    assert np.array_equal(v.view(np.uint32), v_ref.view(np.uint32))


@pytest.mark.parametrize("variant", ["cuda", "typeptr"])
def test_stut_world2(variant):
    res = _run("stut", variant)
    w = synth.stut_lattice(40, 23, seed=3, v_pull=5.0)
    pos_ref, vel_ref, br_ref, _ = oracle.stut_run(w, 30)
    for r in res:
        assert np.array_equal(r["pos"].view(np.uint32), pos_ref.view(np.uint32))
    assert np.array_equal(np.concatenate([r["vel"] for r in res]).view(np.uint32), vel_ref.view(np.uint32))
    br = np.zeros_like(br_ref)
    for r in res:
        br[r["own"] == 1] = r["broken"][r["own"] == 1]
    assert np.array_equal(br, br_ref)


@pytest.mark.parametrize("torus", [False, True])
@pytest.mark.parametrize("variant", ["cuda", "coal", "typeptr"])
def test_gen_row_slabs_world2(variant, torus):
    res = _run("gen_torus" if torus else "gen", variant)
    W, H = 61, 37
    s0 = synth.soup(W, H, seed=42)
    st_ref, ctr_ref, _, _ = oracle.gen_run(W, H, s0, 25, "2", "345", 4, torus)
    for r in res:
        lo, hi = r["lohi"]
        assert np.array_equal(r["state"][lo:hi], st_ref[lo:hi])
        assert np.array_equal(r["ctr"][lo:hi], ctr_ref[lo:hi])
    assert res[0]["lohi"][1] == res[1]["lohi"][0] and res[1]["lohi"][1] == W * H


@pytest.mark.parametrize("variant", ["cuda", "typeptr"])
def test_collide_world2(variant):
    res = _run("collide", variant)
    s = synth.collide_system(3000, seed=11, rm=0.2)
    p_ref, v_ref, calls, _ = oracle.collide_run(s, 3)
    for r in res:
        assert np.array_equal(r["pos"].view(np.uint32), p_ref.view(np.uint32))
    v = np.concatenate([r["vel"] for r in res])
    assert np.array_equal(v.view(np.uint32), v_ref[:, :3].view(np.uint32))
    assert sum(int(r["calls"][0]) for r in res) == calls


def test_ray_strips_world2():
    res = _run("ray", "coal")
    types, P = synth.ray_scene(40, seed=7)
    W, H = 48, 27
    cam = synth.ray_camera(W, H)
    rgb_ref, hid_ref, _, _ = oracle.ray_render(W, H, types, P, cam, synth.RAY_ALBEDO)
    for r in res:
        assert np.array_equal(r["hid"].reshape(-1), np.asarray(hid_ref).reshape(-1))
        assert np.array_equal(r["rgb"].reshape(-1).view(np.uint32),
                              np.asarray(rgb_ref, np.float32).reshape(-1).view(np.uint32))
