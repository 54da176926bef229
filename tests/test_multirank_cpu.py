"""N > 1 paths on CPU: world_size-2 `gloo` process groups (127.0.0.1).

* graph (§8e): each rank owns a contiguous vertex block, runs the per-vertex
  update rules on its block only (written here from the method definitions,
  numpy), and exchanges state with the SAME helpers the GPU path uses
  (graph.allgather_block / allreduce_sum). Results must equal the unsharded
  CPU oracle: BFS depths and CC labels exactly, PageRank to 1e-6.
* micro bench plumbing: per-rank shards seeded seed + rank, checksum
  all-reduce and max-over-ranks timing.
* ray strips: the round-robin 8-row strips of all ranks tile the frame.
"""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _graph_worker(rank, world, port, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_asplos_zhangar21_b200.graph import allgather_block, allreduce_sum, block_range
    offs, col = synth.rmat_graph(11, seed=4)
    V = len(offs) - 1
    lo, hi, per = block_range(V, rank, world)
    deg = np.diff(offs.astype(np.int64))
    src = int(np.argmax(deg))
    # BFS bottom-up probes on owned vertices, depth all-gathered each level
    depth = torch.full((V,), -1, dtype=torch.int32)
    depth[src] = 0
    level = 0
    while True:
        d = depth.numpy()
        new = d.copy()
        cnt = 0
        for v in range(lo, hi):
            if d[v] == -1 and np.any(d[col[offs[v]:offs[v + 1]]] == level):
                new[v] = level + 1
                cnt += 1
        depth.copy_(torch.from_numpy(new))
        allgather_block(depth, V, per, rank, world)
        c = torch.tensor([cnt], dtype=torch.int32)
        allreduce_sum(c, world)
        level += 1
        if int(c) == 0:
            break
    # CC Jacobi on owned vertices
    lab = torch.arange(V, dtype=torch.int32)
    while True:
        l = lab.numpy()
        out = l.copy()
        ch = 0
        for v in range(lo, hi):
            nb = col[offs[v]:offs[v + 1]]
            m = min(l[v], l[nb].min()) if len(nb) else l[v]
            ch |= int(m != l[v])
            out[v] = m
        lab.copy_(torch.from_numpy(out))
        allgather_block(lab, V, per, rank, world)
        c = torch.tensor([ch], dtype=torch.int32)
        allreduce_sum(c, world)
        if int(c) == 0:
            break
    # PageRank: contributions + dangling exchanged, 20 iterations
    r = torch.full((V,), np.float32(1.0 / V), dtype=torch.float32)
    d_ = 0.85
    for _ in range(20):
        rr = r.numpy().astype(np.float64)
        contrib = torch.zeros(V, dtype=torch.float64)
        cn = contrib.numpy()
        dang = 0.0
        for v in range(lo, hi):
            if deg[v]:
                cn[v] = rr[v] / deg[v]
            else:
                dang += rr[v]
        allgather_block(contrib, V, per, rank, world)
        D = torch.tensor([dang], dtype=torch.float64)
        allreduce_sum(D, world)
        cn = contrib.numpy()
        new = r.numpy().copy()
        for v in range(lo, hi):
            s = cn[col[offs[v]:offs[v + 1]]].sum()
            new[v] = np.float32((1 - d_) / V + d_ * (s + float(D) / V))
        r.copy_(torch.from_numpy(new))
        allgather_block(r, V, per, rank, world)
    np.save(os.path.join(outdir, f"g{rank}.npy"), np.stack([depth.numpy().astype(np.float64),
                                                            lab.numpy().astype(np.float64),
                                                            r.numpy().astype(np.float64)]))
    dist.destroy_process_group()


def test_graph_sharded_gloo_matches_oracle():
    world = 2
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_graph_worker, args=(world, _free_port(), td), nprocs=world, join=True)
        res = [np.load(os.path.join(td, f"g{r}.npy")) for r in range(world)]
    offs, col = synth.rmat_graph(11, seed=4)
    t = synth.vertex_types(offs)
    src = int(np.argmax(np.diff(offs.astype(np.int64))))
    depth, _, _, _ = oracle.graph_bfs(offs, col, t, src)
    label, _, _, _ = oracle.graph_cc(offs, col, t)
    rank, _ = oracle.graph_pr(offs, col, t, iters=20)
    for r in res:  # every rank ends with the full, identical state
        assert np.array_equal(r[0].astype(np.int32), depth)
        assert np.array_equal(r[1].astype(np.uint32), label)
        np.testing.assert_allclose(r[2], rank, rtol=1e-6)


def _micro_worker(rank, world, port, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    n, T, R = 50_000, 4, 3
    types = synth.micro_types(n, T, "random", seed=42 + rank)  # bench.py: seed + rank per shard
    init = synth.micro_init(n, seed=42 + rank)
    vals, sec = oracle.micro_run(types, init, T, R)
    cs = torch.tensor([int(vals.astype(np.int64).sum())], dtype=torch.int64)
    dist.all_reduce(cs)
    tt = torch.tensor([sec + rank], dtype=torch.float64)
    dist.all_reduce(tt, op=dist.ReduceOp.MAX)
    np.save(os.path.join(outdir, f"m{rank}.npy"), np.array([int(cs), float(tt)], dtype=np.float64))
    dist.destroy_process_group()


def test_micro_weak_scaling_plumbing_gloo():
    world = 2
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_micro_worker, args=(world, _free_port(), td), nprocs=world, join=True)
        res = [np.load(os.path.join(td, f"m{r}.npy")) for r in range(world)]
    expect = 0
    for rank in range(world):
        t = synth.micro_types(50_000, 4, "random", seed=42 + rank)
        i = synth.micro_init(50_000, seed=42 + rank)
        expect += int((i.astype(np.int64) + 3 * (t.astype(np.int64) + 1)).sum())
    for r in res:
        assert int(r[0]) == expect
        assert r[1] >= 1.0  # max over ranks includes rank 1's +1 s offset


def test_ray_strips_tile_the_frame():
    from paper_conf_asplos_zhangar21_b200.ray import Ray
    H = 1080
    for world in (1, 2, 3, 8):
        rows = []
        for rank in range(world):
            rows += [r for r0, n in Ray.strips(Ray, H, rank, world) for r in range(r0, r0 + n)]
        assert sorted(rows) == list(range(H))


def _exchange_worker(rank, world, port, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_asplos_zhangar21_b200 import exchange
    out = {}
    # BlockArray: padded persistent buffer, each rank writes its block, one gather
    n = 101
    lo, hi, per = exchange.block_range(n, rank, world, align=8)
    ba = exchange.BlockArray(n, per, rank, world, torch.float64, "cpu", rest=(3,), fill=-1.0)
    ptr = ba.data_ptr()
    for it in range(3):  # persistent: repeated gathers reuse the same storage
        ba.view[lo:hi] = torch.arange(lo, hi, dtype=torch.float64)[:, None] * (it + 1) + torch.arange(3)
        ba.gather()
    assert ba.data_ptr() == ptr
    out["ba"] = ba.view.numpy().copy()
    # halo rows of a W x H row-slab decomposition, dead border and torus
    W, H = 5, 11
    for torus in (False, True):
        h = exchange.HaloRows(W, H, rank, world, torus)
        st = torch.full((H * W,), 255, dtype=torch.uint8)
        rows = torch.arange(H, dtype=torch.uint8)[:, None].expand(H, W).reshape(-1)
        st[h.r0 * W:h.r1 * W] = rows[h.r0 * W:h.r1 * W]
        h.exchange(st)
        out[f"halo{int(torus)}"] = st.numpy().copy()
        out[f"r{int(torus)}"] = np.array([h.r0, h.r1])
    c = torch.tensor([rank + 1.5], dtype=torch.float64)
    exchange.allreduce_(c, world)
    out["sum"] = c.numpy()
    np.savez(os.path.join(outdir, f"x{rank}.npz"), **out)
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_exchange_blockarray_halo_gloo(world):
    """exchange.py (the GPU apps' data plane) over real gloo groups: one
    in-place all-gather of padded blocks into a persistent buffer, the GEN
    halo rows (dead border and torus, incl. world 2 where both neighbours are
    the same rank), and the scalar all-reduce."""
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_exchange_worker, args=(world, _free_port(), td), nprocs=world, join=True)
        res = [dict(np.load(os.path.join(td, f"x{r}.npz"))) for r in range(world)]
    n = 101
    expect = np.arange(n, dtype=np.float64)[:, None] * 3 + np.arange(3)
    W, H = 5, 11
    for r in res:
        assert np.array_equal(r["ba"], expect)
        assert r["sum"][0] == sum(k + 1.5 for k in range(world))
        for torus in (0, 1):
            r0, r1 = r[f"r{torus}"]
            st = r[f"halo{torus}"].reshape(H, W)
            assert (st[r0:r1] == np.arange(r0, r1)[:, None]).all()
            for row in (r0 - 1, r1):
                if 0 <= row < H or torus:
                    assert (st[row % H] == row % H).all(), (torus, row)
            untouched = [q for q in range(H) if not (r0 - 1 <= q <= r1) and not (torus and q in ((r0 - 1) % H, r1 % H))]
            assert all((st[q] == 255).all() for q in untouched)


def _vargather_worker(rank, world, port, outdir):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_asplos_zhangar21_b200 import exchange
    vg = exchange.VarGather(world, 6, "cpu")
    out = {}
    for step, extra in enumerate((0, 3, 1)):  # the send buffer grows and keeps its content
        count = rank * 2 + extra
        send = vg.send_buffer(count)
        send[:count] = torch.arange(count * 6, dtype=torch.uint8).view(count, 6) + 10 * rank
        recv, counts, seg = vg.gather(count)
        out[f"recv{step}"] = recv.numpy().copy()
        out[f"counts{step}"] = counts.numpy().copy()
        out[f"seg{step}"] = np.array([seg])
    np.savez(os.path.join(outdir, f"v{rank}.npz"), **out)
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_exchange_vargather_gloo(world):
    """exchange.VarGather (collision's post-update exchange): variable-length
    row lists, every rank's rows in its own segment, counts all-gathered."""
    with tempfile.TemporaryDirectory() as td:
        mp.spawn(_vargather_worker, args=(world, _free_port(), td), nprocs=world, join=True)
        res = [dict(np.load(os.path.join(td, f"v{r}.npz"))) for r in range(world)]
    for step, extra in enumerate((0, 3, 1)):
        counts = [r * 2 + extra for r in range(world)]
        for d in res:
            assert list(d[f"counts{step}"]) == counts
            seg = int(d[f"seg{step}"][0])
            assert seg == max(max(counts), 1)
            recv = d[f"recv{step}"]
            for r, c in enumerate(counts):
                want = np.arange(c * 6, dtype=np.uint8).reshape(c, 6) + 10 * r
                assert np.array_equal(recv[r * seg:r * seg + c], want)
