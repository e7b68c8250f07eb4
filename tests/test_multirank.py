"""Multi-rank path: rows sharded by star, shared slice + scalar norms allreduced.

CPU (gloo, world_size 2, run here): each process takes its O-SHARD star range from the PRODUCT's host shard map,
checks it against the oracle bit-exactly, runs the oracle products on its own shard and combines them with a real
gloo allreduce (AR1: constraint dots; AR2: shared slice), which must equal the single-rank products -- i.e. the
decomposition the CUDA path implements is exact.

GPU (gloo host-callback communicator, 2 processes sharing cuda:0): the product's multi-rank LSQR (AR1/AR2 through
the C ABI's allreduce hook) against the single-rank GPU run and the oracle.
"""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import workloads as W


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _init(rank, world, port):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    return dist


def _cpu_worker(rank, world, port, q):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import oracle
        import paper_conf_sc_malenzacsbvba24_b200 as avu
        dist = _init(rank, world, port)
        w = W.C1C.replace(n_stars=300, n_obs=6000, jitter_pct=50, n_ext_stars=200, seed=17)
        counts = avu.synth_obs_per_star(w.seed, w.n_stars, w.n_obs, w.jitter_pct)
        sb = avu.shard_map(counts, w.n_obs, world)
        S = oracle.System(w, rank=rank, nranks=world)
        assert (sb[rank], sb[rank + 1]) == (S.star_begin, S.star_end)
        rng = np.random.default_rng(5)
        x = rng.standard_normal(S.n_cols)
        y_full = rng.standard_normal(w.n_obs + S.n_constr)
        # aprod1: local rows + owned constraint partial dots, AR1 over the constraint part
        yl = np.zeros(S.m_local)
        S.aprod1(x, yl)
        c = torch.tensor(yl[S.n_rows:])
        dist.all_reduce(c)
        # aprod2: local astro + shared partial, AR2 over the shared slice
        yr = np.concatenate([y_full[S.row_begin:S.row_end], y_full[w.n_obs:]])
        xl = np.zeros(S.n_cols)
        S.aprod2(yr, xl)
        sh = torch.tensor(xl[S.A0:])
        dist.all_reduce(sh)
        q.put((rank, S.row_begin, yl[:S.n_rows], c.numpy(), S.star_begin, S.star_end, xl[:S.A0], sh.numpy()))
        dist.destroy_process_group()
    except Exception as e:  # pragma: no cover
        import traceback
        q.put(("error", traceback.format_exc()))


def test_gloo_two_rank_decomposition_cpu():
    import oracle
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_cpu_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    outs = [q.get(timeout=180) for _ in range(2)]
    for p in ps:
        p.join(60)
    for o in outs:
        assert o[0] != "error", o[1]
    w = W.C1C.replace(n_stars=300, n_obs=6000, jitter_pct=50, n_ext_stars=200, seed=17)
    S = oracle.System(w)
    rng = np.random.default_rng(5)
    x = rng.standard_normal(S.n_cols)
    y_full = rng.standard_normal(w.n_obs + S.n_constr)
    y1 = np.zeros(S.m_local); S.aprod1(x, y1)
    x2 = np.zeros(S.n_cols); S.aprod2(y_full, x2)
    got_y = np.zeros(S.m_local)
    got_x = np.zeros(S.n_cols)
    for (rank, rb, yrows, cdots, sb, se, xast, xsh) in outs:
        got_y[rb:rb + len(yrows)] = yrows
        got_y[S.n_rows:] = cdots  # identical on both ranks after AR1
        got_x[5 * sb:5 * se] = xast[5 * sb:5 * se]
        got_x[S.A0:] = xsh
    assert np.allclose(got_y, y1, rtol=1e-14, atol=1e-13)
    assert np.allclose(got_x, x2, rtol=1e-13, atol=1e-13)


# ------------------------------------------------------------------------------------------------ GPU
def _gpu_worker(rank, world, port, q, itn, fused):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import paper_conf_sc_malenzacsbvba24_b200 as avu
        _init(rank, world, port)
        torch.cuda.set_device(0)
        w = W.C1C.replace(jitter_pct=50)
        s = avu.Solver.synthetic(w, rank=rank, nranks=world, comm="callback")
        s.precondition()
        D = s.get_precond()
        out = s.solve(itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=False, fused=fused)
        # early convergence (fixed_count off): every rank must stop after the same iteration (lsqr_iterate's stop
        # decision may only depend on finished batches, else ranks issue different collectives)
        s.generate(w.seed)
        s.precondition()
        early = s.solve(itn_limit=500, atol=1e-9, btol=1e-9, fused=fused, poll_every=3)
        dist_obj = __import__("torch.distributed", fromlist=["all_gather_object"])
        its = [None] * world
        dist_obj.all_gather_object(its, (early["itn"], early["istop"]))
        assert len(set(its)) == 1, its
        # lsqr_result.t_iter_max_over_ranks_s: the max of every rank's mean iteration time (through the callback)
        tms = [None] * world
        dist_obj.all_gather_object(tms, (early["t_iter_mean_s"], early["t_iter_max_over_ranks_s"]))
        assert all(t[1] == max(m for m, _ in tms) for t in tms), tms
        # plain products through the ABI
        xg = torch.ones(s.n_local_cols, dtype=torch.float64, device="cuda")
        yg = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
        s.aprod1(xg, yg)
        x2 = torch.zeros_like(xg)
        s.aprod2(torch.ones_like(yg), x2)
        q.put((rank, s.star_begin, s.star_end, s.row_begin, out["x"], out["se"], out["itn"], out["r1norm"], D,
               yg.cpu().numpy(), x2.cpu().numpy()))
        s.close()
        import torch.distributed as dist
        dist.destroy_process_group()
    except Exception:
        import traceback
        q.put(("error", traceback.format_exc()))


@pytest.mark.gpu
@pytest.mark.parametrize("fused", [False, True], ids=["twopass", "fused"])
def test_gpu_two_rank_lsqr_matches_single_rank(cuda_device, fused):
    import torch
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    itn = 160  # converged (x parity needs convergence, SURVEY EXP-3)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_gpu_worker, args=(r, 2, port, q, itn, fused)) for r in range(2)]
    for p in ps:
        p.start()
    outs = [q.get(timeout=600) for _ in range(2)]
    for p in ps:
        p.join(60)
    for o in outs:
        assert o[0] != "error", o[1]
    w = W.C1C.replace(jitter_pct=50)
    s = avu.Solver.synthetic(w)
    s.precondition()
    D1 = s.get_precond()
    ref = s.solve(itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True)
    xg = torch.ones(s.n_local_cols, dtype=torch.float64, device="cuda")
    yg = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
    s.aprod1(xg, yg)
    x2 = torch.zeros_like(xg)
    s.aprod2(torch.ones_like(yg), x2)
    y1, x21 = yg.cpu().numpy(), x2.cpu().numpy()
    A0 = 5 * w.n_stars
    n_rows = w.n_obs
    for (rank, sb, se, rb, x, sev, it, r1, D, y, xx) in outs:
        A0l = 5 * (se - sb)
        glob = lambda v: (v[:A0l], v[A0l:])
        xa, xs = glob(x)
        assert it == itn
        assert np.allclose(D[:A0l], D1[5 * sb:5 * se], rtol=1e-14) and np.allclose(D[A0l:], D1[A0:], rtol=1e-14)
        rel = lambda a, b: np.linalg.norm(a - b) / np.linalg.norm(b)
        assert rel(xa, ref["x"][5 * sb:5 * se]) <= 1e-9 and rel(xs, ref["x"][A0:]) <= 1e-9
        assert abs(r1 - ref["r1norm"]) <= 1e-10 * ref["r1norm"]
        assert np.allclose(y[:len(y) - 12], y1[rb:rb + len(y) - 12], rtol=1e-12, atol=1e-12)
        assert np.allclose(y[-12:], y1[n_rows:], rtol=1e-12, atol=1e-12)
        assert np.allclose(xx[:A0l], x21[5 * sb:5 * se], rtol=1e-12, atol=1e-12)
        assert np.allclose(xx[A0l:], x21[A0:], rtol=1e-12, atol=1e-12)
    s.close()


# ------------------------------------------------------------------------------------------------ GPU, repro mode
def _gpu_repro_worker(rank, world, port, q, itn):
    try:
        import sys
        sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
        import torch
        import paper_conf_sc_malenzacsbvba24_b200 as avu
        _init(rank, world, port)
        torch.cuda.set_device(0)
        w = W.C1C.replace(jitter_pct=50)
        s = avu.Solver.synthetic(w, rank=rank, nranks=world, comm="callback")
        s.set_reproducible(True)
        s.precondition()
        D = s.get_precond()
        out = s.solve(itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=False)
        q.put((rank, s.star_begin, s.star_end, out["x"], out["se"], out["itn"], out["r1norm"], out["acond"], D))
        s.close()
        import torch.distributed as dist
        dist.destroy_process_group()
    except Exception:
        import traceback
        q.put(("error", traceback.format_exc()))


@pytest.mark.gpu
@pytest.mark.parametrize("P", [2, 3])
def test_gpu_repro_bitwise_across_rank_counts(cuda_device, P):
    """NEXT-4 across ranks: the digit allreduces are exact, so D, x, sigma and the norm estimates of a P-rank
    reproducible solve are BIT-identical to the 1-rank reproducible solve and to the oracle's repro mode -- after
    40 iterations, long before convergence (where the default mode differs already at k ~ 10)."""
    import oracle
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    itn = 40
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_gpu_repro_worker, args=(r, P, port, q, itn)) for r in range(P)]
    for p in ps:
        p.start()
    outs = [q.get(timeout=600) for _ in range(P)]
    for p in ps:
        p.join(60)
    for o in outs:
        assert o[0] != "error", o[1]
    w = W.C1C.replace(jitter_pct=50)
    s = avu.Solver.synthetic(w)
    s.set_reproducible(True)
    s.precondition()
    D1 = s.get_precond()
    ref = s.solve(itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True)
    s.close()
    ro = oracle.solve_system(oracle.System(w), atol=0, btol=0, conlim=0, itn_limit=itn, fixed_count=True, repro=True)
    same = lambda a, b: np.array_equal(np.ascontiguousarray(a).view(np.uint64), np.ascontiguousarray(b).view(np.uint64))
    assert same(ref["x"], ro["x"]) and same(ref["se"], ro["se"])
    A0 = 5 * w.n_stars
    for (rank, sb, se, x, sev, it, r1, ac, D) in outs:
        A0l = 5 * (se - sb)
        assert it == itn and r1 == ref["r1norm"] and ac == ref["acond"]
        assert same(D[:A0l], D1[5 * sb:5 * se]) and same(D[A0l:], D1[A0:])
        assert same(x[:A0l], ref["x"][5 * sb:5 * se]) and same(x[A0l:], ref["x"][A0:])
        assert same(sev[:A0l], ref["se"][5 * sb:5 * se]) and same(sev[A0l:], ref["se"][A0:])


# ------------------------------------------------------------------------------------------------ GPU, NCCL path
@pytest.mark.gpu
@pytest.mark.parametrize("mode", ["twopass", "fused", "repro"])
def test_gpu_nccl_path_forced_on_one_rank(cuda_device, mode):
    """The multi-rank algorithm (AR1/AR2, or the repro digit reductions) through a REAL NCCL communicator: with
    lsqr_env.force_collectives a single process builds a 1-rank NCCL communicator (dlopen'ed libnccl, internally
    generated unique id) and runs every collective of the P > 1 path, captured in the CUDA graph.  NCCL cannot put
    two ranks on one GPU, so this is how the NCCL plumbing is exercised in a one-GPU run; the results must equal the
    single-rank path (bit-identical in the reproducible mode)."""
    import torch
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    w = W.C1C.replace(jitter_pct=50)
    itn = 160 if mode != "repro" else 40
    kw = dict(itn_limit=itn, atol=0, btol=0, conlim=0, fixed_count=True, use_graph=True, fused=(mode == "fused"))
    outs, Ds, prods = [], [], []
    for force in (False, True):
        s = avu.Solver.synthetic(w, force_collectives=force)
        if mode == "repro":
            s.set_reproducible(True)
        s.precondition()
        Ds.append(s.get_precond())
        xg = torch.ones(s.n_local_cols, dtype=torch.float64, device="cuda")
        yg = torch.zeros(s.n_local_rows + s.n_constr, dtype=torch.float64, device="cuda")
        s.aprod1(xg, yg)
        x2 = torch.zeros_like(xg)
        s.aprod2(torch.ones_like(yg), x2)
        prods.append((yg.cpu().numpy(), x2.cpu().numpy()))
        outs.append(s.solve(**kw))
        s.close()
    a, b = outs
    assert a["itn"] == b["itn"] == itn
    if mode == "repro":
        same = lambda p, q: np.array_equal(np.asarray(p).view(np.uint64), np.asarray(q).view(np.uint64))
        assert same(Ds[0], Ds[1]) and same(a["x"], b["x"]) and same(a["se"], b["se"])
        assert a["r1norm"] == b["r1norm"] and a["acond"] == b["acond"]
    else:
        rel = lambda p, q: np.linalg.norm(p - q) / np.linalg.norm(q)
        assert np.allclose(Ds[0], Ds[1], rtol=1e-14, atol=0)
        assert rel(b["x"], a["x"]) <= 1e-9 and abs(b["r1norm"] - a["r1norm"]) <= 1e-10 * a["r1norm"]
    assert np.allclose(prods[0][0], prods[1][0], rtol=1e-12, atol=1e-12)
    assert np.allclose(prods[0][1], prods[1][1], rtol=1e-12, atol=1e-12)


@pytest.mark.gpu
@pytest.mark.parametrize("fused", [False, True], ids=["twopass", "fused"])
def test_gpu_nccl_forced_early_stop(cuda_device, fused):
    """Early convergence through the asynchronous NCCL path (graph-captured collectives, stop flag polled every 3
    iterations while the next batch runs): the stop is taken after the batch in which the halting iteration ran,
    so itn, istop and x equal the single-rank path's (a decision based on a flag written by a batch still
    in flight could make ranks disagree on the number of batches)."""
    import paper_conf_sc_malenzacsbvba24_b200 as avu
    w = W.C1C.replace(jitter_pct=50)
    outs = []
    for force in (False, True):
        s = avu.Solver.synthetic(w, force_collectives=force)
        s.precondition()
        outs.append(s.solve(itn_limit=500, atol=1e-9, btol=1e-9, fused=fused, poll_every=3, use_graph=True))
        s.close()
    a, b = outs
    assert 0 < a["itn"] < 500 and a["istop"] in (1, 2)
    assert a["istop"] == b["istop"] and abs(a["itn"] - b["itn"]) <= 2  # |d itn| <= 2 across roundings
    # stopped at a 1e-9 tolerance, not converged to rounding: x agrees to the accuracy the stopping rule gives
    assert np.linalg.norm(a["x"] - b["x"]) <= 1e-5 * np.linalg.norm(a["x"])
