"""Row f2: the live advance-forward pipeline runtime (pipeline.PipelineStage)
on K ranks over gloo (CPU).  For every advance (1F1B, one extra, AFAB) the
per-stage parameter gradients of every pipeline must equal a single-process
reference (full model, same micro-batches, loss/M summed); the peak stash of
each stage must be min(a_k+1, M); with the dynamic controller
all stages agree on the advance after every iteration (c16 feasibility)."""
import os
import tempfile

import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle.schedule import advance_forward_schedule, peak_in_flight, simulate_pipeline

D, B = 8, 3


def _model(seed):
    torch.manual_seed(seed)
    return torch.nn.ModuleList([torch.nn.Sequential(torch.nn.Linear(D, D), torch.nn.Tanh()) for _ in range(3)])


def _data(N, M, seed=0):
    g = torch.Generator().manual_seed(seed)
    xs = [[torch.randn(B, D, generator=g) for _ in range(M)] for _ in range(N)]
    ys = [[torch.randn(B, D, generator=g) for _ in range(M)] for _ in range(N)]
    return xs, ys


def _worker(rank, K, N, M, extra, dynamic, port, q, concurrent=False):
    try:
        dist.init_process_group("gloo", init_method=port, rank=rank, world_size=K)
        from paper_conf_ppopp_chen0qz23_b200.pipeline import PipelineStage
        models = [_model(100 + i) for i in range(N)]
        stage_mods = [m[rank] for m in models]
        xs, ys = _data(N, M)
        st = PipelineStage(stage_mods, rank, K, M, extra_advance=extra, dynamic=dynamic, mem_limit=1e9,
                           mem_per_microbatch=1.0, concurrent=concurrent)
        loss_fn = torch.nn.functional.mse_loss
        iters = 3 if dynamic else 1
        for _ in range(iters):
            for m in stage_mods:
                m.zero_grad()
            st.run_iteration(inputs=xs if rank == 0 else None, targets=ys if rank == K - 1 else None,
                             loss_fn=loss_fn, act_shape=(B, D), act_dtype=torch.float32)
        # numpy copies are pickled by value: tensors would travel as shared-memory file descriptors, which fail
        # (FileNotFoundError) when this process exits before the parent has received them
        grads = [[p.grad.detach().numpy().copy() for p in m.parameters()] for m in stage_mods]
        q.put((rank, "ok", grads, st.history))
    except Exception as e:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc(), None, None))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _file_store():
    """A fresh file:// rendezvous (no TCP port to race for between tests)."""
    d = tempfile.mkdtemp(prefix="gloo_")
    return "file://" + os.path.join(d, "store")


def _run(K, N, M, extra, dynamic=False, concurrent=False):
    port = _file_store()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, K, N, M, extra, dynamic, port, q, concurrent)) for r in range(K)]
    for p in procs:
        p.start()
    out = {}
    for _ in range(K):
        r, status, grads, hist = q.get(timeout=300)
        assert status == "ok", status
        out[r] = ([[torch.from_numpy(a) for a in gm] for gm in grads], hist)
    for p in procs:
        p.join(timeout=60)
    return out


def _reference_grads(N, M):
    xs, ys = _data(N, M)
    ref = []
    for i in range(N):
        m = _model(100 + i)
        for j in range(M):
            h = xs[i][j]
            for k in range(3):
                h = m[k](h)
            (torch.nn.functional.mse_loss(h, ys[i][j]) / M).backward()
        ref.append([[p.grad.clone() for p in m[k].parameters()] for k in range(3)])
    return ref


@pytest.mark.parametrize("extra,concurrent", [(0, False), (1, False), (8, False), (1, True), (8, True)])
def test_pipeline_gradients_match_reference(extra, concurrent):
    """concurrent=True: the N pipelines run at once (one thread each, one process group per pipeline)."""
    K, N, M = 3, 2, 6
    out = _run(K, N, M, extra, concurrent=concurrent)
    ref = _reference_grads(N, M)
    for k in range(K):
        grads, hist = out[k]
        for i in range(N):
            for g, r in zip(grads[i], ref[i][k]):
                torch.testing.assert_close(g, r, rtol=1e-5, atol=1e-7)
        e = min(extra, M - (K - 1))                 # GPU 1's advance_num is capped at M (c15/c27)
        a = min(M, K - 1 - k + e)
        assert hist[0]["advance"] == a
        assert hist[0]["peak_stash"] == peak_in_flight(advance_forward_schedule(K, M, k + 1, a))


def test_dynamic_advance_stays_consistent_and_feasible():
    K, N, M = 3, 1, 6
    out = _run(K, N, M, 0, dynamic=True)
    hists = [out[k][1] for k in range(K)]
    for it in range(len(hists[0])):
        e = [hists[k][it]["advance"] - (K - 1 - k) for k in range(K)]
        advs = [hists[k][it]["advance"] for k in range(K)]
        assert len(set(e)) == 1 or max(advs) == M            # one shared extra (capped at M)
        assert simulate_pipeline(K, M, advs)["ok"]
