"""End to end on one GPU: K=2 pipeline stages as 2 processes sharing cuda:0
(activations over gloo, or the library's CUDA-IPC activation channels), N=2 parallel pipelines, advance-forward order, and
after every iteration ONE fused co-located elastic-averaging step per stage
on the stage's parameters (views into flat buffers the kernel updates in
place).  Compared with a single-process reference: the full model's autograd
plus the float64 oracle step (rounded to fp32 storage) -- rows f2 + a1-a5."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

from oracle.ea_oracle import Hyper, ea_step

pytestmark = pytest.mark.gpu

D, B, K, N, M, ITERS = 16, 4, 2, 2, 4, 3
LR, MU = 0.05, 0.9


def _model(seed):
    torch.manual_seed(seed)
    return torch.nn.ModuleList([torch.nn.Sequential(torch.nn.Linear(D, D), torch.nn.Tanh()) for _ in range(K)])


def _data(it):
    g = torch.Generator().manual_seed(1000 + it)
    xs = [[torch.randn(B, D, generator=g) for _ in range(M)] for _ in range(N)]
    ys = [[torch.randn(B, D, generator=g) for _ in range(M)] for _ in range(N)]
    return xs, ys


def _flatten(mod, device):
    """Make mod's parameters (and grads) views of one flat buffer each."""
    params = list(mod.parameters())
    n = sum(p.numel() for p in params)
    flat = torch.empty(n, device=device)
    gflat = torch.zeros(n, device=device)
    off = 0
    for p in params:
        k = p.numel()
        flat[off:off + k].copy_(p.data.reshape(-1))
        p.data = flat[off:off + k].view_as(p)
        p.grad = gflat[off:off + k].view_as(p)
        off += k
    return flat, gflat


def _worker(rank, port, q, concurrent=False, backend="gloo", transport="dist"):
    if transport == "ipc":
        os.environ["CUDA_MODULE_LOADING"] = "EAGER"   # required by the ipc transport (pipeline.py), before CUDA init
    try:
        dev = torch.device("cuda", rank if backend == "nccl" else 0)
        torch.cuda.set_device(dev)
        if backend == "nccl":
            dist.init_process_group("nccl", init_method=port, rank=rank, world_size=K, device_id=dev)
        else:
            dist.init_process_group("gloo", init_method=port, rank=rank, world_size=K)
        from paper_conf_ppopp_chen0qz23_b200.binding import ElasticAveraging
        from paper_conf_ppopp_chen0qz23_b200.pipeline import PipelineStage
        mods = [_model(100 + i)[rank].to(dev) for i in range(N)]
        flats = [_flatten(m, dev) for m in mods]
        P = flats[0][0].numel()
        center = flats[0][0].clone()
        ea = ElasticAveraging([P], N, beta=1.0, rho=1.0, lr=LR, momentum=MU, device=dev.index)   # alpha = 1/N
        st = PipelineStage(mods, rank, K, M, ea=ea, ea_stage=0, center=center,
                           flat_params=[f for f, _ in flats], flat_grads=[g for _, g in flats], extra_advance=1,
                           concurrent=concurrent, transport=transport, act_bytes=B * D * 4, device=dev)
        for it in range(ITERS):
            xs, ys = _data(it)
            if not concurrent:
                for _, g in flats:
                    g.zero_()
            # concurrent: grads zeroed on each pipeline's stream after the previous EA step, and the EA step
            # of this iteration left running on its stream (sync=False): the next forwards wait for it on the GPU
            st.run_iteration(inputs=[[x.to(dev) for x in r] for r in xs] if rank == 0 else None,
                             targets=[[y.to(dev) for y in r] for r in ys] if rank == K - 1 else None,
                             loss_fn=torch.nn.functional.mse_loss, act_shape=(B, D), act_dtype=torch.float32,
                             device=dev, zero_grads=concurrent, sync=not concurrent)
        torch.cuda.synchronize()
        q.put((rank, "ok", [f.cpu().numpy() for f, _ in flats], center.cpu().numpy()))
        st.close()
        ea.close()
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc(), None, None))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def _reference():
    models = [_model(100 + i) for i in range(N)]
    hp = Hyper(alpha=float(np.float32(1 / N)), beta=1.0, rho=1.0, lr=float(np.float32(LR)),
               momentum=float(np.float32(MU)))
    flat = lambda m, k: torch.cat([p.detach().reshape(-1) for p in m[k].parameters()]).double().numpy()
    centers = [flat(models[0], k) for k in range(K)]
    moms = [[np.zeros_like(centers[k]) for _ in range(N)] for k in range(K)]
    for it in range(ITERS):
        xs, ys = _data(it)
        for i, m in enumerate(models):
            m.zero_grad()
            for j in range(M):
                h = xs[i][j]
                for k in range(K):
                    h = m[k](h)
                (torch.nn.functional.mse_loss(h, ys[i][j]) / M).backward()
        for k in range(K):
            xs_k = [flat(models[i], k) for i in range(N)]
            gs_k = [torch.cat([p.grad.reshape(-1) for p in models[i][k].parameters()]).double().numpy()
                    for i in range(N)]
            nx, moms[k], c = ea_step(xs_k, moms[k], centers[k], gs_k, hp)
            centers[k] = c.astype(np.float32).astype(np.float64)                 # fp32 storage
            moms[k] = [mm.astype(np.float32).astype(np.float64) for mm in moms[k]]
            for i in range(N):
                off = 0
                for p in models[i][k].parameters():
                    n = p.numel()
                    p.data.copy_(torch.from_numpy(nx[i][off:off + n].astype(np.float32)).view_as(p))
                    off += n
    return [[flat(models[i], k) for i in range(N)] for k in range(K)], centers


@pytest.mark.parametrize("concurrent,backend,transport", [(False, "gloo", "dist"), (True, "gloo", "dist"),
                                                           (True, "nccl", "dist"), (False, "gloo", "ipc"),
                                                           (True, "gloo", "ipc")])
def test_pipeline_with_elastic_averaging_matches_reference(concurrent, backend, transport):
    """concurrent: the N pipelines at once (thread + stream + process group each), the EA step on its own
    stream.  nccl: activations as device tensors over NCCL, one GPU per stage (needs K GPUs).  ipc: activations
    through the library's channels (ea_chan_*: copy engine into the peer stage's memory over CUDA IPC, the GPU
    waits for messages, not the host); both stages share cuda:0 here, the same code maps NVLink peers."""
    import tempfile
    if backend == "nccl" and torch.cuda.device_count() < K:
        pytest.skip(f"NCCL activations need {K} GPUs (NCCL refuses two ranks on one device)")
    port = "file://" + os.path.join(tempfile.mkdtemp(prefix="gloo_"), "store")   # no TCP port race
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, port, q, concurrent, backend, transport)) for r in range(K)]
    for p in procs:
        p.start()
    out = {}
    for _ in range(K):
        r, status, flats, center = q.get(timeout=600)
        assert status == "ok", status
        out[r] = (flats, center)
    for p in procs:
        p.join(timeout=60)
    ref_params, ref_centers = _reference()
    for k in range(K):
        flats, center = out[k]
        np.testing.assert_allclose(center, ref_centers[k], rtol=1e-4, atol=1e-6)
        for i in range(N):
            np.testing.assert_allclose(flats[i], ref_params[k][i], rtol=1e-4, atol=1e-6)
