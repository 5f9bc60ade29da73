"""GPU: the point-to-point activation channel (ea_chan_*, row f2) -- the pipeline runtime's transfers done by the
library itself (copy engine over a peer mapping, handshake by stream memory operations, P:110 / Alg. 1).

Byte-exact delivery in order, ring wrap-around (more messages than slots), a receiver stream that starts before
the sender (the GPU waits, not the host), sender and receiver on different streams, the error paths, and the
cross-process path through CUDA IPC handles with two processes on one GPU."""
import os

import pytest
import torch

from paper_conf_ppopp_chen0qz23_b200.binding import Channel, EAError

pytestmark = pytest.mark.gpu


def _pair(slot_bytes, slots):
    s, r = Channel("send", slot_bytes, slots), Channel("recv", slot_bytes, slots)
    Channel.pair(s, r)
    return s, r


@pytest.mark.parametrize("slots", [1, 3, 8])
def test_channel_delivers_in_order_with_wraparound(slots):
    n_msgs, numel = 4 * slots + 3, 50_001
    snd, rcv = _pair(numel * 4, slots)
    s_send, s_recv = torch.cuda.Stream(), torch.cuda.Stream()
    gen = torch.Generator(device="cuda").manual_seed(7)
    msgs = [torch.randn(numel, device="cuda", generator=gen) for _ in range(n_msgs)]
    torch.cuda.synchronize()
    outs = [torch.empty(numel, device="cuda") for _ in range(n_msgs)]
    # interleave so the sender never runs more than `slots` ahead on the host side of the GPU queues
    for k in range(n_msgs):
        snd.send(msgs[k], stream=s_send)
        rcv.recv(outs[k], stream=s_recv)
    torch.cuda.synchronize()
    for k in range(n_msgs):
        assert torch.equal(outs[k], msgs[k]), k
    assert snd.count == rcv.count == n_msgs
    snd.close()
    rcv.close()


def test_receiver_enqueued_first_waits_on_the_gpu():
    """All receives are enqueued before any send: the receiver's stream waits on the device (a host-blocking
    receive would deadlock here) and completes once the sends are enqueued."""
    snd, rcv = _pair(4096 * 4, 4)
    s_send, s_recv = torch.cuda.Stream(), torch.cuda.Stream()
    msgs = [torch.full((4096,), float(k), device="cuda") for k in range(4)]
    outs = [torch.zeros(4096, device="cuda") for _ in range(4)]
    torch.cuda.synchronize()
    for k in range(4):
        rcv.recv(outs[k], stream=s_recv)
    assert not s_recv.query()          # waiting for the first message
    for k in range(4):
        snd.send(msgs[k], stream=s_send)
    torch.cuda.synchronize()
    for k in range(4):
        assert torch.equal(outs[k], msgs[k])


def test_sender_waits_for_a_free_slot():
    """With 2 slots the third send must wait until the receiver freed slot 0: the bytes of message 0 are not
    overwritten before they are read."""
    snd, rcv = _pair(1024 * 4, 2)
    s_send, s_recv = torch.cuda.Stream(), torch.cuda.Stream()
    msgs = [torch.full((1024,), float(k + 1), device="cuda") for k in range(6)]
    outs = [torch.zeros(1024, device="cuda") for _ in range(6)]
    # load the sleep kernel now: CUDA's lazy module loading synchronises the context to load a kernel, which
    # cannot finish while s_send waits for the receiver (include/ea.h, "Activation channels")
    torch.cuda._sleep(1)
    torch.cuda.synchronize()
    for k in range(6):
        snd.send(msgs[k], stream=s_send)   # sends 2..5 wait on the GPU for acknowledgements
    assert not s_send.query()
    with torch.cuda.stream(s_recv):
        torch.cuda._sleep(1_000_000)       # the receiver runs late
    for k in range(6):
        rcv.recv(outs[k], stream=s_recv)
    torch.cuda.synchronize()
    for k in range(6):
        assert torch.equal(outs[k], msgs[k])


def test_mixed_dtypes_and_sizes():
    snd, rcv = _pair(1 << 20, 3)
    torch.cuda.synchronize()
    msgs = [torch.arange(1000, dtype=torch.int64, device="cuda"), torch.randn(7, 5, device="cuda").to(torch.bfloat16),
            torch.randn(1, device="cuda"), torch.empty(0, device="cuda"), torch.randn(262_144, device="cuda")]
    outs = [torch.empty_like(m) for m in msgs]
    for m, o in zip(msgs, outs):
        snd.send(m)
        rcv.recv(o)
    torch.cuda.synchronize()
    for m, o in zip(msgs, outs):
        assert torch.equal(m, o)


def test_channel_errors():
    snd, rcv = _pair(256, 2)
    with pytest.raises(EAError, match="does not fit"):
        snd.send(torch.zeros(65, device="cuda"))
    with pytest.raises(EAError, match="receiving end"):
        rcv.send(torch.zeros(4, device="cuda"))
    with pytest.raises(EAError, match="sending end"):
        snd.recv(torch.zeros(4, device="cuda"))
    lone = Channel("send", 256, 2)
    with pytest.raises(EAError, match="not connected"):
        lone.send(torch.zeros(4, device="cuda"))
    g = torch.cuda.CUDAGraph()
    x = torch.zeros(4, device="cuda")
    side = torch.cuda.Stream()
    with pytest.raises(EAError, match="CUDA graph"):
        with torch.cuda.graph(g, stream=side):
            snd.send(x)
    with pytest.raises(EAError):
        Channel("send", 0, 2)
    # connect checks the exported geometry and role before mapping anything
    other_send, other_recv3 = Channel("send", 256, 2), Channel("recv", 256, 3)
    with pytest.raises(EAError, match="opposite role"):
        Channel("send", 256, 2).connect(other_send.export())
    with pytest.raises(EAError, match="differs"):
        Channel("send", 256, 2).connect(other_recv3.export())
    with pytest.raises(ValueError):
        lone.connect(b"\0" * 64)
    assert snd.count == 0 and rcv.count == 0   # nothing was enqueued by the failing calls


def test_stalled_peer_is_detected_by_the_deadline():
    """pipeline.wait_streams: a receive whose message never comes raises TimeoutError instead of hanging; the
    late send then releases the stream."""
    from paper_conf_ppopp_chen0qz23_b200.pipeline import wait_streams
    snd, rcv = _pair(1024, 2)
    s_recv = torch.cuda.Stream()
    out = torch.zeros(256, device="cuda")
    ones = torch.ones(256, device="cuda")     # no kernel launches while s_recv is blocked (lazy loading, above)
    torch.cuda.synchronize()
    rcv.recv(out, stream=s_recv)
    with pytest.raises(TimeoutError, match="peer stage stalled"):
        wait_streams([s_recv], 0.5, "stage 1")
    snd.send(ones)
    wait_streams([s_recv], 60.0)
    assert torch.equal(out, ones)


def _ipc_worker(rank, port, q, n_msgs):
    import torch.distributed as dist
    os.environ["CUDA_MODULE_LOADING"] = "EAGER"   # before this process initialises CUDA (see pipeline.py)
    try:
        torch.cuda.set_device(0)
        dist.init_process_group("gloo", init_method=port, rank=rank, world_size=2)
        ch = Channel("send" if rank == 0 else "recv", 8192 * 4, 3)
        handles = [None, None]
        dist.all_gather_object(handles, ch.export())
        ch.connect(handles[1 - rank])
        s = torch.cuda.Stream()
        gen = torch.Generator(device="cuda").manual_seed(11)
        msgs = [torch.randn(8192, device="cuda", generator=gen) for _ in range(n_msgs)]
        torch.cuda.synchronize()
        if rank == 0:
            for m in msgs:
                ch.send(m, stream=s)
            s.synchronize()
            ok = True
        else:
            outs = [torch.empty(8192, device="cuda") for _ in range(n_msgs)]
            for o in outs:
                ch.recv(o, stream=s)
            s.synchronize()
            ok = all(torch.equal(a, b) for a, b in zip(outs, msgs))
        dist.barrier()
        ch.close()
        q.put((rank, "ok" if ok else "mismatch"))
    except Exception:  # pragma: no cover
        import traceback
        q.put((rank, traceback.format_exc()))
    finally:
        if dist.is_initialized():
            dist.destroy_process_group()


def test_channel_across_processes_via_cuda_ipc():
    import tempfile
    import torch.multiprocessing as mp
    port = "file://" + os.path.join(tempfile.mkdtemp(prefix="gloo_"), "store")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_ipc_worker, args=(r, port, q, 10)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
    assert res == {0: "ok", 1: "ok"}, res
