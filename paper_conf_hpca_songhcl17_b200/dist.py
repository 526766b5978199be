"""Multi-GPU plumbing for the data-parallel hot path.

One process per GPU (torchrun), torch.distributed over NCCL (NVLink /
NVSwitch) -- plumbing only; every compute step runs in libpcnn's kernels.

* C1 weights: rank 0 owns the parameters and broadcasts ONE flat fp32 buffer
  once (NVLS multicast on NVSwitch when NCCL picks it); every rank then packs
  it into its own net with pcnn_create_net.
* C2 inputs: none -- each rank regenerates its shard of images from their
  global indices (synth.images), or a shard range for a fixed global batch.
* C3 logits: all_gather_into_tensor of the [B/W, classes] fp32 outputs.

The images are independent, so there is no exchange inside the hot path and
no collective is fused into a kernel.  Works with the gloo
backend on CPU tensors for the host-logic tests.
"""
import time

import numpy as np


def shard_range(global_batch, world, rank):
    """Contiguous shard [start, start+count) of `global_batch` images for
    `rank`; the remainder goes to the low ranks."""
    base, rem = divmod(global_batch, world)
    count = base + (1 if rank < rem else 0)
    start = rank * base + min(rank, rem)
    return start, count


def _device():
    import torch
    import torch.distributed as dist
    if dist.get_backend() == "nccl":
        return torch.device("cuda", torch.cuda.current_device())
    return torch.device("cpu")


def flatten_params(weights, biases):
    """Concatenate every non-None weight / bias into one fp32 vector plus the
    shapes needed to split it again."""
    parts, shapes = [], []
    for w, b in zip(weights, biases):
        for t in (w, b):
            if t is None:
                shapes.append(None)
            else:
                a = np.ascontiguousarray(t, dtype=np.float32)
                shapes.append(a.shape)
                parts.append(a.ravel())
    flat = np.concatenate(parts) if parts else np.zeros(0, np.float32)
    return flat, shapes


def unflatten_params(flat, shapes):
    ws, bs, off = [], [], 0
    out = []
    for shp in shapes:
        if shp is None:
            out.append(None)
            continue
        n = int(np.prod(shp))
        out.append(flat[off:off + n].reshape(shp))
        off += n
    for i in range(0, len(out), 2):
        ws.append(out[i])
        bs.append(out[i + 1])
    return ws, bs


def broadcast_params(net, rank, src=0, make=None):
    """Rank `src` builds the parameters (synth.net_params, or `make()`), then one
    broadcast of the flat buffer.  Returns (weights, biases, broadcast_ms)."""
    import torch
    import torch.distributed as dist
    import synth
    dev = _device()
    if rank == src:
        w, b = make() if make else synth.net_params(net)
        flat, shapes = flatten_params(w, b)
        meta = [flat.size, shapes]
    else:
        meta = [None, None]
    dist.broadcast_object_list(meta, src=src)
    size, shapes = meta
    if rank == src:
        t = torch.from_numpy(flat).to(dev)
    else:
        t = torch.empty(size, dtype=torch.float32, device=dev)
    if dev.type == "cuda":
        torch.cuda.synchronize()
    t0 = time.perf_counter()
    dist.broadcast(t, src=src)
    if dev.type == "cuda":
        torch.cuda.synchronize()
    ms = (time.perf_counter() - t0) * 1000.0
    flat = t.cpu().numpy()
    w, b = unflatten_params(flat, shapes)
    return w, b, ms


def gather_logits(local_out, world):
    """All-gather the per-rank [B_r, N] outputs (equal B_r) into [W*B_r, N]."""
    import torch
    import torch.distributed as dist
    g = torch.empty((world * local_out.shape[0],) + tuple(local_out.shape[1:]),
                    dtype=local_out.dtype, device=local_out.device)
    dist.all_gather_into_tensor(g, local_out.contiguous())
    return g


def free_port():
    import socket
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def torchrun_command(n_procs, script_argv, port=None, python=None):
    """The one-node launch line `bench.py --gpus N` re-executes itself with
    when it is started without torchrun: one process per GPU, rendezvous on
    127.0.0.1 (the container hostname may not resolve)."""
    import sys
    return [python or sys.executable, "-m", "torch.distributed.run", "--nnodes=1",
            "--nproc-per-node", str(int(n_procs)), "--master-addr", "127.0.0.1",
            "--master-port", str(port or free_port())] + list(script_argv)


def relaunch(n_procs, script_argv, port=None, env=None):
    """Run script_argv under torchrun with n_procs ranks; returns the exit
    code (the ranks inherit stdout, so rank 0's JSON line passes through)."""
    import os
    import subprocess
    e = dict(os.environ)
    e.update(env or {})
    return subprocess.call(torchrun_command(n_procs, script_argv, port), env=e)


def check_world(expected):
    """Every rank asserts that the process group has the requested size."""
    import torch.distributed as dist
    w = dist.get_world_size() if dist.is_initialized() else 1
    if w != expected:
        raise SystemExit("world size %d != --gpus %d" % (w, expected))
    return w
