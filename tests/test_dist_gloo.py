"""Multi-process host logic of the data-parallel path on the
CPU with the gloo backend, world size 2: shard ranges, the one-time weight
broadcast (C1) and the logits gather (C3).  The GPU run uses the same code
over NCCL."""
import os
import socket

import numpy as np
import pytest
import torch.multiprocessing as mp

import synth
from paper_conf_hpca_songhcl17_b200 import dist as pdist


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def test_shard_range_partitions_the_batch():
    for gb in (1, 7, 1024, 1023):
        for world in (1, 2, 3, 8):
            spans = [pdist.shard_range(gb, world, r) for r in range(world)]
            assert spans[0][0] == 0
            for (s0, c0), (s1, _) in zip(spans, spans[1:]):
                assert s0 + c0 == s1
            assert sum(c for _, c in spans) == gb
            assert max(c for _, c in spans) - min(c for _, c in spans) <= 1


def test_flatten_roundtrip():
    net = synth.cifar_quick()
    w, b = synth.net_params(net)
    flat, shapes = pdist.flatten_params(w, b)
    w2, b2 = pdist.unflatten_params(flat, shapes)
    for x, y in zip(w + b, w2 + b2):
        if x is None:
            assert y is None
        else:
            np.testing.assert_array_equal(x, y)


def _worker(rank, world, port, q):
    import torch
    import torch.distributed as dist
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        net = synth.cifar_quick()
        # only rank 0 can build the parameters: the others must receive them
        make = (lambda: synth.net_params(net)) if rank == 0 else (lambda: (_ for _ in ()).throw(
            RuntimeError("non-root rank built parameters")))
        w, b, ms = pdist.broadcast_params(net, rank, make=make)
        ref_w, ref_b = synth.net_params(net)
        ok_w = all(np.array_equal(x, y) for x, y in zip(w[:1], ref_w[:1]))
        ok_b = np.array_equal(b[0], ref_b[0])
        # each rank's "logits" = its global image indices, gathered in rank order
        start, count = pdist.shard_range(8, world, rank)
        local = torch.arange(start, start + count, dtype=torch.float32).reshape(count, 1).repeat(1, 3)
        g = pdist.gather_logits(local, world)
        ok_g = bool((g[:, 0] == torch.arange(8, dtype=torch.float32)).all())
        q.put((rank, ok_w, ok_b, ok_g, ms >= 0))
    finally:
        dist.destroy_process_group()


def test_broadcast_and_gather_world2():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in procs]
    for p in procs:
        p.join(timeout=60)
    assert sorted(r[0] for r in res) == [0, 1]
    for r in res:
        assert all(r[1:]), r


def test_relaunch_under_torchrun_world2():
    """bench.py --gpus N without torchrun re-executes itself through
    dist.relaunch: N ranks on 127.0.0.1 that all see world size N."""
    import json
    import subprocess
    import sys
    probe = os.path.join(os.path.dirname(__file__), "_dist_probe.py")
    cmd = pdist.torchrun_command(2, [probe, "2"])
    assert cmd[1:3] == ["-m", "torch.distributed.run"] and "127.0.0.1" in cmd
    r = subprocess.run(cmd, capture_output=True, text=True, timeout=300)
    assert r.returncode == 0, r.stderr[-2000:]
    line = [l for l in r.stdout.splitlines() if l.startswith("{")][-1]
    d = json.loads(line)
    assert d["world"] == 2 and d["ranks"] == [0, 1]
    assert d["env"][0] == "127.0.0.1"
    # a world-size mismatch fails loudly
    r2 = subprocess.run(pdist.torchrun_command(2, [probe, "3"]), capture_output=True, text=True,
                        timeout=300)
    assert r2.returncode != 0
    assert sys.executable
