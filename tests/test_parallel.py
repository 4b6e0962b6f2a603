"""Multi-process sharding logic on CPU with the gloo backend,
world size 2.  The per-shard compute is the fp64 oracle here (test-only); on
GPUs the same planner/gather code runs the C-ABI library over NCCL."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synth
from paper_conf_cgo_xuzc025_b200.parallel import shard_plan, sharded_forward


@pytest.mark.parametrize("N,K,world", [(32, 128, 8), (7, 64, 2), (256, 64, 8), (1, 128, 8), (1, 10, 4),
                                       (3, 5, 4), (5, 3, 8)])
def test_shard_plan_partitions_work(N, K, world):
    seen = np.zeros((N, K), int)
    for r in range(world):
        s = shard_plan(N, K, world, r)
        seen[s.n0:s.n1, s.k0:s.k1] += 1
        if s.mode == "batch":
            assert s.k0 == 0 and s.k1 == K
        else:
            assert s.k_pad % world == 0 and s.k_pad >= K
    assert (seen == 1).all()


def _oracle_compute(x, w, stride, padding, math, out=None):
    y = torch.from_numpy(oracle.conv2d(x.numpy(), w.numpy(), stride, padding))
    if out is None:
        return y
    out.copy_(y)
    return out


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        out = {}
        # batch mode: N >= world, each rank its images, no collective
        shape = synth.ConvShape("b", 5, 3, 7, 6, 4, 3, 3, 1, 1, 1, 1)
        x, w = synth.make_inputs(shape, 11, "int")
        xt, wt = torch.from_numpy(x).double(), torch.from_numpy(w).double()
        sh, y = sharded_forward(xt, wt, shape.stride, shape.padding, "fp32", compute=_oracle_compute)
        out["batch"] = (sh.mode, sh.n0, sh.n1, y.numpy())
        # output-channel mode: N=1 < world, K-blocks all-gathered (K not divisible by world)
        shape = synth.ConvShape("k", 1, 4, 9, 8, 5, 3, 3, 2, 2, 1, 1)
        x, w = synth.make_inputs(shape, 12, "int")
        xt, wt = torch.from_numpy(x).double(), torch.from_numpy(w).double()
        sh, y = sharded_forward(xt, wt, shape.stride, shape.padding, "fp32", compute=_oracle_compute)
        out["kshard"] = (sh.mode, sh.k0, sh.k1, y.numpy())
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_gloo_world2_batch_and_kshard():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=180) for _ in range(2))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    # batch: the two local shards are the oracle's result for those images
    shape = synth.ConvShape("b", 5, 3, 7, 6, 4, 3, 3, 1, 1, 1, 1)
    x, w = synth.make_inputs(shape, 11, "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    got = np.concatenate([res[r]["batch"][3] for r in range(2)])
    assert [res[r]["batch"][:3] for r in range(2)] == [("batch", 0, 3), ("batch", 3, 5)]
    assert np.array_equal(got, ref)
    # kshard: every rank holds the full gathered output
    shape = synth.ConvShape("k", 1, 4, 9, 8, 5, 3, 3, 2, 2, 1, 1)
    x, w = synth.make_inputs(shape, 12, "int")
    ref = oracle.conv2d(x, w, shape.stride, shape.padding)
    for r in range(2):
        mode, k0, k1, y = res[r]["kshard"]
        assert mode == "kshard"
        assert np.array_equal(y, ref)
    assert (res[0]["kshard"][1:3], res[1]["kshard"][1:3]) == ((0, 3), (3, 5))


@pytest.mark.gpu
def test_sharded_forward_single_rank_cuda():
    """World size 1: the CUDA path through the same entry point."""
    shape = synth.ConvShape("g", 2, 64, 14, 14, 128, 3, 3, 1, 1, 1, 1)
    x, w = synth.make_inputs(shape, 13, "int")
    sh, y = sharded_forward(torch.from_numpy(x).cuda(), torch.from_numpy(w).cuda(), shape.stride, shape.padding,
                            "bf16")
    torch.cuda.synchronize()
    assert sh.mode == "batch"
    assert np.array_equal(y.cpu().numpy(), oracle.conv2d(x, w, shape.stride, shape.padding))
