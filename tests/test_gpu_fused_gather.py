"""f4: the output-channel-sharded forward with the all-gather fused into the
MAC epilogue -- polyconv_forward_scatter stores the plan's channel block at its offset in every
output buffer (peers' buffers mapped over NVLink in a multi-GPU job).  On one GPU: several local
buffers through the C-ABI, and the torch symmetric-memory path of parallel.sharded_forward at
world size 1 (NCCL).  Integer data: bit-exact against the fp64 oracle."""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import synth
from helpers import bf16_round
import paper_conf_cgo_xuzc025_b200 as pc
from paper_conf_cgo_xuzc025_b200.parallel import sharded_forward

pytestmark = pytest.mark.gpu


@pytest.mark.parametrize("shape,k_total,k_off", [
    (synth.ConvShape("blk64", 2, 64, 14, 14, 64, 3, 3, 1, 1, 1, 1), 160, 64),   # middle block
    (synth.ConvShape("blk32", 3, 32, 28, 28, 32, 3, 3, 1, 1, 1, 1), 96, 64),    # last block
    (synth.ConvShape("blk_oddw", 2, 64, 9, 7, 64, 3, 3, 1, 1, 1, 1), 128, 0)])  # odd width
def test_forward_scatter_into_several_outputs(shape, k_total, k_off):
    x, w = synth.make_inputs(shape, synth.seed_for(41, shape.K), "int")
    ref = bf16_round(oracle.conv2d(x, w, shape.stride, shape.padding))
    xt = torch.from_numpy(x).cuda().bfloat16()
    wt = torch.from_numpy(w).cuda().bfloat16()
    plan = pc.Plan(xt.shape, wt.shape, shape.stride, shape.padding, math="bf16", io_dtype="bf16",
                   kernel="tc_hankel")
    P, Q = plan.output_shape[2], plan.output_shape[3]
    ys = [torch.full((shape.N, k_total, P, Q), 7.0, dtype=torch.bfloat16, device="cuda") for _ in range(3)]
    plan.forward_scatter(xt, wt, [y.data_ptr() for y in ys], k_total, k_off)
    torch.cuda.synchronize()
    for y in ys:
        y = y.float().cpu().numpy()
        assert np.array_equal(y[:, k_off:k_off + shape.K], ref)
        # channels outside the block are untouched
        assert (y[:, :k_off] == 7).all() and (y[:, k_off + shape.K:] == 7).all()


def test_forward_scatter_errors():
    shape = synth.ConvShape("e", 1, 64, 8, 8, 64, 3, 3, 1, 1, 1, 1)
    xt = torch.zeros((1, 64, 8, 8), dtype=torch.bfloat16, device="cuda")
    wt = torch.zeros((64, 64, 3, 3), dtype=torch.bfloat16, device="cuda")
    plan = pc.Plan(xt.shape, wt.shape, shape.stride, shape.padding, math="bf16", io_dtype="bf16",
                   kernel="tc_hankel")
    y = torch.zeros((1, 128, 8, 8), dtype=torch.bfloat16, device="cuda")
    with pytest.raises(pc.PolyconvError):      # block past k_total
        plan.forward_scatter(xt, wt, [y.data_ptr()], 128, 96)
    with pytest.raises(pc.PolyconvError):      # more than 8 outputs
        plan.forward_scatter(xt, wt, [y.data_ptr()] * 9, 128, 0)
    x2 = torch.zeros((1, 64, 16, 16), dtype=torch.bfloat16, device="cuda")   # stride 2: phase mode
    p2 = pc.Plan(x2.shape, wt.shape, (2, 2), (1, 1), math="bf16", io_dtype="bf16", kernel="tc_hankel")
    with pytest.raises(pc.PolyconvError) as ei:
        p2.forward_scatter(x2, wt, [y.data_ptr()], 128, 0)
    assert ei.value.status == pc.NOT_SUPPORTED
    x32, w32 = xt.float(), wt.float()          # FP32_FMA plan: not the hankel kernel
    p32 = pc.Plan(x32.shape, w32.shape, shape.stride, shape.padding, math="fp32", io_dtype="f32")
    with pytest.raises(pc.PolyconvError) as ei:
        p32.forward_scatter(x32, w32, [y.data_ptr()], 128, 0)
    assert ei.value.status == pc.NOT_SUPPORTED


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def test_sharded_forward_fused_symmetric_memory_world1():
    """The fused output-channel path end to end: torch symmetric memory + forward_scatter +
    the cross-rank barrier, NCCL process group of one rank."""
    import torch.distributed as dist
    own = not dist.is_initialized()
    if own:
        os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
        os.environ["MASTER_PORT"] = str(_free_port())
        dist.init_process_group("nccl", rank=0, world_size=1, device_id=torch.device("cuda", 0))
    try:
        shape = synth.ConvShape("fz", 2, 64, 14, 14, 96, 3, 3, 1, 1, 1, 1)
        x, w = synth.make_inputs(shape, synth.seed_for(42, 0), "int")
        sh, y = sharded_forward(torch.from_numpy(x).cuda().bfloat16(), torch.from_numpy(w).cuda().bfloat16(),
                                shape.stride, shape.padding, "bf16", mode="kshard", fused=True)
        torch.cuda.synchronize()
        assert sh.mode == "kshard" and (sh.k0, sh.k1) == (0, 96)
        assert np.array_equal(y.float().cpu().numpy(), bf16_round(oracle.conv2d(x, w, shape.stride, shape.padding)))
    finally:
        if own:
            dist.destroy_process_group()
