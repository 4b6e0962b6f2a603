"""Multi-GPU sharding of the PolyHankel forward convolution.

Images are independent units (Eq. 12 applies per batch item, P.1396-1403),
and so are output channels (each (n,k) product polynomial is its own), so the
path shards without any exchange in its arithmetic:

  * batch mode (N >= world): rank r computes images [n0, n1) with the full
    filters; the output shard stays on its rank (data-parallel inference) --
    no collective on the data path.
  * output-channel mode (N < world, e.g. N=1 layers): rank r computes filters
    [k0, k1) for all images and the K-blocks are all-gathered (NCCL over
    NVLink on GPUs).  For N=1, rank-ordered K blocks are exactly NCHW.

One process per GPU (torch.distributed); PyTorch supplies the process group
and the collective, the convolution itself runs in the C-ABI library.  The
per-shard compute is injectable only so the CPU tests can drive the layout
logic with gloo; the default is the CUDA path.
"""
from __future__ import annotations

from dataclasses import dataclass


@dataclass(frozen=True)
class Shard:
    mode: str       # "batch" or "kshard"
    n0: int
    n1: int
    k0: int
    k1: int
    k_pad: int      # K rounded up to a multiple of world (kshard mode), else K


def shard_plan(N: int, K: int, world: int, rank: int, mode: str = "auto") -> Shard:
    """Which images / output channels rank `rank` of `world` computes (mode "auto": batch
    when N >= world, else output channels; "batch" / "kshard" force one)."""
    if world < 1 or not (0 <= rank < world) or N < 1 or K < 1 or mode not in ("auto", "batch", "kshard"):
        raise ValueError("bad shard request")
    if mode == "batch" and N < world:
        raise ValueError("batch sharding needs N >= world")
    if mode == "batch" or (mode == "auto" and N >= world):
        base, extra = divmod(N, world)  # uneven shards: the first `extra` ranks take one more image
        n0 = rank * base + min(rank, extra)
        n1 = n0 + base + (1 if rank < extra else 0)
        return Shard("batch", n0, n1, 0, K, K)
    kb = -(-K // world)  # equal blocks (all-gather needs equal sizes); the tail block is padded
    k0 = min(rank * kb, K)
    k1 = min(k0 + kb, K)
    return Shard("kshard", 0, N, k0, k1, kb * world)


def _cuda_compute(x, w, stride, padding, math, out=None):
    """The CUDA path; `out` (optional) receives the result in place (polyconv_forward writes it)."""
    from . import conv2d
    return conv2d(x, w, stride=stride, padding=padding, math=math, out=out)


def _fused_kshard(x, w_loc, sh, kb, K, stride, padding, math, group, world, rank):
    """f4: every rank's K-block stored by its MAC epilogue straight into all ranks' outputs
    (torch symmetric memory: peer buffers mapped over NVLink), then one cross-rank barrier."""
    import torch
    import torch.distributed as dist
    import torch.distributed._symmetric_memory as symm_mem
    from . import Plan
    N = x.shape[0]
    P, Q = _out_hw(x, w_loc, stride, padding)
    y = symm_mem.empty((N, kb * world, P, Q), dtype=x.dtype, device=x.device)
    hdl = symm_mem.rendezvous(y, group if group is not None else dist.group.WORLD)
    io = "bf16" if x.dtype == torch.bfloat16 else "f32"
    key = ("scatter", tuple(x.shape), tuple(w_loc.shape), tuple(stride), tuple(padding), math, io, x.device.index or 0)
    plan = _SCATTER_PLANS.get(key)
    if plan is None:
        plan = _SCATTER_PLANS[key] = Plan(x.shape, w_loc.shape, stride, padding, math, io, x.device.index or 0,
                                          kernel="tc_hankel")
    plan.forward_scatter(x, w_loc, list(hdl.buffer_ptrs), kb * world, rank * kb)
    hdl.barrier()  # every rank's stores have landed in every buffer
    return sh, y[:, :K]


_SCATTER_PLANS: dict = {}


def sharded_forward(x, w, stride=(1, 1), padding=(0, 0), math="bf16", group=None, compute=None, mode="auto",
                    fused=False):
    """Distributed forward.  x: the FULL input batch [N][C][H][W] as seen by every
    rank (batch mode slices it; pass only the local images with N >= world for
    zero-copy use through `local_batch`), w: full filters.  Returns
    (shard, y): in batch mode y is the local shard [n1-n0][K][P][Q]; in
    output-channel mode y is the full gathered output [N][K][P][Q].

    `compute(x, w, stride, padding, math, out)` runs one shard and writes `out` when given.
    Output-channel mode computes the local block straight into the all-gather's send buffer
    (the last rank's filter block is zero-padded to the common block size, so its padding
    channels come out zero without a fill); for N = 1 the rank-ordered blocks are NCHW and
    NCCL gathers straight into the output.

    fused=True (CUDA, NCCL group, output-channel mode): the all-gather is fused into the MAC
    epilogue (`Plan.forward_scatter` into symmetric-memory buffers of every rank) -- no
    separate collective; SURVEY §8(e)/(f) f4."""
    import torch
    import torch.distributed as dist
    compute = compute or _cuda_compute
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    N, K = x.shape[0], w.shape[0]
    sh = shard_plan(N, K, world, rank, mode)
    if sh.mode == "batch":
        return sh, compute(x[sh.n0:sh.n1].contiguous(), w, stride, padding, math)
    kb = sh.k_pad // world
    P, Q = _out_hw(x, w, stride, padding)
    w_loc = w[sh.k0:sh.k1]
    if sh.k1 - sh.k0 < kb:  # tail block: zero filters for the padding channels
        w_loc = torch.cat([w_loc, w.new_zeros((kb - (sh.k1 - sh.k0),) + tuple(w.shape[1:]))])
    if fused:
        from . import PolyconvError, NOT_SUPPORTED
        try:
            return _fused_kshard(x, w_loc.contiguous(), sh, kb, K, stride, padding, math, group, world, rank)
        except PolyconvError as e:  # a plan whose kernel does not store to peers: the NCCL gather
            if e.status != NOT_SUPPORTED:
                raise
    send = torch.empty((N, kb, P, Q), dtype=x.dtype, device=x.device)
    compute(x, w_loc.contiguous(), stride, padding, math, send)
    # gather the K blocks: [world][N][kb][P][Q] -> [N][K][P][Q]
    if dist.is_initialized() and dist.get_backend(group) == "nccl":
        if N == 1:
            y = torch.empty((1, world * kb, P, Q), dtype=x.dtype, device=x.device)
            dist.all_gather_into_tensor(y.view(world, kb, P, Q), send.view(kb, P, Q), group=group)
            return sh, y[:, :K]
        out = torch.empty((world * N, kb, P, Q), dtype=x.dtype, device=x.device)
        dist.all_gather_into_tensor(out, send, group=group)
        blocks = out.reshape(world, N, kb, P, Q)
    else:
        parts = [torch.empty_like(send) for _ in range(world)]
        if dist.is_initialized():
            dist.all_gather(parts, send, group=group)
        else:
            parts = [send]
        blocks = torch.stack(parts)
    y = blocks.permute(1, 0, 2, 3, 4).reshape(N, world * kb, P, Q)[:, :K]
    return sh, y.contiguous()


def _out_hw(x, w, stride, padding):
    H, W = x.shape[2], x.shape[3]
    R, S = w.shape[2], w.shape[3]
    return (H + 2 * padding[0] - R) // stride[0] + 1, (W + 2 * padding[1] - S) // stride[1] + 1
