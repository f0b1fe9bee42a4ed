"""Multi-process (one process per GPU) orchestration of the point-sharded MSM.

Each rank owns the contiguous point shard [floor(r*n/W), floor((r+1)*n/W)), computes its
partial sum with msm_run_partial (an XYZZ point, msm_partial_words words), the W partials
are all-gathered over torch.distributed (NCCL over NVLink on GPUs; gloo in CPU tests), and
rank 0 adds them with msm_finalize ("only N_gpu points are left to sum").
torch is used here only as the process-group plumbing.
"""
from __future__ import annotations


def shard_bounds(n: int, world: int, rank: int) -> tuple[int, int]:
    """[off, off + count) of rank's contiguous shard."""
    off = n * rank // world
    return off, n * (rank + 1) // world - off


def gather_partials(partial, group=None):
    """All-gather one partial (1-D int32 tensor) from every rank -> [world, words] tensor
    in rank order (on the partial's device)."""
    import torch
    import torch.distributed as dist
    world = dist.get_world_size(group)
    out = torch.empty(world * partial.numel(), dtype=partial.dtype, device=partial.device)
    dist.all_gather_into_tensor(out, partial.contiguous().view(-1), group=group)
    return out.view(world, -1)


def gather_and_finalize(curve, partial, group=None):
    """Collective; returns the affine result (x, y) on rank 0 and None elsewhere."""
    import torch.distributed as dist
    from . import msm
    allp = gather_partials(partial, group)
    if allp.is_cuda:
        # the all-gather's result is ordered on torch's current stream; the library orders
        # itself only after the legacy default stream, so make the data complete here
        import torch
        torch.cuda.current_stream(allp.device).synchronize()
    if dist.get_rank(group) == 0:
        return msm.finalize(curve, allp, allp.shape[0])
    return None
