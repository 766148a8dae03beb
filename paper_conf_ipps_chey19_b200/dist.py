"""Multi-process (one rank per GPU, torchrun) plumbing for the C-subtree
partition of S§8(e): region bookkeeping and the optional final gather of C
(`replicate_result` in the multi-process mode) over torch.distributed
(NCCL on GPUs, gloo in the CPU tests).  No arithmetic of the GEMM happens
here: every rank's region is computed by northup_gemm through the C ABI."""
from __future__ import annotations

from . import partition, partition_region


def my_region(M: int, N: int, K: int, rank: int, world: int) -> tuple[int, int, int, int]:
    """Rows [r0, r1) and columns [c0, c1) of C owned by `rank` (northup_partition_region)."""
    return partition_region(world, M, N, K, rank) if world > 1 else (0, M, 0, N)


def gather_regions(c_region, M: int, N: int, K: int, rank: int, world: int, group=None):
    """Every rank contributes its C region (a (r1-r0) x (c1-c0) tensor) and
    receives the full M x N C: one broadcast per region (regions may differ in
    size, so all_gather's equal-count contract does not apply)."""
    import torch
    import torch.distributed as dist

    full = torch.empty((M, N), dtype=c_region.dtype, device=c_region.device)
    for root in range(world):
        r0, r1, c0, c1 = my_region(M, N, K, root, world)
        if r1 <= r0 or c1 <= c0:
            continue
        buf = c_region.contiguous() if root == rank else torch.empty(
            (r1 - r0, c1 - c0), dtype=c_region.dtype, device=c_region.device)
        dist.broadcast(buf, src=root, group=group)
        full[r0:r1, c0:c1] = buf
    return full


def grid(world: int, M: int, N: int) -> tuple[int, int]:
    return partition(world, M, N)
