"""ORACLE — TEST INFRASTRUCTURE ONLY.  O2: plain CPU recursive blocking.

Follows PAPER.md Listing 3 and the dense
matrix-multiply steps of §IV-A literally, on host buffers:

  myfunction(level, A(l), B(l), C(l)):
    if level == max_level:  compute_task()  -> O1 on the leaf block
    else: divide A(l) into dim_{A-x} x dim_{A-y} blocks and B(l) into
          dim_{B-x} x dim_{B-y} blocks with dim_{A-y} = dim_{B-x}
          for each C_{i,j}(l):
              setup_buffer()                     (Listing 3)
              for each block k of the dot product:
                  data_down(): copy the row-shard block A_{i,k} and the
                               column-shard block B_{k,j} to level l+1
                  northup_spawn(myfunction(l+1)) -> partial result
                  accumulate the partial sums in fp64
              data_up(): copy C_{i,j}(l+1) back to level l

`reuse_row_shard` implements P:299's optimisation (row shard m stays at
level l+1 while column shards stream); it must not change the result.

It shares no code with O1 except the leaf call, so it pins the
decomposition semantics (index arithmetic, ragged edges, accumulation)
independently of the GPU planner.  Readings: x = rows, y = columns
(R2); the last block at each level is ragged (R5).
"""
from __future__ import annotations

import numpy as np


def _ceil_div(a: int, b: int) -> int:
    return -(-a // b)


def recursive(A: np.ndarray, B: np.ndarray, levels, leaf=None,
              reuse_row_shard: bool = False, order: str = "mn") -> np.ndarray:
    """C = A B through the recursion.

    levels : list of (bm, bn, bk) for tree levels 0 .. max_level-1; the
             leaf level (max_level = len(levels)) multiplies what it receives.
    leaf   : callable(A_blk, B_blk) -> fp64 block (default: oracle O1).
    order  : "mn" (row shards outer) or "nm" (column shards outer).
    """
    if leaf is None:
        from . import gemm as leaf  # O1
    A = np.ascontiguousarray(A, dtype=np.float32)
    B = np.ascontiguousarray(B, dtype=np.float32)
    max_level = len(levels)
    M, K = A.shape
    N = B.shape[1]
    C = np.zeros((M, N), dtype=np.float64)

    def myfunction(level, A_l, B_l, C_l):
        if level == max_level:                       # get_level() == get_max_treelevel()
            C_l[...] = leaf(A_l, B_l)                 # compute_task()
            return
        bm, bn, bk = levels[level]
        m_l, k_l = A_l.shape
        n_l = B_l.shape[1]
        nx, ny, nk = _ceil_div(m_l, bm), _ceil_div(n_l, bn), _ceil_div(k_l, bk)
        pairs = [(i, j) for i in range(nx) for j in range(ny)]
        if order == "nm":
            pairs = [(i, j) for j in range(ny) for i in range(nx)]
        resident_row = None                           # row shard kept at l+1
        resident_idx = -1
        for i, j in pairs:
            r0, r1 = i * bm, min((i + 1) * bm, m_l)
            c0, c1 = j * bn, min((j + 1) * bn, n_l)
            C_child = np.zeros((r1 - r0, c1 - c0), dtype=np.float64)   # setup_buffer
            if reuse_row_shard and resident_idx != i:
                resident_row = A_l[r0:r1, :].copy()                    # data_down, once
                resident_idx = i
            for kb in range(nk):
                k0, k1 = kb * bk, min((kb + 1) * bk, k_l)
                if reuse_row_shard:
                    A_child = np.ascontiguousarray(resident_row[:, k0:k1])
                else:
                    A_child = A_l[r0:r1, k0:k1].copy()                 # data_down
                B_child = B_l[k0:k1, c0:c1].copy()                     # data_down
                partial = np.zeros((r1 - r0, c1 - c0), dtype=np.float64)
                myfunction(level + 1, A_child, B_child, partial)       # northup_spawn
                C_child += partial                                     # accumulate
            C_l[r0:r1, c0:c1] = C_child                                # data_up

    myfunction(0, A, B, C)
    return C
