"""Multi-GPU C = A*B by n_prod-balanced row blocks of A.

Rows of C are independent (Alg. 1 loops over rows of A), so the only exchange
steps are replicating B (and A when it lives on one rank) and exchanging the per-rank nnz(C)
counts.  One process per GPU (torch.distributed, NCCL over NVLink/NVSwitch):

  1. broadcast B (and A) from `src` — the sizes first, then rpt / col / val in 64 MB chunks;
  2. the n_prod-balanced split points (spgemm_row_partition) are computed on `src` while the
     chunks of step 1 are in flight, then broadcast (P+1 integers);
  3. rank p runs the two-phase SpGEMM on rows [s_p, s_{p+1}) of A as a zero-copy slice
     (a_rpt[0] != 0 is allowed by the C ABI);
  4. all_gather of the P nnz counts -> each rank's offset into the global C;
  5. optionally all_gather of the rpt blocks (global rpt of C); col/val stay sharded.

The local multiply and the partition are passed in as callables, so the same driver runs on
NCCL with the CUDA library (product) and on gloo in CPU tests (with the test's own reference).
"""
from __future__ import annotations

from dataclasses import dataclass
from typing import Callable, Optional

import torch
import torch.distributed as dist

from .spgemm import CsrMatrix


@dataclass
class ShardResult:
    rank: int
    world: int
    row0: int                 # first global row of this shard
    row1: int                 # one past the last
    C: CsrMatrix              # local block: rows [row0, row1) of C, local rpt (starts at 0)
    nnz_offset: int           # offset of this block's entries in the global C
    nnz_total: int            # nnz(C)
    nprod: int                # intermediate products of this shard
    splits: list


BCAST_CHUNK_BYTES = 64 << 20  # NCCL broadcast granularity (many in flight; large tensors pipelined)


def _bcast_chunked(t: torch.Tensor, src: int, group=None, chunk_bytes: int = BCAST_CHUNK_BYTES, wait: bool = True):
    """Broadcast a contiguous tensor in chunks (asynchronous ops, waited together), so a
    gigabyte-sized B is pipelined through the collective instead of one monolithic call.
    wait=False returns the pending works (the caller overlaps other work with them)."""
    flat = t.view(-1)
    per = max(1, chunk_bytes // max(1, t.element_size()))
    works = [dist.broadcast(flat[i:i + per], src, group=group, async_op=True) for i in range(0, flat.numel(), per)]
    if not wait:
        return works
    for w in works:
        w.wait()
    return []


def broadcast_csr(M: Optional[CsrMatrix], src: int, device, dtype, group=None, wait: bool = True):
    """Replicate a CSR matrix held by rank `src` on every rank of `group` (sizes first, then
    rpt / col / val in chunks).  wait=False returns (matrix, pending works): the arrays are valid
    once the works are waited."""
    rank = dist.get_rank(group)
    meta = torch.zeros(3, dtype=torch.int64, device=device)
    if rank == src:
        meta[0], meta[1], meta[2] = M.m, M.n, M.nnz
    dist.broadcast(meta, src, group=group)
    m, n, nnz = (int(x) for x in meta.tolist())
    if rank == src:
        rpt, col, val = M.rpt.to(device), M.col.to(device), M.val.to(device)
    else:
        rpt = torch.empty(m + 1, dtype=torch.int64, device=device)
        col = torch.empty(nnz, dtype=torch.int32, device=device)
        val = torch.empty(nnz, dtype=dtype, device=device)
    works = []
    for t in (rpt, col, val):
        if t.numel():
            works += _bcast_chunked(t, src, group, wait=wait)
    Md = CsrMatrix(m, n, rpt, col, val)
    return Md if wait else (Md, works)


_bcast_csr = broadcast_csr


def broadcast_and_partition(A: Optional[CsrMatrix], B: Optional[CsrMatrix], *, src: int, device, dtype, world: int,
                            partition: Callable[[CsrMatrix, CsrMatrix, int], list], square: bool = False,
                            group=None):
    """Replicate B (and A) from `src` and agree on the n_prod-balanced split points, with the
    n_prod pass overlapped with the broadcast: `src` holds both matrices, so it computes the split
    while the chunks are in flight (collective stream) and sends the P+1 points afterwards; the
    other ranks only receive.  Returns (A, B, splits) on every rank."""
    rank = dist.get_rank(group)
    Bd, works = broadcast_csr(B if not square else A, src, device, dtype, group, wait=False)
    if square:
        Ad = Bd
    else:
        Ad, wa = broadcast_csr(A, src, device, dtype, group, wait=False)
        works += wa
    sp = torch.zeros(world + 1, dtype=torch.int64, device=device)
    if rank == src:  # the local copies are complete on src: no need to wait for the collective
        sp.copy_(torch.as_tensor([int(x) for x in partition(Ad, Bd, world)], dtype=torch.int64))
    for w in works:
        w.wait()
    dist.broadcast(sp, src, group=group)
    return Ad, Bd, [int(x) for x in sp.tolist()]


def row_slice(A: CsrMatrix, r0: int, r1: int) -> CsrMatrix:
    """Rows [r0, r1) of A without copying col/val (rpt values keep their global offsets)."""
    return CsrMatrix(r1 - r0, A.n, A.rpt[r0:r1 + 1].contiguous(), A.col, A.val)


def distributed_spgemm(A: Optional[CsrMatrix], B: Optional[CsrMatrix], *, device, dtype=torch.float32,
                       src: int = 0, square: bool = False,
                       partition: Callable[[CsrMatrix, CsrMatrix, int], list],
                       local_multiply: Callable[[CsrMatrix, CsrMatrix], tuple],
                       gather_rpt: bool = False, group=None):
    """C = A*B row-partitioned over the ranks of `group`.

    A/B need only exist on `src` (None elsewhere); `square=True` means B is A (C = A^2, one
    broadcast).  partition(A, B, P) -> P+1 split points; local_multiply(A_rows, B) ->
    (CsrMatrix C_rows, nprod).  Returns a ShardResult (and the global rpt when gather_rpt)."""
    rank, world = dist.get_rank(group), dist.get_world_size(group)
    Ad, Bd, splits = broadcast_and_partition(A, B, src=src, device=device, dtype=dtype, world=world,
                                             partition=partition, square=square, group=group)
    r0, r1 = splits[rank], splits[rank + 1]
    C, nprod = local_multiply(row_slice(Ad, r0, r1), Bd)
    counts = torch.tensor([C.nnz], dtype=torch.int64, device=device)
    allc = [torch.zeros_like(counts) for _ in range(world)]
    dist.all_gather(allc, counts, group=group)
    allc = [int(c.item()) for c in allc]
    res = ShardResult(rank, world, r0, r1, C, sum(allc[:rank]), sum(allc), int(nprod), splits)
    if not gather_rpt:
        return res
    # global rpt: pad every block to the largest block, all_gather, stitch with offsets
    width = max(splits[p + 1] - splits[p] for p in range(world))
    mine = torch.zeros(width + 1, dtype=torch.int64, device=device)
    mine[:r1 - r0 + 1] = C.rpt.to(device) + res.nnz_offset
    blocks = [torch.zeros_like(mine) for _ in range(world)]
    dist.all_gather(blocks, mine, group=group)
    parts = [blocks[0][:1]] + [blocks[p][1:splits[p + 1] - splits[p] + 1] for p in range(world)]
    return res, torch.cat(parts)


def cuda_partition(handle):
    """partition() for the product path: spgemm_row_partition on this rank's GPU."""
    def part(A, B, P):
        return handle.row_partition(A, B, P).tolist()
    return part


def cuda_local_multiply(handle):
    """local_multiply() for the product path: the two-phase SpGEMM of this rank's rows."""
    def mult(Arows, B):
        C = handle.multiply(Arows, B)
        return C, handle.nprod
    return mult
