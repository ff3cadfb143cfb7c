"""Multi-process (world_size 2 and 3, gloo, CPU) tests of the row-partition driver
(paper_conf_icpp_nagasakanm17_b200/dist.py) — -m "not gpu".

The product path runs the local multiply and the partition on each rank's GPU; here the same
driver runs on gloo with the test's reference callables (the oracle, test infrastructure), and
the test checks the collective plumbing: broadcast of B, identical split points on every
rank, n_prod balance, nnz offsets from all_gather, stitched global rpt, and that the
concatenated shards equal the single-process C bit-exactly on rpt/col (integer values)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _oracle_partition(A, B, P):
    import oracle
    from synth import Csr
    rpt = A.rpt.numpy()
    Ah = Csr(A.m, A.n, rpt - rpt[0], A.col.numpy()[rpt[0]:rpt[-1]], None)
    Bh = Csr(B.m, B.n, B.rpt.numpy(), B.col.numpy(), None)
    nprod, total = oracle.nprod(Ah, Bh)
    excl = np.concatenate([[0], np.cumsum(nprod)])
    return [int(np.searchsorted(excl, (total * p) // P, side="left")) for p in range(P)] + [A.m]


def _oracle_multiply(Arows, B):
    import oracle
    from synth import Csr
    from paper_conf_icpp_nagasakanm17_b200.spgemm import CsrMatrix
    rpt = Arows.rpt.numpy()
    s, e = int(rpt[0]), int(rpt[-1])
    Ah = Csr(Arows.m, Arows.n, rpt - s, Arows.col.numpy()[s:e], Arows.val.numpy()[s:e].astype(np.float64))
    Bh = Csr(B.m, B.n, B.rpt.numpy(), B.col.numpy(), B.val.numpy().astype(np.float64))
    c_rpt, c_col, c_val, _ = oracle.spgemm(Ah, Bh, np.float64)
    _, nprod = oracle.nprod(Ah, Bh)
    return CsrMatrix(Ah.m, Bh.n, torch.from_numpy(c_rpt), torch.from_numpy(c_col),
                     torch.from_numpy(c_val)), nprod


def _worker(rank, world, port, cfg, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        from paper_conf_icpp_nagasakanm17_b200.dist import distributed_spgemm
        from paper_conf_icpp_nagasakanm17_b200.spgemm import CsrMatrix
        A = None
        if rank == 0:
            H = synth.banded(*cfg) if isinstance(cfg, tuple) else synth.webbase_like(M=cfg, seed=2, lmax=300)
            H = H.with_values("int", 1)
            A = CsrMatrix.from_host(H, device=None, dtype=torch.float64)
        res, grpt = distributed_spgemm(A, None, device="cpu", dtype=torch.float64, square=True,
                                       partition=_oracle_partition, local_multiply=_oracle_multiply,
                                       gather_rpt=True)
        np.savez(os.path.join(out_dir, f"r{rank}.npz"), rpt=res.C.rpt.numpy(), col=res.C.col.numpy(),
                 val=res.C.val.numpy(), row0=res.row0, row1=res.row1, off=res.nnz_offset, tot=res.nnz_total,
                 nprod=res.nprod, splits=np.array(res.splits), grpt=grpt.numpy())
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,cfg", [(2, (3000, 5, 40, 25, 3)), (3, 4000), (2, 1)])
def test_row_partition_driver_gloo(tmp_path, world, cfg):
    import oracle
    import synth
    mp.spawn(_worker, args=(world, _free_port(), cfg, str(tmp_path)), nprocs=world, join=True)
    H = synth.banded(*cfg) if isinstance(cfg, tuple) else synth.webbase_like(M=cfg, seed=2, lmax=300)
    H = H.with_values("int", 1)
    ref_rpt, ref_col, ref_val, _ = oracle.spgemm(H, H, np.float64)
    nprod_rows, total = oracle.nprod(H, H)
    shards = [np.load(os.path.join(tmp_path, f"r{p}.npz")) for p in range(world)]
    splits = shards[0]["splits"]
    for sh in shards:                                   # identical split points everywhere
        assert np.array_equal(sh["splits"], splits)
        assert np.array_equal(sh["grpt"], ref_rpt)      # stitched global rpt
        assert sh["tot"] == ref_rpt[-1]
    assert splits[0] == 0 and splits[-1] == H.m and np.all(np.diff(splits) >= 0)
    col = np.concatenate([sh["col"] for sh in shards])
    val = np.concatenate([sh["val"] for sh in shards])
    assert np.array_equal(col, ref_col) and np.array_equal(val, ref_val)
    offs = [int(sh["off"]) for sh in shards]
    assert offs == [int(ref_rpt[splits[p]]) for p in range(world)]
    assert sum(int(sh["nprod"]) for sh in shards) == total
    if H.m >= world * 100:                              # n_prod balance of the split
        per = [nprod_rows[splits[p]:splits[p + 1]].sum() for p in range(world)]
        assert max(per) <= total / world + nprod_rows.max()
