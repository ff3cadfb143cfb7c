"""Row-partitioned C = A^2 through the product callables (spgemm_row_partition and the CUDA
two-phase SpGEMM) with two ranks sharing cuda:0 over gloo (NCCL needs one GPU per rank; the
box has one) — -m gpu.  Concatenated shards must equal the oracle bit-exactly (int values)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _port():
    with socket.socket() as s:
        s.bind(("127.0.0.1", 0))
        return s.getsockname()[1]


def _worker(rank, world, port, name, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import synth
        import paper_conf_icpp_nagasakanm17_b200 as P
        from paper_conf_icpp_nagasakanm17_b200.dist import (cuda_local_multiply, cuda_partition,
                                                            distributed_spgemm)
        torch.cuda.set_device(0)
        A = None
        if rank == 0:
            A = P.CsrMatrix.from_host(synth.config(name, "int"), "cuda:0", torch.float32)
        with P.Handle(0) as h:
            res, grpt = distributed_spgemm(A, None, device="cuda:0", dtype=torch.float32, square=True,
                                           partition=cuda_partition(h), local_multiply=cuda_local_multiply(h),
                                           gather_rpt=True)
            torch.cuda.synchronize()
            rpt, col, val = res.C.numpy()
        np.savez(os.path.join(out_dir, f"r{rank}.npz"), col=col, val=val, splits=np.array(res.splits),
                 grpt=grpt.cpu().numpy(), nprod=res.nprod)
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("name", ["cant", "webbase"])
def test_two_rank_row_partition(tmp_path, name):
    import oracle
    import synth
    if not torch.cuda.is_available():
        pytest.fail("needs a GPU")
    mp.spawn(_worker, args=(2, _port(), name, str(tmp_path)), nprocs=2, join=True)
    H = synth.config(name, "int").astype(np.float32)
    r_rpt, r_col, r_val, _ = oracle.spgemm(H, H, np.float32)
    _, total = oracle.nprod(H, H)
    sh = [np.load(os.path.join(tmp_path, f"r{p}.npz")) for p in range(2)]
    assert np.array_equal(sh[0]["splits"], sh[1]["splits"])
    assert np.array_equal(sh[0]["grpt"], r_rpt)
    assert np.array_equal(np.concatenate([s["col"] for s in sh]), r_col)
    assert np.array_equal(np.concatenate([s["val"] for s in sh]), r_val)
    assert sum(int(s["nprod"]) for s in sh) == total


def test_bench_sharded_two_ranks_gloo(tmp_path):
    """bench.py's N>1 path (broadcast of B, n_prod-balanced split, per-rank multiply, all-gather,
    max over ranks, e2e) with two ranks on one GPU over gloo (the driver runs it over NCCL on one GPU
    per rank); the two ranks' products must add up to the whole matrix's n_prod."""
    import json
    import subprocess
    import sys
    import oracle
    import synth
    if not torch.cuda.is_available():
        pytest.fail("needs a GPU")
    env = dict(os.environ, BENCH_BACKEND="gloo")
    r = subprocess.run([sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=2",
                        "--master-addr", "127.0.0.1", "--master-port", str(_port()), os.path.join(ROOT, "bench.py"),
                        "--gpus", "2", "--steps", "2", "--warmup", "1", "--config", "rmat16"],
                       capture_output=True, text=True, env=env, cwd=ROOT, timeout=900)
    assert r.returncode == 0, r.stderr[-3000:]
    line = json.loads([x for x in r.stdout.splitlines() if x.startswith("{")][-1])
    A = synth.config("rmat16", "uniform", 7)
    _, total = oracle.nprod(A, A)
    assert line["n_gpus"] == 2 and line["nprod"] == total and line["scaling"] == "strong"
    sp = line["multi_gpu"]["splits"]
    assert sp[0] == 0 and sp[-1] == A.m and len(sp) == 3
    assert line["e2e"]["value"] > 0 and line["gpu_launches"] > 0


def _nccl_worker(rank, world, port, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    torch.cuda.set_device(0)
    dist.init_process_group("nccl", rank=rank, world_size=world, device_id=torch.device("cuda", 0))
    try:
        import synth
        import paper_conf_icpp_nagasakanm17_b200 as P
        from paper_conf_icpp_nagasakanm17_b200.dist import (broadcast_csr, cuda_local_multiply, cuda_partition,
                                                            distributed_spgemm)
        A = P.CsrMatrix.from_host(synth.config("webbase", "int"), "cuda:0", torch.float32)
        B = broadcast_csr(A, 0, "cuda:0", torch.float32)  # NCCL chunked broadcast (sizes, rpt, col, val)
        with P.Handle(0) as h:
            res, grpt = distributed_spgemm(A, B, device="cuda:0", dtype=torch.float32, square=False,
                                           partition=cuda_partition(h), local_multiply=cuda_local_multiply(h),
                                           gather_rpt=True)
            torch.cuda.synchronize()
            rpt, col, val = res.C.numpy()
        np.savez(os.path.join(out_dir, "nccl.npz"), col=col, val=val, grpt=grpt.cpu().numpy(),
                 nprod=res.nprod, total=res.nnz_total, b_equal=int(torch.equal(B.col, A.col)))
    finally:
        dist.destroy_process_group()


def test_nccl_backend_world_one(tmp_path):
    """The product's collective calls (chunked broadcast of B, all_gather of the shard counts and
    rpt blocks) on the NCCL backend — one rank on the box's one GPU (ranks that wait on each other
    must not share a GPU); results equal the oracle bit-exactly (int values)."""
    import oracle
    import synth
    if not torch.cuda.is_available():
        pytest.fail("needs a GPU")
    mp.spawn(_nccl_worker, args=(1, _port(), str(tmp_path)), nprocs=1, join=True)
    H = synth.config("webbase", "int").astype(np.float32)
    r_rpt, r_col, r_val, _ = oracle.spgemm(H, H, np.float32)
    got = np.load(os.path.join(tmp_path, "nccl.npz"))
    assert int(got["b_equal"]) == 1
    assert np.array_equal(got["grpt"], r_rpt)
    assert np.array_equal(got["col"], r_col) and np.array_equal(got["val"], r_val)
    assert int(got["total"]) == r_col.size
