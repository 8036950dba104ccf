"""NEXT #3: the assembled C in NCCL symmetric windows (include/sg.h sg_sym_c_*): the
numeric kernels write the rank's rows straight into its window, one push kernel stores them into every
LSA peer's window, an LSA barrier closes it (Alg. 2 l.7). On this one-GPU box the
communicator has one rank (the LSA team is the rank itself), so the test checks the functional path —
windows, layout exchange, the fused numeric epilogue, the push kernel and its barrier — against the
oracle; multi-GPU scaling of the path is unmeasured here."""
import os
import socket

import numpy as np
import pytest
import torch

import oracle
import sginputs as gen
from _util import compare_rows

pytestmark = pytest.mark.gpu

sg = pytest.importorskip("paper_conf_icpp_hardhikbrks17_b200")


@pytest.fixture(scope="module")
def comm():
    import torch.distributed as dist
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    dist.barrier()
    yield dist.group.WORLD._get_backend(dev)._comm_ptr()
    dist.destroy_process_group()


@pytest.mark.parametrize("name,dtype", [("rmat14", "f64"), ("rmat14", "f32"), ("C1", "f64")])
def test_symmetric_assembly_equals_oracle(comm, name, dtype):
    A = gen.config(name, dtype=dtype)
    dA = sg.DeviceCSR.from_host(A)
    thr, _ = sg.sg_sample_threshold(dA, dA, 0.05, 2)
    plan = sg.sg_symbolic(dA, dA, thr)
    S = sg.SymC(comm, A.nrows, plan.nnz + 17, torch.float64 if dtype == "f64" else torch.float32)
    off, tot = S.layout(plan)
    assert off == 0 and tot == plan.nnz
    S.numeric_into(plan, dA, dA)
    S.assemble(plan)
    rp, col, val = S.tensors()
    torch.cuda.synchronize()
    R = oracle.spgemm(A, A, with_absmag=True)
    rp = rp.cpu().numpy()
    assert np.array_equal(rp, R.row_ptr)
    compare_rows(rp, col.cpu().numpy(), val.cpu().numpy(), R, dtype)
    S.destroy()
    plan.destroy()


def test_symmetric_assembly_capacity_and_order_errors(comm):
    A = gen.config("C1")
    dA = sg.DeviceCSR.from_host(A)
    plan = sg.sg_symbolic(dA, dA, 16)
    S = sg.SymC(comm, A.nrows, plan.nnz - 1)  # too small
    with pytest.raises(sg.SgError, match="SHAPE"):
        S.layout(plan)
    with pytest.raises(sg.SgError, match="INVALID_ARG"):
        S.assemble(plan)  # layout did not succeed
    S.destroy()
    S = sg.SymC(comm, A.nrows + 1, plan.nnz)  # wrong row count
    with pytest.raises(sg.SgError, match="SHAPE"):
        S.layout(plan)
    S.destroy()
    plan.destroy()
