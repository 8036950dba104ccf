"""Multi-rank host logic on CPU with the gloo backend, world size 2.

Every rank derives the same cuts (closest work prefix, PAPER L216-L218 / L106) and the same sampled
threshold from the same inputs and seed, without exchanging them ("does not require any
runtime communication"); the row blocks are computed independently (oracle on CPU here) and
assembled with the exact arithmetic sg_gather uses on the GPU (sg_gather_layout, host-only C) —
the concatenation must equal the single-process C bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q, split="flops"):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        import sginputs as gen
        import paper_conf_icpp_hardhikbrks17_b200 as sg
        A = gen.config("rmat11")
        w = oracle.row_work(A, A)
        cm = oracle.CostModel(**sg.sg_default_cost_model().as_dict())
        smp = oracle.sampled_threshold(A, A, 0.05, 3, cm, w_all=w)
        thr = smp.thr
        if split == "cost":  # cost-weighted split with the default partition model
            pm = oracle.CostModel(**sg.sg_default_partition_model().as_dict())
            cuts, _ = oracle.partition_cost(pm, thr, oracle.sample_comp(smp), w, np.diff(A.row_ptr), world)
        else:
            cuts = oracle.partition(w, world)
        mine = [cuts.tolist(), thr]
        every = [None] * world
        dist.all_gather_object(every, mine)
        same = all(e == mine for e in every)
        rb, re = int(cuts[rank]), int(cuts[rank + 1])
        R = oracle.spgemm(A, A, rows=np.arange(rb, re))
        lays = [None] * world
        dist.all_gather_object(lays, (rb, re, R.nnz))
        begin, off, n, total = sg.sg_gather_layout(lays)
        parts = [None] * world
        dist.all_gather_object(parts, (R.row_ptr, R.col, R.val))
        rp = np.zeros(n + 1, dtype=np.int64)
        col = np.zeros(total, dtype=np.int32)
        val = np.zeros(total, dtype=np.float64)
        for r, (prp, pcol, pval) in enumerate(parts):
            rows = lays[r][1] - lays[r][0]
            rp[begin[r]:begin[r] + rows] = prp[:-1] + off[r]
            col[off[r]:off[r + 1]] = pcol
            val[off[r]:off[r + 1]] = pval
        rp[n] = total
        q.put((rank, same, rp, col, val, cuts.tolist(), lays))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("split", ["flops", "cost"])
def test_two_rank_partition_and_assembly(split):
    import oracle
    import sginputs as gen
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, 2, port, q, split)) for r in range(2)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
    A = gen.config("rmat11")
    whole = oracle.spgemm(A, A)
    for rank, same, rp, col, val, cuts, lays in res:
        assert same, "ranks derived different cuts / thresholds"
        assert np.array_equal(rp, whole.row_ptr)
        assert np.array_equal(col, whole.col)
        assert np.array_equal(val, whole.val)
        assert cuts[0] == 0 and cuts[-1] == A.nrows and 0 < cuts[1] < A.nrows


def test_gather_layout_rejects_gaps_and_overlaps():
    import paper_conf_icpp_hardhikbrks17_b200 as sg
    b, off, n, tot = sg.sg_gather_layout([(0, 5, 10), (5, 9, 3), (9, 9, 0)])
    assert list(b) == [0, 5, 9] and list(off) == [0, 10, 13, 13] and n == 9 and tot == 13
    for bad in ([(1, 5, 1)], [(0, 5, 1), (6, 9, 2)], [(0, 5, 1), (4, 9, 2)]):
        with pytest.raises(sg.SgError, match="SHAPE"):
            sg.sg_gather_layout(bad)
