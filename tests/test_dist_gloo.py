"""world_size-2 gloo tests (CPU) of the multi-GPU orchestration in
paper_conf_sosp_kamathb21_b200.dist: uneven all-to-all routing, variable all-gather, reductions and
the end-to-end sharded check with a CPU stand-in stage, compared with the oracle on the full trace."""
import os
import socket
import tempfile

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, outdir, case):
    import sys

    here = os.path.dirname(os.path.abspath(__file__))
    sys.path.insert(0, here)
    sys.path.insert(0, os.path.dirname(here))
    import torch.distributed as dist

    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_sosp_kamathb21_b200 import dist as D

    comm = D.TorchComm()
    if case == "exchange":
        # rank r sends (r+1)*(d+1) rows to rank d, each row tagged (src, dst, i)
        rows, counts = [], []
        for d in range(world):
            c = (rank + 1) * (d + 1) + (3 if d == 0 else 0)
            counts.append(c)
            rows += [[rank, d, i, 0] for i in range(c)]
        recv = comm.all_to_all_var(torch.tensor(rows, dtype=torch.int32), counts)
        g = comm.all_gather_var(torch.arange(rank * 5 + 1, dtype=torch.int32).reshape(-1, 1))
        lo = comm.allreduce_u64(100 + rank, "min", "cpu")
        hi = comm.allreduce_u64(100 + rank, "max", "cpu")
        nb = comm.allreduce_u64(D.NONE64 if rank == 0 else 7, "min_none", "cpu")
        np.savez(os.path.join(outdir, f"r{rank}.npz"), recv=recv.numpy(), g=g.numpy(), red=np.array([lo, hi, nb]))
    else:
        import tracegen as tg
        import tracegen.families as F
        from cpu_stage import CpuStage

        if case.startswith("fam"):
            ev, nb, bd, _ = F.generate(int(case[3:]), 1_500_000, rate=8.0)
        else:
            ev, nb, bd = tg.random_trace(int(case[4:]), 300, n_words=20, lock_words=4, p_lock_data=0.2,
                                         weights=[12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1])
        lo, cnt = D.chunk_bounds(len(ev), world, rank)
        st = CpuStage()
        st.rank = rank
        st.load(ev[lo:lo + cnt], lo, len(ev), nb, bd)
        rep = D.sharded_detect(st, comm)
        np.save(os.path.join(outdir, f"r{rank}.npy"), rep)
    dist.destroy_process_group()


def _spawn(case, world=2):
    # spawn, not fork: the parent may already run OpenMP (tracegen), which does not survive fork
    here = os.path.dirname(os.path.abspath(__file__))
    os.environ["PYTHONPATH"] = os.pathsep.join([here, os.path.dirname(here), os.environ.get("PYTHONPATH", "")])
    with tempfile.TemporaryDirectory() as d:
        mp.start_processes(_worker, args=(world, _free_port(), d, case), nprocs=world, start_method="spawn")
        if case == "exchange":
            return [dict(np.load(os.path.join(d, f"r{r}.npz"))) for r in range(world)]
        return [np.load(os.path.join(d, f"r{r}.npy")) for r in range(world)]


def test_exchange_semantics():
    out = _spawn("exchange")
    for me in range(2):
        recv = out[me]["recv"]
        # rows from rank 0 first, then rank 1; each source's rows in order, all destined to me
        exp = []
        for src in range(2):
            c = (src + 1) * (me + 1) + (3 if me == 0 else 0)
            exp += [[src, me, i, 0] for i in range(c)]
        assert recv.tolist() == exp
        assert out[me]["g"].reshape(-1).tolist() == [0] + list(range(6))
        assert out[me]["red"].tolist() == [100, 101, 7]


@pytest.mark.parametrize("case", ["rand1", "rand2", "rand3", "fam2", "fam4"])
def test_sharded_orchestration_equals_oracle(case):
    import oracle
    import tracegen as tg
    import tracegen.families as F

    res = _spawn(case)
    assert np.array_equal(res[0], res[1])  # every rank holds the global set
    if case.startswith("fam"):
        ev, nb, bd, _ = F.generate(int(case[3:]), 1_500_000, rate=8.0)
    else:
        ev, nb, bd = tg.random_trace(int(case[4:]), 300, n_words=20, lock_words=4, p_lock_data=0.2,
                                     weights=[12, 10, 6, 10, 8, 12, 2, 2, 1, 1, 1, 1])
    want = oracle.run(ev, nb, bd)
    got = res[0]
    assert len(want) > 0
    assert [(int(r["addr"]), int(r["cur"]), int(r["prev"]), int(r["type"])) for r in got] == \
           [(int(r["addr"]), int(r["cur"]), int(r["prev"]), int(r["type"])) for r in want]
