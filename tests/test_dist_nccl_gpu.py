"""Real multi-GPU row-banded SAT across >= 2 GPUs (skips on a 1-GPU box).

Each rank regenerates its band from global coordinates and runs, three times
with fresh data each time: sat_dist (colsum -> ncclAllGather -> carry -> band
SAT), sat_dist_chained (links bootstrapped over NCCL, then one kernel per rank
publishing into the next GPU's link over NVLink peer memory) and SatChain (the
same, bootstrapped over the torch process group).  Every rank compares its
band with the oracle streamed from row 0."""
import os
import socket

import numpy as np
import pytest

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, pair, H, W, q):
    import torch
    import torch.distributed as dist

    import oracle
    import paper_conf_cluster_chenwttm18_b200 as sat
    import satgen

    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        torch.cuda.set_device(rank)
        dist.init_process_group("nccl", rank=rank, world_size=world,
                                device_id=torch.device("cuda", rank))
        comm = sat.SatComm()
        chain = sat.SatChain(pair, W)
        r0, r1 = sat.band_partition(H, world, rank)
        dt = {0: torch.uint8, 1: torch.float32, 2: torch.float64}[pair]
        rows = list(range(r0, r1))
        ok, why = True, ""
        for it in range(3):
            band = torch.empty((r1 - r0, W), dtype=dt, device="cuda")
            satgen.fill_device(band, seed=5 + it, y0=r0)
            ref = oracle.sat_gen_rows(pair, H, W, rows, seed=5 + it)
            for name, fn in (("sat_dist", lambda: sat.sat_dist(band, comm)),
                             ("sat_dist_chained", lambda: sat.sat_dist_chained(band, comm)),
                             ("SatChain", lambda: chain.sat(band))):
                out = fn()
                torch.cuda.synchronize()
                got = out.cpu().numpy()
                if pair == 0:
                    good = np.array_equal(got, ref)
                else:
                    tol = 1e-4 if pair == 1 else 1e-12
                    good = float(np.max(np.abs(got - ref) / np.abs(ref))) <= tol
                if not good:
                    ok, why = False, f"{name} iteration {it}"
        chain.close()
        comm.close()
        dist.destroy_process_group()
        q.put((rank, ok, why))
    except Exception as e:
        q.put((rank, False, repr(e)))


@pytest.mark.parametrize("pair", [0, 1, 2])
def test_sat_dist_nccl(pair):
    import torch
    import torch.multiprocessing as mp

    world = min(torch.cuda.device_count(), 4)
    if world < 2:
        pytest.skip("needs >= 2 GPUs")
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    H, W = 3001, 2049  # every rank holds >= 1 row
    procs = [ctx.Process(target=_worker, args=(r, world, port, pair, H, W, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    for rank, ok, err in res:
        assert ok, f"rank {rank}: {err}"
