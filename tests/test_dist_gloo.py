"""Multi-process host logic of the row-banded paths, on CPU with gloo (world 2).

The CUDA steps of sat_compute_dist / the chained bands are covered on one GPU
by test_parity_gpu.py::test_dist_virtual_ranks, tests/test_chain_gpu.py and the
two-process tests/test_chain_ipc_gpu.py.  Here two real processes check what
crosses process boundaries, driving libsat's own host code where it has any:
the band partition (libsat's sat_band_partition, reading R14), the NCCL
unique-id bootstrap over a torch process group (SatComm's protocol), the
all_gather_object exchange that SatChain uses for its IPC handles, and the carry
algebra of SURVEY Sec. 8(e) -- each rank's column totals are all-gathered, the
exclusive prefix over lower ranks is scanned horizontally, and the result must
equal the oracle's row S(r0 - 1, .).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import paper_conf_cluster_chenwttm18_b200 as sat
import satgen

H, W, SEED = 257, 301, 77


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    try:
        os.environ["MASTER_ADDR"] = "127.0.0.1"
        os.environ["MASTER_PORT"] = str(port)
        dist.init_process_group("gloo", rank=rank, world_size=world)
        r0, r1 = sat.band_partition(H, world, rank)
        spans = [None] * world
        dist.all_gather_object(spans, (r0, r1))
        # 1. local band, regenerated from global coordinates (no data exchange)
        band = satgen.generate(satgen.KIND_U8, r1 - r0, W, seed=SEED, y0=r0)
        colsum = band.astype(np.int64).sum(axis=0) & 0xFFFFFFFF  # u32 accumulator
        # 2. all-gather of the W-vectors (the one exchange of the dist path)
        gathered = [torch.zeros(W, dtype=torch.int64) for _ in range(world)]
        dist.all_gather(gathered, torch.from_numpy(colsum))
        # 3. exclusive prefix over lower ranks, horizontal inclusive prefix
        c = sum((g.numpy() for g in gathered[:rank]), np.zeros(W, dtype=np.int64))
        carry = (np.cumsum(c) & 0xFFFFFFFF).astype(np.uint32).view(np.int32)
        # the carry must be the SAT row just above the band (oracle)
        if r0 > 0:
            ref = oracle.sat_gen_rows(0, H, W, [r0 - 1], seed=SEED)[0]
        else:
            ref = np.zeros(W, dtype=np.int32)
        ok_carry = bool(np.array_equal(carry, ref))
        # 4. NCCL unique-id bootstrap as SatComm does it (rank 0 creates, broadcast)
        ok_id = None
        try:
            buf = np.zeros(sat.COMM_ID_BYTES, dtype=np.uint8)
            if rank == 0:
                st = sat.lib().sat_comm_unique_id(buf.ctypes.data)
                if st != 0:
                    raise RuntimeError("no NCCL")
            t = torch.from_numpy(buf.copy())
            dist.broadcast(t, src=0)
            ids = [None] * world
            dist.all_gather_object(ids, bytes(t.numpy()))
            ok_id = ids[0] == ids[1] and any(ids[0])
        except RuntimeError:
            ok_id = "skip"
        # 5. the SatChain handle exchange pattern (fixed-size byte strings, rank order)
        blobs = [None] * world
        dist.all_gather_object(blobs, bytes([rank]) * sat.IPC_HANDLE_BYTES)
        ok_id = ok_id if blobs == [bytes([r]) * sat.IPC_HANDLE_BYTES for r in range(world)] else False
        q.put((rank, spans, ok_carry, ok_id))
        dist.destroy_process_group()
    except Exception as e:  # report, don't hang the parent
        q.put((rank, repr(e), False, False))


def test_row_band_protocol_two_ranks():
    world = 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    results = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
    results.sort(key=lambda r: r[0])
    for rank, spans, ok_carry, ok_id in results:
        assert isinstance(spans, list), spans
        assert spans == [sat.band_partition(H, world, r) for r in range(world)]
        assert ok_carry, f"rank {rank}: carry row != oracle S(r0-1, .)"
        if ok_id != "skip":
            assert ok_id, f"rank {rank}: unique id not shared"


def test_band_partition_host_code():
    """libsat's partition (host-only C): contiguous, covering, sizes differ by
    at most one with the larger bands first (R14); invalid requests refused."""
    for h in (0, 1, 5, 257, 65536, 65537):
        for n in (1, 2, 3, 8):
            spans = [sat.band_partition(h, n, r) for r in range(n)]
            assert spans[0][0] == 0 and spans[-1][1] == h
            assert all(spans[i][1] == spans[i + 1][0] for i in range(n - 1))
            sizes = [b - a for a, b in spans]
            assert max(sizes) - min(sizes) <= (1 if h else 0) and sizes == sorted(sizes, reverse=True)
    with pytest.raises(sat.SatError):
        sat.band_partition(10, 2, 2)
    with pytest.raises(sat.SatError):
        sat.band_partition(-1, 2, 0)
