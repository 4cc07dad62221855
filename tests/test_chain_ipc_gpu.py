"""Chained row bands across PROCESSES: two ranks of a
gloo process group share one GPU; each owns a ChainLink, the links' CUDA IPC
handles are exchanged over the group (SatChain), and every call is one kernel
per rank with device-side flow control (acknowledgement words, two slots).
Rank 0 runs its band and publishes its bottom row into rank 1's link through
the IPC mapping (st.relaxed.sys), a barrier follows, rank 1 runs its band,
which reads it and writes its acknowledgement back into rank 0's link; three
epochs per pair exercise both slots and the acknowledgements.  Each rank
checks its whole band against the oracle (bit-exact / 1e-4 / 1e-12)."""
import os
import socket
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

SCRIPT = r'''
import sys, numpy as np, torch, torch.distributed as dist
sys.path.insert(0, sys.argv[1])
import oracle, satgen
import paper_conf_cluster_chenwttm18_b200 as sat
rank, world, port = int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
torch.cuda.set_device(0)
dist.init_process_group("gloo", init_method=f"tcp://127.0.0.1:{port}", rank=rank, world_size=world)
bad = 0
for dt, H, W in [(torch.uint8, 1500, 1300), (torch.float32, 1100, 900), (torch.float64, 700, 500)]:
    pair = sat.pair_of_dtype(dt)
    chain = sat.SatChain(pair, W)
    r0, r1 = sat.band_partition(H, world, rank)
    plan = sat.Plan(pair, r1 - r0, W, 1)
    for ep in range(1, 4):
        x = torch.empty((H, W), dtype=dt, device="cuda")
        satgen.fill_device(x, seed=900 + ep)            # identical on every rank (counter based)
        ref = oracle.sat(x.cpu().numpy())[r0:r1]
        for turn in range(world):                       # ranks take turns, in rank order
            if turn == rank:
                y = chain.sat(x[r0:r1], plan=plan)
                torch.cuda.synchronize()
                plan.status()                           # no bounded wait ran out
            dist.barrier()
        got = y.cpu().numpy()
        if dt == torch.uint8:
            ok = np.array_equal(got, ref)
        else:
            tol = 1e-4 if dt == torch.float32 else 1e-12
            nz = ref != 0
            ok = bool(np.all(np.abs(got[nz] - ref[nz]) / np.abs(ref[nz]) <= tol)) and np.all(got[~nz] == 0)
        if not ok:
            bad += 1
            print("MISMATCH", rank, dt, ep, flush=True)
    dist.barrier()
    chain.close()
print("RANK", rank, "BAD", bad, flush=True)
dist.destroy_process_group()
'''


def _port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def test_chain_two_processes_ipc():
    port = str(_port())
    procs = [subprocess.Popen([sys.executable, "-c", SCRIPT, ROOT, str(r), "2", port],
                              stdout=subprocess.PIPE, stderr=subprocess.PIPE, text=True)
             for r in range(2)]
    outs = []
    for p in procs:
        try:
            o, e = p.communicate(timeout=600)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append((p.returncode, o, e))
    for r, (rc, o, e) in enumerate(outs):
        assert rc == 0, f"rank {r} rc={rc}\n{o[-2000:]}\n{e[-3000:]}"
        assert f"RANK {r} BAD 0" in o, o[-2000:]
