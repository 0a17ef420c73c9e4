"""fi_profile_peers: the multi-GPU profile fused with its exchange —
K1 stores its chunk-count rows straight into the peer ranks' memory (IPC-mapped),
pushes partial instance counts, and the ranks meet on device flags.  Two or three
ranks share the one GPU here (processes, IPC on the same device, gloo only for the
handle exchange); counts, chunk counts, histograms and per-replica outcomes must
equal the single-rank campaign's, over several epochs."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    from fi_inputs import programs as P
    from paper_conf_dsn_0002hsvk21_b200 import fi
    from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    prog = P.c2(full=False)
    camp = Campaign(prog, 7, [fi.G_GP, fi.G_FP32], [0, 1, 2, 3], 96, rank, world, "cuda:0", exchange="peers")
    res = []
    for _ in range(3):                                # three epochs of the device-flag protocol
        dist.barrier()
        camp.step()
        torch.cuda.synchronize()
        dist.barrier()
        res.append((camp.inst_counts.cpu().numpy().copy(), camp.chunk_counts.cpu().numpy().copy(),
                    camp.hist.cpu().numpy().copy()))
    inj = camp.inj_np()["outcome"].copy()
    camp.peers.close()
    q.put((rank, res, camp.j0, inj))
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_profile_peers_equals_single_rank(world):
    from fi_inputs import programs as P
    from paper_conf_dsn_0002hsvk21_b200 import fi
    from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign
    ref = Campaign(P.c2(full=False), 7, [fi.G_GP, fi.G_FP32], [0, 1, 2, 3], 96, 0, 1, "cuda:0")
    ref.step()
    torch.cuda.synchronize()
    ic, cc, hist = ref.inst_counts.cpu().numpy(), ref.chunk_counts.cpu().numpy(), ref.hist.cpu().numpy()
    ref_out = ref.inj_np()["outcome"]
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    import queue as _queue
    import time
    got, t0 = [], time.time()
    while len(got) < world:
        try:
            got.append(q.get(timeout=5))
        except _queue.Empty:
            assert not any(p.exitcode not in (None, 0) for p in procs), "a rank died"
            assert time.time() - t0 < 600, "timeout"
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank, res, j0, inj in got:
        for e_ic, e_cc, e_h in res:
            assert np.array_equal(e_ic, ic), f"rank {rank}: instance counts"
            assert np.array_equal(e_cc, cc), f"rank {rank}: chunk counts"
            assert np.array_equal(e_h, hist), f"rank {rank}: histogram"
        assert np.array_equal(inj, ref_out[j0: j0 + len(inj)]), f"rank {rank}: outcomes"
