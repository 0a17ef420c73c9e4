"""Small workloads that drive every libfi kernel once, for compute-sanitizer
(memcheck / racecheck / synccheck) on the GPU box:

    compute-sanitizer --tool memcheck --target-processes all python tools/sanitize_run.py [--peers]

C1 and mini-C2 (SGEMM 256^3, few replicas): golden passes (interpreter and
JIT), K1 profile (+ per-opcode, approximate), K2 index (decoupled-lookback
scans), K3 select (+ approximate), K4 inject (both engines), K5 classify (fast,
slow, tolerance), a 4-launch chain and the scatter chain through K7 and K8
(interpreter and JIT page mode), permanent faults (K7 / K8), and with --peers
fi_profile_peers with two processes on one GPU (IPC, device flags)."""
from __future__ import annotations

import os
import socket
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402
import torch  # noqa: E402


def single(fi, prog, n, groups, engine, multi=False):
    dp = fi.DeviceProgram(prog)
    gt = fi.golden_run(dp, engine=engine)
    ic, cc = fi.profile(gt)
    fi.profile_opcodes(gt)
    fi.profile_approx(gt)
    idx = fi.SiteIndex(gt, ic, cc)
    sites = fi.select_sites(idx, fi.schedule(11, groups, [0, 1, 2, 3]), 0, n)
    iidx = fi.InstanceIndex(gt, fi.profile_approx(gt))
    fi.select_sites_approx(iidx, fi.schedule(12, groups, [0]), 0, n)
    cap = fi.log_capacity(gt)
    out, log = fi.inject(gt, sites, n, cap, engine=engine)
    out2 = out.clone()
    hist_tol = torch.zeros((8, 4, 3), dtype=torch.int64, device=dp.device)
    fi.classify(gt, sites, n, out, log, cap, rtol=1e-6, hist_tol=hist_tol)
    if multi:
        fi.classify_batched(gt, sites, n, out2, log, cap, engine=engine, rtol=1e-6, hist_tol=hist_tol,
                            mem_budget=1 << 30)
        pf = np.zeros(4, dtype=fi.PFAULT_DTYPE)
        pf["opcode"], pf["sm"], pf["lane"], pf["mask"], pf["n_sm"] = 16, [0, 1, 2, 3], [1, 5, 9, 30], 1 << 22, 4
        fi.inject_permanent(gt, pf)
        fi.inject_permanent_batched(gt, pf, mem_budget=1 << 30)
    torch.cuda.synchronize()
    r = fi.as_numpy(out, fi.INJ_DTYPE, n)["outcome"]
    del gt, dp, out, out2, log, sites, idx, iidx
    torch.cuda.empty_cache()
    return r


def _peer(rank, world, port):
    import torch.distributed as dist
    from fi_inputs import programs as P
    from paper_conf_dsn_0002hsvk21_b200 import fi
    from paper_conf_dsn_0002hsvk21_b200.campaign import Campaign
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    torch.cuda.set_device(0)
    camp = Campaign(P.c1(), 7, [fi.G_GP], [0, 1, 2, 3], 32, rank, world, "cuda:0", exchange="peers")
    for _ in range(2):
        dist.barrier()
        camp.step()
        torch.cuda.synchronize()
        dist.barrier()
    camp.peers.close()
    dist.destroy_process_group()


def main():
    from fi_inputs import programs as P
    from paper_conf_dsn_0002hsvk21_b200 import fi
    torch.cuda.set_device(0)
    small = "--small" in sys.argv                  # racecheck: C1 and the chain only (it is slow)
    for engine in ("interp", "jit"):
        print("C1", engine, np.bincount(single(fi, P.c1(), 64, [fi.G_GP, fi.G_FP32], engine), minlength=3))
        if small:
            print("chain", engine, np.bincount(single(fi, P.multi_instance_chain(3), 32, [fi.G_GP], engine, True),
                                               minlength=3))
            continue
        print("mini-C2", engine, np.bincount(single(fi, P.c2(full=False), 24, [fi.G_GP], engine), minlength=3))
        print("chain", engine, np.bincount(single(fi, P.multi_instance_chain(4), 48, [fi.G_GP], engine, True),
                                           minlength=3))
        print("scatter", engine, np.bincount(single(fi, P.scatter_chain(), 48, [fi.G_GP], engine, True),
                                             minlength=3))
    if "--peers" in sys.argv:
        import torch.multiprocessing as mp
        s = socket.socket()
        s.bind(("127.0.0.1", 0))
        port = s.getsockname()[1]
        s.close()
        ctx = mp.get_context("spawn")
        ps = [ctx.Process(target=_peer, args=(r, 2, port)) for r in range(2)]
        for p in ps:
            p.start()
        for p in ps:
            p.join()
            assert p.exitcode == 0
        print("peers ok")
    print("sanitize_run done")


if __name__ == "__main__":
    main()
