"""Row bands end to end with the CUDA kernels on several ranks (config 5's
path, dist.bilateral_bands), checked against the ORACLE (VERDICT round 1,
"Next round" item 2).

The driver's GPU box has one GPU and NCCL refuses two ranks on one device, so
the ranks share cuda:0 and exchange halos over gloo through host memory
(dist.Bands' host-staged transport); everything else -- band buffers, band
views, interior/edge launches, REPEAT ring -- is the multi-GPU code path.
The concatenated band outputs must equal the oracle within 1e-5 and the
single-rank whole-image CUDA call bit for bit.
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synthetic

pytestmark = pytest.mark.gpu

MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]
H, W, SEED = 301, 263, 61


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_membarthhtke12_b200 as lop
        from paper_conf_ipps_membarthhtke12_b200 import dist as ldist
        res = {}
        for mode in MODES:
            for sigma_r in (5.0, 0.1):
                band = ldist.Bands(H, W, world, rank, 6, device="cuda", mode=mode)
                assert band.staged()
                # rows drawn on the host (the CPU and CUDA noise generators differ),
                # so the oracle below sees the same image
                band.fill(lambda a, b: synthetic.angio(H, W, seed=SEED, row_range=(a, b)).cuda())
                band.top.fill_(float("nan"))           # must be overwritten by the exchange
                band.bottom.fill_(float("nan"))
                s = torch.cuda.Stream()                # a side stream
                s.wait_stream(torch.cuda.current_stream())   # after the fill
                out = ldist.bilateral_bands(lop, band, 3.0, sigma_r, mode, constant=0.5,
                                            size=13, stream=s)
                s.synchronize()
                res[(mode, sigma_r)] = (band.y0, out.cpu().numpy())   # by value
        q.put((rank, res, lop.launch_count()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_bands_cuda_kernels_on_several_ranks_match_oracle(world):
    import paper_conf_ipps_membarthhtke12_b200 as lop
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    got = {}
    for _ in range(world):
        rank, res, launches = q.get(timeout=600)
        assert launches > 0                            # the CUDA kernels ran on every rank
        got[rank] = res
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    img = synthetic.angio(H, W, seed=SEED)
    for mode in MODES:
        for sigma_r in (5.0, 0.1):
            bands = [got[r][(mode, sigma_r)] for r in range(world)]
            assert [b[0] for b in bands] == [H * r // world for r in range(world)]
            full = np.concatenate([b[1] for b in bands])
            ref, valid = oracle.bilateral_f32(img.numpy(), 3.0, sigma_r, mode, cval=0.5, size=13)
            sel = valid if mode == "undefined" else np.ones_like(valid)
            err = float(np.abs(full[sel] - ref[sel]).max())
            assert err <= 1e-5, (mode, sigma_r, err)
            whole = lop.bilateral(img.cuda(), 3.0, sigma_r, mode, constant=0.5, size=13).cpu()
            assert torch.equal(torch.from_numpy(full), whole), (mode, sigma_r)
