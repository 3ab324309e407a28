"""Multi-process (gloo, CPU) tests of the row-band halo exchange and the
frame partition (paper_conf_ipps_membarthhtke12_b200/dist.py).

The band decomposition is checked against the oracle: the oracle run on each
halo-extended band reproduces the whole-image oracle output bit for bit
(SURVEY §4(3)(i)), for every boundary mode (REPEAT through the ring halo)."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import synthetic
from paper_conf_ipps_membarthhtke12_b200 import dist as ldist

MODES = ["undefined", "clamp", "repeat", "mirror", "constant"]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    return port


def _worker(rank, world, port, H, W, halo, q):
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        img = synthetic.angio(H, W, seed=99)
        results = {}
        for mode in MODES:
            band = ldist.Bands(H, W, world, rank, halo, device="cpu", mode=mode)
            band.fill(lambda y0, y1: synthetic.angio(H, W, seed=99, row_range=(y0, y1)))
            band.top.fill_(float("nan"))
            band.bottom.fill_(float("nan"))
            band.exchange()
            ht, hb, y0, gh = band.band_args()
            ext = band.buf[halo - ht:halo + band.rows + hb]
            # halo rows are exactly the neighbours' rows (ring-wrapped for REPEAT)
            rows = [(y % H) for y in range(y0 - ht, y0 + band.rows + hb)]
            halo_ok = torch.equal(ext, img[rows])
            # oracle on the extended band == whole-image oracle on the owned rows
            out, _ = oracle.bilateral_f32(ext.numpy(), 1.0, 0.1, mode, cval=0.5, size=2 * halo + 1,
                                          rows=(ht, ht + band.rows))
            g, _ = oracle.convolve_f32(ext.numpy(), np.ones((2 * halo + 1, 3)) / 3.0, mode, 0.5,
                                       rows=(ht, ht + band.rows))
            results[mode] = (y0, halo_ok, out, g)
        q.put((rank, results))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_band_exchange_matches_whole_image_oracle(world):
    H, W, halo = 23, 17, 3
    port = _free_port()
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    procs = [ctx.Process(target=_worker, args=(r, world, port, H, W, halo, q))
             for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    img = synthetic.angio(H, W, seed=99).numpy()
    for mode in MODES:
        whole, _ = oracle.bilateral_f32(img, 1.0, 0.1, mode, cval=0.5, size=2 * halo + 1)
        wg, _ = oracle.convolve_f32(img, np.ones((2 * halo + 1, 3)) / 3.0, mode, 0.5)
        got = np.concatenate([res[r][mode][2] for r in range(world)])
        gotg = np.concatenate([res[r][mode][3] for r in range(world)])
        assert all(res[r][mode][1] for r in range(world)), mode
        assert np.array_equal(got, whole), mode
        assert np.array_equal(gotg, wg), mode


def test_single_rank_repeat_ring_and_ranges():
    H, W = 20, 8
    band = ldist.Bands(H, W, 1, 0, 4, mode="repeat")
    img = synthetic.angio(H, W, seed=5)
    band.fill(lambda a, b: img[a:b])
    band.exchange()
    assert torch.equal(band.top, img[-4:]) and torch.equal(band.bottom, img[:4])
    assert band.band_args() == (4, 4, 0, H)
    clamp = ldist.Bands(H, W, 1, 0, 4, mode="clamp")
    assert clamp.band_args() == (0, 0, 0, H)
    assert [ldist.frame_range(1024, 8, r) for r in (0, 7)] == [(0, 128), (896, 1024)]
    assert [ldist.band_range(32768, 3, r) for r in range(3)] == [(0, 10922), (10922, 21845),
                                                                 (21845, 32768)]
    with pytest.raises(ValueError):
        ldist.Bands(10, 4, 4, 1, 6)


def test_synthetic_row_range_is_consistent():
    full = synthetic.angio(600, 64, seed=7)
    assert torch.equal(synthetic.angio(600, 64, seed=7, row_range=(250, 517)), full[250:517])
