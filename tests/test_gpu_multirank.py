"""The sharded multi-rank pipeline (pipeline.DeviceSkycube under torch.distributed) with the real kernels:
world sizes 2 and 3 share the one GPU of the box (gloo for the collectives, staged through host memory),
and every output byte must equal the single-process C-ABI build ("output bytes must not
depend on k").  Needs a B200."""
from __future__ import annotations

import os
import socket

import numpy as np
import pytest

import datagen

pytestmark = pytest.mark.gpu


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, x, q):
    import torch
    import torch.distributed as dist
    from paper_conf_sigmod_boghcsa17_b200.pipeline import DeviceSkycube
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        eng = DeviceSkycube(0)
        out = eng.build(torch.from_numpy(x).cuda(), lists=True, membership=True, hashcube_w=32)
        torch.cuda.synchronize()
        res = {"membership": out["membership"].cpu().numpy().view(np.uint32).copy(),
               "ext_ids": out["ext_ids"].cpu().numpy().copy(),
               "offsets": out["offsets"].cpu().numpy().copy(), "ids": out["ids"].cpu().numpy().copy()}
        for k, v in out["hashcube"].items():
            res["hc_" + k] = v.cpu().numpy().copy()
        q.put((rank, res))
        dist.barrier()
        eng.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,name", [(2, "C3I"), (3, "A-small"), (2, "ct-small")])
def test_multirank_bytes_equal_single_rank(world, name):
    import torch
    import torch.multiprocessing as mp
    import paper_conf_sigmod_boghcsa17_b200 as sky
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    if name == "A-small":
        x = datagen.generate("A", 60000, 10, 91)
    elif name == "ct-small":
        x = datagen.generate("ct", 80000, 10, 92)
    else:
        x = datagen.config(name).data()
    want = sky.skycube_build(x)
    want_hc = sky.skycube_build_hashcube(x, 32)
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, x, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = dict(q.get(timeout=600) for _ in range(world))
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    for rank in range(world):
        r = res[rank]
        assert np.array_equal(r["membership"], want["rows"]), rank
        assert np.array_equal(r["ext_ids"], want["ext_ids"]), rank
        assert np.array_equal(r["offsets"], want["offsets"]) and np.array_equal(r["ids"], want["ids"]), rank
        for k in ("word_offsets", "keys", "key_offsets", "ids"):
            got = r["hc_" + k].view(np.uint32) if k == "keys" else r["hc_" + k]
            assert np.array_equal(got, want_hc[k]), (rank, k)


@pytest.mark.parametrize("k,name", [(2, "C3I"), (3, "A-small"), (4, "ct-small"), (2, "C2")])
def test_capi_num_gpus_bytes_equal_single_gpu(tuning, k, name):
    """The C-ABI's single-process multi-GPU path (skycube_opts.num_gpus = k): k logical ranks, here sharing
    the one GPU (skycube_set_tuning("share_devices", 1)), with the flag OR-combine, the peer-copy gathers and the sharded
    K1/K3 ranges; every output byte must equal the one-GPU build."""
    import torch
    import paper_conf_sigmod_boghcsa17_b200 as sky
    if not torch.cuda.is_available():
        pytest.skip("no GPU")
    if name == "A-small":
        x = datagen.generate("A", 60000, 10, 91)
    elif name == "ct-small":
        x = datagen.generate("ct", 80000, 10, 92)
    else:
        x = datagen.config(name).data()
    want = sky.skycube_build(x)
    tuning("share_devices", 1)
    with sky.skycube_build_raw(x, num_gpus=k, stats=True) as r:
        assert np.array_equal(r.membership(), want["rows"])
        assert np.array_equal(r.ext_ids(), want["ext_ids"])
        assert np.array_equal(r.offsets(), want["offsets"]) and np.array_equal(r.ids(), want["ids"])
        assert r.stats["kernel_launches"] > 0
    with sky.skycube_build_raw(x, num_gpus=k, max_level=3) as r:
        assert np.array_equal(r.membership(), sky.skycube_build(x, max_level=3)["rows"])
