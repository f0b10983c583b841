"""GPU checks of the native multi-GPU driver gsh_join_sharded (include/gsh.h; SURVEY §8(b)
"gsh_join_sharded(..., ncclComm_t)", §8(e)) against the oracle on the whole input:

* G = 1, 2, 4, 8 logical ranks sharing the one GPU through the library's in-process local world,
  both exchanges (a2a: collectives, the normal all-to-all on a second stream beside the skewed-key
  join; p2p: the route kernel's stores into the peers' receive buffers), COUNT and MATERIALIZE;
* buffer reuse and growth across calls of the same per-rank drivers;
* a rank failing its argument checks aborts the world instead of hanging its peers;
* the same per-rank numbers as the Python driver (sharded.join_sharded);
* NCCL with world size 1: a new communicator (gsh_nccl_unique_id / gsh_comm_nccl_init) and the
  torch process group's own ncclComm_t (gsh_comm_nccl);
* two processes on the one GPU with torch.distributed gloo collectives called back from the
  library, receive buffers shared through CUDA IPC (the cross-process path of p2p).
"""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import datagen
import oracle

pytestmark = pytest.mark.gpu


def _shard(t, g, G):
    lo, hi = g * t.numel() // G, (g + 1) * t.numel() // G
    return t[lo:hi]


def _u32(t):
    return t.cpu().numpy().view(np.uint32)


_CASES = [
    (1, "zipf", 1 << 17, 1.0, {}),
    (2, "zipf", 1 << 18, 1.0, {}),
    (4, "zipf", 1 << 18, 1.25, dict(large_threshold=512)),
    (4, "pkfk", 1 << 18, 0.0, {}),
    (2, "graph", 1 << 18, 0.909, {}),
    (8, "uniform", 1 << 17, 0.0, {}),
    (8, "zipf", 1 << 17, 0.75, {}),
    (4, "pkfk_zipf", 1 << 18, 1.0, dict(heavy_threshold=64)),
    (8, "pkfk_zipf", 1 << 18, 0.8, dict(heavy_threshold=16, large_threshold=64)),
]


@pytest.mark.parametrize("exchange", ["a2a", "p2p"])
@pytest.mark.parametrize("world,kind,n,theta,kw", _CASES)
def test_native_local_world_vs_oracle(world, kind, n, theta, kw, exchange):
    from paper_conf_icde_caic24_b200 import make_config, sharded
    dev = torch.device("cuda", 0)
    full = datagen.make_workload(kind, n, theta, seed=23)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    cfg = make_config(**kw)
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    res = sharded.run_local_native(world, shards, config=cfg, exchange=exchange, repeat=2)
    P = sharded.shard_plan(n, n, world, cfg)
    oh, _, _ = oracle.heavy_rule(full[0].numpy().view(np.uint32), full[2].numpy().view(np.uint32),
                                 int(P.part_bits), int(P.large_threshold), int(P.heavy_threshold))
    for r in res:
        assert (r.count, r.checksum) == (on, oc), (r.stats, on, oc)
        assert r.stats["n_heavy"] == len(oh)
        assert r.stats["cand_overflow"] == 0
        assert r.stats["route_bits"] == world.bit_length() - 1
    assert sum(r.stats["normal_s"] + r.stats["heavy_s"] for r in res) == n
    assert len({r.stats["heavy_r"] for r in res}) == 1
    assert sum(r.stats["normal_r"] for r in res) + res[0].stats["heavy_r"] == n
    assert sum(r.stats["count_normal"] + r.stats["count_heavy"] for r in res) == on
    if kind in ("zipf", "pkfk_zipf") and theta >= 1.0:
        assert len(oh) > 0 and res[0].stats["heavy_r"] > 0


@pytest.mark.parametrize("exchange", ["a2a", "p2p"])
def test_native_materialize(exchange):
    from paper_conf_icde_caic24_b200 import sharded
    dev = torch.device("cuda", 0)
    world, n = 4, 1 << 16
    full = datagen.make_workload("zipf", n, 1.0, seed=4)
    on, oc, want = oracle.join_sorted_pairs(*(t.numpy().view(np.uint32) for t in full))
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    res = sharded.run_local_native(world, shards, mode="materialize", out_capacity=on, exchange=exchange)
    assert sum(r.written for r in res) == on and all(not r.overflow for r in res)
    got = np.concatenate([r.pairs.cpu().numpy().view(np.uint32) for r in res])
    got = got[np.lexsort((got[:, 1], got[:, 0]))]
    assert np.array_equal(got, want)
    for r in res:
        assert (r.count, r.checksum) == (on, oc)


@pytest.mark.parametrize("exchange", ["a2a", "p2p"])
def test_native_buffers_grow_across_calls(exchange):
    """Small, then 8x larger, then small again, then an empty rank: the per-rank drivers reuse and
    grow their receive buffers (p2p: re-shared with the peers) and stay exact."""
    from paper_conf_icde_caic24_b200 import sharded
    dev = torch.device("cuda", 0)
    world = 4
    calls, want = [], []
    for kind, n, theta, seed in (("zipf", 1 << 14, 1.0, 1), ("zipf", 1 << 17, 1.25, 2), ("graph", 1 << 15, 0.909, 3),
                                 ("pkfk", 1 << 14, 0.0, 4)):
        full = datagen.make_workload(kind, n, theta, seed=seed)
        want.append(oracle.join(*(t.numpy().view(np.uint32) for t in full))[:2])
        sh = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
        if seed == 4:   # rank 3 holds nothing
            sh[2] = tuple(torch.cat([a, b]) for a, b in zip(sh[2], sh[3]))
            sh[3] = tuple(t[:0] for t in sh[3])
        calls.append(sh)
    out = sharded.run_local_native(world, None, calls=calls, exchange=exchange)
    for res, (on, oc) in zip(out, want):
        for r in res:
            assert (r.count, r.checksum) == (on, oc)


def test_native_rank_failure_aborts_world():
    """Rank 1 passes a config the driver refuses: it returns GSH_ERR_INVALID and aborts the local
    world, so rank 0 (already inside a collective) returns an error instead of waiting forever."""
    from paper_conf_icde_caic24_b200 import GshError, make_config, sharded
    dev = torch.device("cuda", 0)
    full = datagen.make_workload("zipf", 1 << 14, 1.0, seed=3)
    shards = [tuple(_shard(t, g, 2).to(dev) for t in full) for g in range(2)]
    with pytest.raises(GshError, match="route_bits"):
        sharded.run_local_native(2, shards, configs=[make_config(), make_config(route_bits=1)])


def test_native_matches_python_driver():
    from paper_conf_icde_caic24_b200 import sharded
    dev = torch.device("cuda", 0)
    world = 4
    full = datagen.make_workload("zipf", 1 << 17, 1.0, seed=9)
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    py = sharded.run_local(world, shards, exchange="p2p")
    nat = sharded.run_local_native(world, shards, exchange="p2p")
    for a, b in zip(py, nat):
        assert (a.count, a.checksum) == (b.count, b.checksum)
        for k in ("normal_r", "normal_s", "heavy_r", "heavy_s", "count_normal", "count_heavy"):
            assert a.stats[k] == b.stats[k], k
        assert a.stats["n_heavy_global"] == b.stats["n_heavy"]
        assert a.stats["exchange_send_bytes"] == b.stats["exchange_bytes"]


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _nccl_worker(port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dev = torch.device("cuda", 0)
    dist.init_process_group("nccl", rank=0, world_size=1, device_id=dev)
    try:
        from paper_conf_icde_caic24_b200 import sharded
        dist.barrier()
        rk, rp, sk, sp = (t.cuda() for t in datagen.make_workload("zipf", 1 << 16, 1.0, seed=23))
        got = []
        for use_group in (False, True):
            comm = sharded.nccl_comm(device=dev, use_group_comm=use_group)
            drv = sharded.ShardedJoin(comm, dev)
            for ex in ("a2a", "p2p"):
                r = drv.join(rk, rp, sk, sp, exchange=ex)
                got.append((r.count, r.checksum, r.stats["n_heavy"]))
            drv.close()
            comm.close()
        q.put(got)
    finally:
        dist.destroy_process_group()


def test_native_nccl_single_rank():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    p = ctx.Process(target=_nccl_worker, args=(_free_port(), q))
    p.start()
    got = q.get(timeout=300)
    p.join(timeout=60)
    assert p.exitcode == 0
    full = datagen.make_workload("zipf", 1 << 16, 1.0, seed=23)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    assert len(got) == 4
    for c, k, nh in got:
        assert (c, k) == (on, oc) and nh > 0


def _gloo_worker(rank, world, port, q):
    import torch.distributed as dist
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    torch.cuda.set_device(0)
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        from paper_conf_icde_caic24_b200 import sharded
        dev = torch.device("cuda", 0)
        full = datagen.make_workload("zipf", 1 << 17, 1.0, seed=43)
        rk, rp, sk, sp = (_shard(t, rank, world).cuda() for t in full)
        comm = sharded.TorchGroupComm()
        drv = sharded.ShardedJoin(comm, dev)
        out = []
        for ex in ("p2p", "a2a", "p2p"):
            r = drv.join(rk, rp, sk, sp, exchange=ex)
            out.append((r.count, r.checksum))
        drv.close()
        q.put((rank, out))
    finally:
        dist.destroy_process_group()


def test_native_two_processes_gloo_ipc():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_gloo_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in procs:
        p.start()
    out = [q.get(timeout=300) for _ in range(2)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    full = datagen.make_workload("zipf", 1 << 17, 1.0, seed=43)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    for _, res in out:
        assert res == [(on, oc)] * 3


@pytest.mark.parametrize("exchange", ["a2a", "p2p"])
@pytest.mark.parametrize("world,theta", [(2, 1.0), (4, 1.5)])
def test_native_with_hybrid_local_joins(world, theta, exchange):
    """gsh_config.hybrid reaches the ranks' local joins (the routed normal shard keeps route_bits =
    log2 G): the global result is unchanged."""
    from paper_conf_icde_caic24_b200 import make_config, sharded
    dev = torch.device("cuda", 0)
    full = datagen.make_workload("zipf", 1 << 18, theta, seed=31)
    on, oc, _ = oracle.join(*(t.numpy().view(np.uint32) for t in full))
    shards = [tuple(_shard(t, g, world).to(dev) for t in full) for g in range(world)]
    res = sharded.run_local_native(world, shards, config=make_config(hybrid=True, hybrid_stride=10, hybrid_share=1),
                                   exchange=exchange)
    for r in res:
        assert (r.count, r.checksum) == (on, oc), (r.stats, on, oc)
