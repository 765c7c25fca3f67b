"""World-size-2 run of the multi-GPU host logic on CPU (gloo): each rank takes its LPT shard,
factors it (the CPU oracle stands in for the GPU kernels here), and the ranks gather
(index, info) pairs and the max time exactly as bench.py does over NCCL."""
import os
import socket

import numpy as np
import torch.multiprocessing as mp

import vbgen

WORLD = 2


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, port, q):
    import torch.distributed as dist

    import oracle
    from paper_conf_ipps_abdelfattahhtd16_b200 import shard
    os.environ["MASTER_ADDR"] = "127.0.0.1"
    os.environ["MASTER_PORT"] = str(port)
    dist.init_process_group("gloo", rank=rank, world_size=WORLD)
    try:
        cfg = vbgen.Config("T", 120, "uniform", 48, 7, 20)  # 5 % non-SPD like C4
        n_all = vbgen.sizes(cfg)
        mine = shard.shard_indices(n_all, WORLD, rank)
        infos = []
        for g in mine:
            _, info = oracle.dpotrf(vbgen.config_matrix(cfg, int(g), int(n_all[g])))
            infos.append(info)
        info_all = shard.gather_info(len(n_all), mine, infos)
        tmax = shard.max_over_ranks(10.0 + rank)
        tot = shard.sum_over_ranks(float(len(mine)))
        q.put((rank, info_all.tolist(), tmax, tot, mine.tolist()))
    finally:
        dist.destroy_process_group()


def test_two_rank_shard_and_gather():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, port, q)) for r in range(WORLD)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(WORLD)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    res.sort()
    cfg = vbgen.Config("T", 120, "uniform", 48, 7, 20)
    n_all = vbgen.sizes(cfg)
    expect = [vbgen.nonspd_k(cfg.seed, g, int(n_all[g])) if vbgen.is_nonspd(cfg, g) else 0
              for g in range(len(n_all))]
    for rank, info_all, tmax, tot, mine in res:
        assert info_all == expect  # every rank holds the complete, correct info[]
        assert tmax == 11.0 and tot == float(len(n_all))
    assert sorted(res[0][4] + res[1][4]) == list(range(len(n_all)))
