"""Multi-process (world size 2, gloo, CPU) test of the multi-GPU host logic: head sharding with
mask re-packing and the gather of output shards.  Each rank computes its shard with the fp64 oracle
(standing in for its GPU), shards are all-gathered, and rank 0's concatenation must equal the full
layer exactly.  On B200s the same code runs with NCCL (tools/multi_gpu_validate.py)."""
import os

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import oracle
import workloads as W
from paper_conf_iiswc_choilkha22_b200 import shard as SH

CASES = {
    "padded": dict(B=4, H=3, S=128, D=8, kv_len=[128, 5, 70, 1]),
    "block": dict(B=2, H=3, S=256, D=8, layout="rand"),
    "dense": dict(B=1, H=5, S=128, D=8),
}


def _oracle_mask(kv_len=None, layout=None):
    if layout is not None:
        return oracle.Mask(kind="block", layout=layout)
    return oracle.Mask(kv_len=kv_len)


def _worker(rank, world, port, case, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    c = dict(CASES[case])
    lay = W.random_layout(c["H"], c["S"] // 64, 64, 0.5, seed=5) if c.pop("layout", None) else None
    Bb, H, S, D = c["B"], c["H"], c["S"], c["D"]
    kv = c.get("kv_len")
    t = W.make_qkv(Bb, H, S, D, "f32", seed_base=9)
    sh = SH.make_shard(rank, world, Bb, H, S, kv_len=kv, layout=lay)
    qs, ks, vs = (SH.shard_view(torch.from_numpy(x), sh).numpy() for x in (t.q64, t.k64, t.v64))
    if sh.n:
        o = oracle.attention(qs, ks, vs, 0.3, _oracle_mask(sh.kv_len, sh.layout))
    else:
        o = np.zeros((0, 1, S, D))
    # variable-size shards: pad to the max shard, gather, trim (all_gather needs equal sizes)
    n_all = [torch.zeros(1, dtype=torch.int64) for _ in range(world)]
    dist.all_gather(n_all, torch.tensor([sh.n]))
    n_max = int(max(x.item() for x in n_all))
    buf = torch.zeros(n_max, S, D, dtype=torch.float64)
    buf[:sh.n] = torch.from_numpy(o.reshape(sh.n, S, D))
    parts = [torch.zeros_like(buf) for _ in range(world)]
    dist.all_gather(parts, buf)
    if rank == 0:
        full = torch.cat([p[:int(n.item())] for p, n in zip(parts, n_all)]).numpy()
        ref = oracle.attention(t.q64, t.k64, t.v64, 0.3, _oracle_mask(kv, lay)).reshape(Bb * H, S, D)
        q.put((full.shape == ref.shape and np.array_equal(full, ref), [int(n.item()) for n in n_all]))
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4, 8])
@pytest.mark.parametrize("case", list(CASES))
def test_shard_and_gather(case, world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + (abs(hash(case)) % 500) + 500 * (world // 4)
    procs = [ctx.Process(target=_worker, args=(r, world, port, case, q)) for r in range(world)]
    for p in procs:
        p.start()
    ok, sizes = q.get(timeout=240)
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    assert ok, sizes
    assert sum(sizes) == CASES[case]["B"] * CASES[case]["H"]


def test_head_costs_match_library_schedule():
    """shard.py's per-head cost model counts exactly the tiles the library's schedule lists
    (sr_schedule_stats on a one-head layer), for padding + causal and per-head block layouts."""
    import paper_conf_iiswc_choilkha22_b200 as sr
    S = 512
    kv = [512, 300, 65, 1]
    for causal in (False, True):
        costs = SH.head_costs(len(kv), 1, S, 64, kv_len=kv, causal=causal)
        for b, k in enumerate(kv):
            n, _ = sr.schedule_stats(sr.dense_mask([k]), 1, 1, S, causal=causal, tile_n=64)
            assert costs[b] - 1.5 * (S // 128) == n, (k, causal)
    lay = W.random_layout(3, S // 64, 64, 0.4, seed=2)
    costs = SH.head_costs(1, 3, S, 64, layout=lay)
    for h in range(3):
        one = W.csr_from_sets(64, [[set(lay.blocks(h, r)) for r in range(S // 64)]])
        n, _ = sr.schedule_stats(sr.block_mask(one), 1, 1, S, tile_n=64)
        assert costs[h] - 1.5 * (S // 128) == n


def test_bench_shards_cover_the_layer():
    """bench.py --gpus N splits each BASELINE config's heads into N contiguous shards that cover
    every head exactly once, with per-shard masks re-packed."""
    import bench
    for idx in (2, 3, 4, 5):
        cfg = W.config(idx)
        for world in (2, 4, 8):
            shards = [bench.make_shard(cfg, r, world) for r in range(world)]
            assert shards[0].g0 == 0 and shards[-1].g1 == cfg.BH
            assert all(a.g1 == b.g0 for a, b in zip(shards, shards[1:]))
            for sh in shards:
                if cfg.kv_len is not None:
                    assert list(sh.kv_len) == [cfg.kv_len[g // cfg.H] for g in range(sh.g0, sh.g1)]
                if cfg.kind == "blocksparse":
                    assert sh.layout.layout_heads == sh.n


def test_contiguous_ranges_balance():
    costs = [4, 4, 3, 3, 3, 1, 1, 1] * 12
    for world in (1, 2, 4, 8):
        rr = SH.contiguous_ranges(costs, world)
        assert rr[0][0] == 0 and rr[-1][1] == len(costs)
        assert all(a[1] == b[0] for a, b in zip(rr, rr[1:]))
        loads = [sum(costs[a:b]) for a, b in rr]
        assert max(loads) - min(loads) <= max(costs)
