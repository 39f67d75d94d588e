"""The N > 1 path on CPU: world_size-2 gloo process group (127.0.0.1), as bench.py runs it under
torchrun -- every rank routes the same request pool with Alg. 2 (library planner on the host),
shares are disjoint and cover the pool, and the step time is the max over ranks."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import synth

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, out_dir):
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    g = synth.rng(42)
    L_img, L_txt = 4096, 512
    ratios = synth.sample_mask_ratios(g, 12)
    n_active = [synth.n_masked_for(float(m), L_img) + L_txt for m in ratios]
    cm = sched.CostModel(57, 3072, 12288, "kv", comp=(1 / 1.0e9, 0.1), load=(1 / 5e7, 0.01))
    mine, assign, held = sched.shard_requests(n_active, L_img + L_txt, world, rank, cm, 8)
    # every rank must hold the identical assignment (no data-path communication is used)
    gathered = [None] * world
    dist.all_gather_object(gathered, assign)
    # max-over-ranks timing reduction, as in bench.run_engine_timed
    t = torch.tensor([10.0 + rank])
    dist.all_reduce(t, op=dist.ReduceOp.MAX)
    np.save(os.path.join(out_dir, f"r{rank}.npy"),
            np.array([mine, gathered, held, float(t.item())], dtype=object), allow_pickle=True)
    dist.barrier()
    dist.destroy_process_group()


@pytest.mark.parametrize("world", [2])
def test_request_sharding_world2(tmp_path, world):
    port = _free_port()
    mp.spawn(_worker, args=(world, port, str(tmp_path)), nprocs=world, join=True)
    res = [np.load(tmp_path / f"r{r}.npy", allow_pickle=True) for r in range(world)]
    mines = [list(r[0]) for r in res]
    for r in res:
        gathered = r[1]
        assert all(a == gathered[0] for a in gathered)        # identical routing on every rank
        assert r[3] == 10.0 + world - 1                       # max over ranks
    flat = sorted(i for m in mines for i in m)
    assert flat == list(range(12)) and not list(res[0][2])   # disjoint cover, nothing held
    assert all(len(m) > 0 for m in mines)


def test_mask_aware_routing_balances_predicted_latency():
    """Alg. 2 (cost = planner latency of batch + request) vs request-count round robin on a
    skewed pool: the slowest worker's predicted step latency is no worse (L261, L398)."""
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    g = synth.rng(7)
    ratios = np.sort(synth.sample_mask_ratios(g, 16))[::-1]
    n_active = [synth.n_masked_for(float(m), 4096) + 512 for m in ratios]
    cm = sched.CostModel(57, 3072, 12288, "kv", comp=(1 / 1.0e9, 0.1), load=(1 / 5e7, 0.01))
    reqs = [sched.Request(i, n, 4608) for i, n in enumerate(n_active)]
    ma, _ = sched.assign_all(reqs, 4, cm.step_latency, 8)
    rr = [[reqs[i] for i in range(w, 16, 4)] for w in range(4)]
    worst = lambda ws: max(cm.step_latency(w) for w in ws)
    assert worst(ma) <= worst(rr) + 1e-9


def _bench_worker(rank, world, port, out_dir):
    """One rank of bench.py's multi-GPU routing path (bench.make_requests + bench.route_job) on
    a C4 job: a pool of 16 x world heterogeneous masks (5-60 %), max batch 16 per GPU."""
    import sys
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port), RANK=str(rank),
                      WORLD_SIZE=str(world))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from paper_conf_eurosys_jianglyfdlzllyl26_b200 import sched
    w = dict(bench.WORKLOADS["C4"], block="flux")
    pool = bench.make_requests(w, w["batch"] * world, bench.SEED)
    # per-block-kind compute models as the bench fits them (double-stream / single-stream)
    cm = sched.CostModel(57, 3072, 12288, "kv", comp=(7.3e-13, 0.10), load=(1 / 5.5e7, 0.003),
                         full_entry_rows=4096, kind="double",
                         layer_comp=[(7.4e-13, 0.10)] * 19 + [(7.2e-13, 0.09)] * 38)
    mine, assign, held = bench.route_job(pool, w, world, rank, cm)
    gathered = [None] * world
    dist.all_gather_object(gathered, assign)
    lat = cm.step_latency([sched.Request(i, pool[i]["n_active"], 4608) for i in mine])
    lats = [None] * world
    dist.all_gather_object(lats, lat)
    np.save(os.path.join(out_dir, f"b{rank}.npy"),
            np.array([mine, gathered, held, lats, [p["ratio"] for p in pool]], dtype=object),
            allow_pickle=True)
    dist.barrier()
    dist.destroy_process_group()


def test_bench_routing_path_world2(tmp_path):
    """bench.py's own N > 1 routing (the function its main() calls) on 2 gloo ranks: identical
    assignment on every rank, a disjoint cover of the heterogeneous pool, 16 requests per GPU,
    and predicted step latencies within 5 % of each other (Alg. 2 balances mask sizes, L261)."""
    world = 2
    mp.spawn(_bench_worker, args=(world, _free_port(), str(tmp_path)), nprocs=world, join=True)
    res = [np.load(tmp_path / f"b{r}.npy", allow_pickle=True) for r in range(world)]
    for r in res:
        assert all(a == r[1][0] for a in r[1])
    mines = [list(r[0]) for r in res]
    assert sorted(i for m in mines for i in m) == list(range(32)) and not list(res[0][2])
    assert all(len(m) == 16 for m in mines)
    assert len(set(res[0][4])) == 16                  # the pool really is heterogeneous
    lats = res[0][3]
    assert max(lats) <= 1.05 * min(lats), lats


def test_bench_refuses_mismatched_world(tmp_path):
    """`bench.py --gpus 2` inside a 1-rank launch must not report a 1-rank run as 2 GPUs."""
    import subprocess
    import sys
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2"],
                       env=env, capture_output=True, text=True, timeout=120)
    assert p.returncode == 2, p.stderr[-2000:]
