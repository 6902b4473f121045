"""Multi-process host logic (gloo, world size 2, CPU): every rank restores its own
instance (distinct seeds, no data exchange) and the job time is the max over
ranks -- the same helpers and the same gloo group bench.py uses (no NCCL);
bench.py --gpus 2 starts its own rank processes when no launcher did."""
import json
import os
import socket
import subprocess
import sys

import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, ws, port, out):
    import torch
    import torch.distributed as dist
    sys.path.insert(0, ROOT)
    import bench
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=ws)
    seed = bench.rank_seed("toy", rank)
    from workloads import make_graph_set
    gs = make_graph_set("toy", seed=seed)
    local_ms = 10.0 + rank  # rank 1 is the slow one
    job_ms = bench.max_over_ranks(local_ms, dist, torch.device("cpu"))
    out[rank] = (seed, int(gs.words.sum() % 1000003), job_ms)
    dist.barrier()
    dist.destroy_process_group()


def test_two_ranks_independent_instances_and_max_time():
    ws, port = 2, _free_port()
    mgr = mp.Manager()
    out = mgr.dict()
    mp.spawn(_worker, args=(ws, port, out), nprocs=ws, join=True)
    (s0, h0, t0), (s1, h1, t1) = out[0], out[1]
    assert s0 != s1 and h0 != h1          # each rank has its own instance
    assert t0 == t1 == 11.0               # job time = slowest rank, agreed on every rank


def test_reference_arm_runs_on_cpu():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "toy",
                        "--steps", "2", "--warmup", "1"], capture_output=True, text=True, cwd=ROOT, timeout=300)
    assert r.returncode == 0, r.stderr
    d = json.loads(r.stdout.strip().splitlines()[-1])
    assert d["impl"] == "reference" and d["unit"] == "nodes/s" and d["value"] > 0
    assert d["cpu_baseline"]["kind"] == "oracle" and d["e2e"]["h2d_bytes_per_step"] == 0


def test_bench_launches_its_own_ranks_over_gloo():
    """`bench.py --gpus 2` outside torchrun: two rank processes with the launcher's
    environment, a gloo group, the max over ranks and the gather (plumbing only)."""
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--selftest-plumbing"],
                       capture_output=True, text=True, cwd=ROOT, timeout=300, env=env)
    assert r.returncode == 0, r.stderr
    d = json.loads(r.stdout.strip().splitlines()[-1])
    assert d["world_size"] == 2 and d["max_ms"] == 11.0
    assert [x["rank"] for x in d["ranks"]] == [0, 1] and [x["local"] for x in d["ranks"]] == [0, 1]
    assert d["ranks"][0]["pid"] != d["ranks"][1]["pid"]
    assert [x["seed_c5"] for x in d["ranks"]] == [100, 101]  # C5: seed 100 + gpu
    assert d["ranks"][0]["seed_all10"] != d["ranks"][1]["seed_all10"]


def test_launcher_world_size_must_match_gpus():
    env = dict(os.environ, WORLD_SIZE="2", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "4", "--selftest-plumbing"],
                       capture_output=True, text=True, cwd=ROOT, timeout=300, env=env)
    assert r.returncode != 0 and "WORLD_SIZE=2" in r.stderr


def test_reference_arm_config_equals_ours():
    """The reference arm prints the config object bench.py's own arm builds for the
    same workload (same keys and values; the slot count is the oracle's, which the
    GPU arm's parity check equals)."""
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--workload", "toy",
                        "--steps", "1", "--warmup", "1", "--gpus", "2"], capture_output=True, text=True, cwd=ROOT,
                       timeout=300, env={k: v for k, v in os.environ.items() if k != "WORLD_SIZE"})
    assert r.returncode == 0, r.stderr
    d = json.loads(r.stdout.strip().splitlines()[-1])
    sys.path.insert(0, ROOT)
    import bench
    import oracle
    from workloads import make_graph_set
    seed = bench.rank_seed("toy", 0)
    gs = make_graph_set("toy", seed=seed)
    n_slots = oracle.materialize(gs.words, gs.node_word_off, gs.node_t, gs.allocs)["n_slots"]
    ours = bench.config_dict("toy", bench.WORKLOADS["toy"][1], gs, n_slots, seed, 2)
    assert d["config"] == ours and d["n_gpus"] == 2
