"""N > 1 host logic on CPU (gloo, world size 2): rank 0 schedules HIOS-LP,
the other rank imports the broadcast schedule through the C-ABI and must end
with the identical Q and predicted latency; logical-GPU ownership and the
max-over-ranks timing reduction."""
import os
import sys

import pytest
import torch.distributed as dist
import torch.multiprocessing as mp

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _worker(rank, world, port, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    import bench
    from paper_conf_cluster_kundus23_b200 import hios as h
    from workloads import gen, graphs
    g = graphs.inception_v3(299)
    W = gen.make_weights(g)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
    S = None
    if rank == 0:
        import random
        rng = random.Random(3)
        for op in g.ops:
            h.hios_set_op_cost(G, op.id, 0 if op.kind == "input" else rng.randint(2000, 60000))
        for e in range(g.n_edges):
            h.hios_set_edge_cost(G, e, rng.randint(500, 20000))
        h.hios_set_group_model(G, 7, 10)
        S = h.hios_schedule_lp(G, 4, 3)
    S = bench.share_schedule(h, dist, G, g, S, 4, 3, rank)
    Q = h.stages_to_Q(S)
    L = h.hios_schedule_latency_ns(S)
    t = bench.max_over_ranks(dist, 1.5 + rank, world)
    q.put((rank, Q, L, t, bench.owners(4, world)))
    dist.barrier()
    dist.destroy_process_group()


def test_schedule_broadcast_and_import_two_ranks():
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29611
    ps = [ctx.Process(target=_worker, args=(r, 2, port, q)) for r in range(2)]
    for p in ps:
        p.start()
    res = sorted([q.get(timeout=300) for _ in ps])
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    (r0, Q0, L0, t0, own0), (r1, Q1, L1, t1, own1) = res
    assert Q0 == Q1                      # identical schedule on both ranks
    assert t0 == t1 == 2.5               # max over ranks
    assert own0 == own1 == [0, 1, 0, 1]  # logical GPU i -> rank i % world
    assert L0 > 0 and L1 > 0
