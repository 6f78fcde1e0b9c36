"""Multi-process (one process per GPU) correctness check, run under torchrun:
rank 0 schedules HIOS-LP over `world` logical GPUs, every rank imports it,
binds its logical GPU, exchanges CUDA IPC handles, and runs; the rank owning
the sink compares the logits with a single-process M=1 run (bit-identical:
placement never changes arithmetic).  Works with all ranks on one physical
GPU (IPC between processes on the same device)."""
import os
import sys

import numpy as np
import torch
import torch.distributed as dist

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import bench  # noqa: E402
from paper_conf_cluster_kundus23_b200 import hios as h  # noqa: E402
from workloads import gen, graphs  # noqa: E402


def main():
    model = sys.argv[1] if len(sys.argv) > 1 else "tiny"
    size = int(sys.argv[2]) if len(sys.argv) > 2 and sys.argv[2] != "-" else None
    transport = sys.argv[3] if len(sys.argv) > 3 else "peer"
    stage_mode = sys.argv[4] if len(sys.argv) > 4 else "streams"
    dist.init_process_group("gloo")
    rank, world = dist.get_rank(), dist.get_world_size()
    dev = int(os.environ.get("LOCAL_RANK", "0")) % torch.cuda.device_count()
    torch.cuda.set_device(dev)
    g = graphs.build(model, size)
    W = gen.make_weights(g)
    x = gen.make_input(g)
    G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
    S = None
    if rank == 0:
        # synthetic costs that force a multi-GPU mapping (cheap edges)
        for op in g.ops:
            h.hios_set_op_cost(G, op.id, 0 if op.kind == "input" else 10000)
        for e in range(g.n_edges):
            h.hios_set_edge_cost(G, e, 100)
        h.hios_set_group_model(G, 9, 10)
        S = h.hios_schedule_lp(G, world, 2)
    S = bench.share_schedule(h, dist, G, g, S, world, 2, rank)
    h.hios_schedule_transport(S, transport)
    h.hios_schedule_stage_mode(S, stage_mode)
    own = bench.bind_and_exchange(h, dist, S, world, world, rank, dev, transport=transport)
    op_gpu, _, _ = h.hios_schedule_stages(S)
    used = sorted(set(op_gpu.tolist()))
    ys = []
    import time
    for i in range(3):
        dist.barrier()
        t0 = time.time()
        ys.append(h.hios_run(S, x))
        print(f"rank {rank}: run {i} {time.time() - t0:.3f} s", flush=True)
    sink_rank = own[int(op_gpu[g.n_ops - 1])]
    ok = True
    if rank == sink_rank:
        G1 = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", W)
        for op in g.ops:
            h.hios_set_op_cost(G1, op.id, 1000)
        for e in range(g.n_edges):
            h.hios_set_edge_cost(G1, e, 1000)
        S1 = h.hios_schedule_lp(G1, 1, 1)
        y1 = h.hios_run(S1, x)
        ok = all(np.array_equal(y, y1) for y in ys)
        print(f"rank {rank}: world {world}, transport {transport}, stage mode {stage_mode}, GPUs used {used}, "
              f"sink on rank {sink_rank}, "
              f"bit-identical to 1-process run: {ok}", flush=True)
    flag = torch.tensor([1 if ok else 0])
    dist.all_reduce(flag, op=dist.ReduceOp.MIN)
    dist.barrier()
    dist.destroy_process_group()
    sys.exit(0 if int(flag.item()) == 1 else 1)


if __name__ == "__main__":
    main()
