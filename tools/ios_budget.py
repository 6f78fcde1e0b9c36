import sys, time
sys.path.insert(0, ".")
from paper_conf_cluster_kundus23_b200 import hios as h
from workloads import gen, graphs
g = graphs.build("nasnet_a_large", 2048)
G = h.hios_graph_create(g.ops, g.edges, g.in_c, g.in_h, g.in_w, "bf16", gen.make_weights(g))
t0 = time.time(); h.hios_profile(G, [0], 5); print("profile", time.time() - t0, flush=True)
for b in (14, 16, 18, 20):
    t0 = time.time()
    try:
        S = h.hios_schedule_ios(G, 5, 1 << b)
        print(b, "ok", time.time() - t0, h.hios_schedule_latency_ns(S) / 1e6, flush=True)
    except h.HiosError as e:
        print(b, "fail", time.time() - t0, e, flush=True)
S = h.hios_schedule_lp(G, 1, 5); print("lp", h.hios_schedule_latency_ns(S) / 1e6)
