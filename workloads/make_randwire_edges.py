"""Regenerate workloads/randwire_ws_edges.json (run once; output is committed).

WS(N=32, K=4, P=0.75) random graphs of RandWire-WS (Xie et al.), seeds 0/1/2,
undirected edges oriented from the lower to the higher node id.
"""
import json
import os

import networkx as nx


def main():
    stages = []
    for seed in (0, 1, 2):
        g = nx.connected_watts_strogatz_graph(32, 4, 0.75, seed=seed)
        stages.append(sorted((min(a, b), max(a, b)) for a, b in g.edges()))
    out = os.path.join(os.path.dirname(__file__), "randwire_ws_edges.json")
    with open(out, "w") as f:
        json.dump({"generator": "networkx.connected_watts_strogatz_graph(32, 4, 0.75, seed=s)",
                   "networkx": nx.__version__, "stages": stages}, f)


if __name__ == "__main__":
    main()
