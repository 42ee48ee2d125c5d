#!/usr/bin/env python3
"""Degree concentration of a BASELINE config's graph: the share of CSR entries (= the stationary visit
share of a random walk on an undirected graph) held by the top-k vertices, and by the vertices whose
row_ptr entries share an L2-sized footprint in natural ID order vs degree order. Diagnostics only."""
import argparse
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import lt_inputs  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", type=int, default=5)
    a = ap.parse_args()
    import torch
    c = lt_inputs.CONFIGS[a.config]
    g = lt_inputs.rmat_gpu(c["scale"], c["tuples"], seed=1, permute=c["permute"])
    deg = (g.row_ptr[1:] - g.row_ptr[:-1]).to(torch.float64)
    tot = float(deg.sum())
    sd, _ = torch.sort(deg, descending=True)
    cs = torch.cumsum(sd, 0) / tot
    for k in [10 ** 4, 10 ** 5, 10 ** 6, 4 * 10 ** 6, 8 * 10 ** 6, 16 * 10 ** 6, 32 * 10 ** 6]:
        if k <= g.n:
            print(f"top {k:>10d} vertices by degree: {100 * float(cs[k - 1]):6.2f} % of visits")
    # natural order: visit share of the hottest 32-B row_ptr sectors (4 vertices each)
    sec = deg[: (g.n // 4) * 4].view(-1, 4).sum(1)
    ss, _ = torch.sort(sec, descending=True)
    css = torch.cumsum(ss, 0) / tot
    for mb in [32, 64, 126]:
        k = mb * 2 ** 20 // 32
        print(f"hottest {mb:>4d} MB of row_ptr sectors, natural order: {100 * float(css[min(k, len(css)) - 1]):6.2f} % of visits")
    print(f"n={g.n} m={g.m} max_deg={g.max_deg}")


if __name__ == "__main__":
    main()
