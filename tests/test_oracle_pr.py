"""Oracle Page-Rank-style pins (DESIGN.md R-pr-*).

* the iteration equals the textbook dense power iteration
  r' = (1-d)/n + d * A^T D^-1 r (numpy, within 1e-14) on the same graph;
* with no dangling nodes (every out-degree >= 1) the total rank stays 1:
  fsum == 1 within rounding, for any graph and iteration count;
* the graph has the stated out-degree distribution and (source, edge)-ordered
  in-lists.
"""
import numpy as np
import pytest


def dense_pagerank(deg, ptr, src, iters, d=0.85):
    n = len(deg)
    M = np.zeros((n, n))
    for v in range(n):
        for u in src[ptr[v]:ptr[v + 1]]:
            M[v, u] += 1.0 / deg[u]
    r = np.full(n, 1.0 / n)
    for _ in range(iters):
        r = (1 - d) / n + d * (M @ r)
    return r


@pytest.mark.parametrize("n,avg,iters,seed", [(7, 2, 3, 1), (50, 4, 10, 2), (200, 8, 20, 3), (1, 1, 5, 4)])
def test_matches_dense_power_iteration(oracle, n, avg, iters, seed):
    deg, ptr, src = oracle.pr_graph(n, avg, seed)
    r = oracle.run_text(f"-n {n} -e {avg} -i {iters} -R {seed}\n", app=oracle.APP_PAGERANK)
    rec = r.records[0]
    assert rec["exit_code"] == 0 and rec["work"] == len(src) * iters
    ref = dense_pagerank(deg, ptr, src, iters)
    assert abs(rec["fsum"] - ref.sum()) < 1e-13
    top = int(r.stdout[0].split(b"top=")[1])
    assert abs(ref[top] - ref.max()) < 1e-14


@pytest.mark.parametrize("n,avg,iters", [(1000, 8, 10), (3000, 3, 25), (500, 16, 0)])
def test_rank_mass_is_conserved(oracle, n, avg, iters):
    r = oracle.run_text(f"-n {n} -e {avg} -i {iters}\n", app=oracle.APP_PAGERANK)
    assert abs(r.records[0]["fsum"] - 1.0) < 1e-12
    assert r.records[0]["fabs"] == r.records[0]["fsum"]


def test_graph_statistics(oracle):
    n, avg = 20000, 8
    deg, ptr, src = oracle.pr_graph(n, avg, 7)
    assert deg.min() >= 1 and deg.max() <= 2 * avg - 1
    assert abs(deg.mean() - avg) < 0.1
    assert ptr[-1] == len(src) == deg.sum()
    for v in range(0, n, 997):  # in-lists in (source, edge) order
        assert np.all(np.diff(src[ptr[v]:ptr[v + 1]]) >= 0)
    indeg = np.diff(ptr)
    assert abs(indeg.mean() - deg.mean()) < 1e-9


@pytest.mark.parametrize("line", ["-n 0", "-e", "-i x", "-q 1", "-n 16777216 -e 1024"])
def test_usage_errors(oracle, line):
    r = oracle.run_text(line + "\n", app=oracle.APP_PAGERANK)
    assert r.records[0]["exit_code"] == 1 and b"usage: pagerank" in r.stdout[0]
