"""Page-Rank-style instances on the GPU vs the oracle,
plus the mass-conservation invariant at full size (fsum == 1 within rounding:
every node has out-degree >= 1, so no rank leaks)."""
import numpy as np
import pytest

pytestmark = pytest.mark.gpu

from parity import assert_parity  # noqa: E402

CASES = [
    "pagerank -n 1 -e 1 -i 3",
    "pagerank -n 7 -e 2 -i 5 -R 3",
    "pagerank -n 1000 -e 8 -i 10 -R 4",
    "pagerank -n 4097 -e 3 -i 7 -R 5",
    "pagerank -n 20000 -e 16 -i 4 -R 6",
    "pagerank -n 300 -e 5 -i 0",
    "pagerank -n 0",
    "pagerank -x 1",
]


@pytest.mark.parametrize("threads", [64, 256, 1024])
def test_pagerank_parity(oracle, threads):
    from paper_conf_icppw_tiancd23_b200.ensemble import run_text
    text = "".join(l + "\n" for l in CASES)
    g = run_text(text, app="auto", threads=threads)
    o = oracle.run_text(text)
    assert_parity(g, o)


def test_pagerank_ensemble_full_size():
    """256 instances of the HeCBench-like size the paper could fit only 2-4 of."""
    from paper_conf_icppw_tiancd23_b200.ensemble import run_text
    text = "".join(f"pagerank -n 100000 -e 8 -i 10 -R {i}\n" for i in range(256))
    r = run_text(text, app="auto", threads=1024)
    assert np.all(r.records["exit_code"] == 0)
    assert np.all(np.abs(r.records["fsum"] - 1.0) < 1e-12)
