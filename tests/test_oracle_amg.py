"""Oracle AMGmk-style pins.

* the CSR equals an independently built 7-point Laplacian (scipy kron sums),
  diagonal first then ascending columns (AMG-2 order), nnz closed form;
* A*1 == f exactly; u0 = 1 is a fixed point (upstream's error = 0 test);
* Jacobi sweeps match the dense textbook formula and contract the error.
"""
import numpy as np
import pytest
import scipy.sparse as sp


def lap(nx, ny, nz):
    def d1(n):
        return sp.diags([-np.ones(n - 1), -np.ones(n - 1)], [-1, 1], shape=(n, n))
    Ix, Iy, Iz = sp.identity(nx), sp.identity(ny), sp.identity(nz)
    off = sp.kron(Iz, sp.kron(Iy, d1(nx))) + sp.kron(Iz, sp.kron(d1(ny), Ix)) + sp.kron(d1(nz), sp.kron(Iy, Ix))
    return (6 * sp.identity(nx * ny * nz) + off).tocsr()


@pytest.mark.parametrize("dims", [(1, 1, 1), (2, 1, 1), (3, 4, 5), (5, 5, 5), (8, 3, 2)])
def test_csr_is_7pt_laplacian(oracle, dims):
    nx, ny, nz = dims
    rp, col, val = oracle.amg_csr(nx, ny, nz)
    n = nx * ny * nz
    ref = lap(nx, ny, nz)
    ref.sort_indices()
    assert len(col) == 7 * n - 2 * (nx * ny + ny * nz + nx * nz)
    for r in range(n):
        c = col[rp[r]:rp[r + 1]]
        v = val[rp[r]:rp[r + 1]]
        assert c[0] == r and v[0] == 6.0
        assert np.all(np.diff(c[1:]) > 0)
        rc = ref.indices[ref.indptr[r]:ref.indptr[r + 1]]
        rv = ref.data[ref.indptr[r]:ref.indptr[r + 1]]
        assert sorted(c) == list(rc)
        assert dict(zip(c, v)) == dict(zip(rc, rv))


def test_rhs_and_fixed_point(oracle):
    nx, ny, nz = 6, 5, 4
    n = nx * ny * nz
    y = oracle.amg_apply(nx, ny, nz, np.ones(n))
    ref = lap(nx, ny, nz) @ np.ones(n)
    assert np.array_equal(y, ref)  # integers: exact
    u = oracle.amg_sweeps(nx, ny, nz, 7, np.ones(n))
    assert np.array_equal(u, np.ones(n))


def test_relax_run_u0_ones(oracle):
    r = oracle.run_text("-x 7 -y 6 -z 5 -i 4 -r 0\n", app=oracle.APP_AMGMK)
    rec = r.records[0]
    n = 210
    assert rec["bitsum"] == (n * 0x3FF0000000000000) % (1 << 64)
    assert rec["fsum"] == n and rec["work"] == n * 4
    assert b"maxerr=0\n" in r.stdout[0]


def test_sweep_matches_dense_formula(oracle):
    nx, ny, nz = 5, 4, 3
    n = nx * ny * nz
    A = lap(nx, ny, nz).toarray()
    f = A @ np.ones(n)
    rng = np.random.default_rng(2)
    u = rng.random(n)
    D = np.diag(A)
    exp = (f - (A - np.diag(D)) @ u) / D
    got = oracle.amg_sweeps(nx, ny, nz, 1, u)
    assert np.allclose(got, exp, rtol=1e-14, atol=1e-15)


def test_jacobi_contracts(oracle):
    nx, ny, nz = 6, 6, 6
    n = nx * ny * nz
    rng = np.random.default_rng(5)
    u = rng.random(n)
    prev = np.abs(u - 1).max()
    for _ in range(10):
        u = oracle.amg_sweeps(nx, ny, nz, 1, u)
        e = np.abs(u - 1).max()
        assert e <= prev + 1e-15
        prev = e


def test_matvec_kind(oracle):
    r = oracle.run_text("-x 4 -y 4 -z 4 -i 3 -k matvec -r 0\n", app=oracle.APP_AMGMK)
    n = 64
    f = lap(4, 4, 4) @ np.ones(n)
    assert r.records[0]["fsum"] == f.sum()
    assert b"maxerr=0\n" in r.stdout[0]


@pytest.mark.parametrize("line", ["-x 0", "-i", "-k jacobi", "-x 1024 -y 1024 -z 1024", "-z a"])
def test_usage_errors(oracle, line):
    r = oracle.run_text(line + "\n", app=oracle.APP_AMGMK)
    assert r.records[0]["exit_code"] == 1 and b"usage: amgmk" in r.stdout[0]
