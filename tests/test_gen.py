"""Generator tests (-m "not gpu"): CSR contract, closed-form sizes, determinism, and loose
pins against the paper's Table I statistics."""
from __future__ import annotations

import hashlib
import os
import subprocess
import sys

import numpy as np
import pytest

from paper_conf_ipps_licqfsty16_b200 import gen

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_splitmix64_reference_vector():
    # first output of the standard splitmix64 stream seeded with 0
    assert gen.splitmix64(0) == 0xE220A8397B1DCDAF


@pytest.mark.parametrize("N", [1, 2, 3, 7, 10])
def test_stencil_sizes_closed_form(N):
    assert gen.stencil3d(N, N, N, 27).nnz == (3 * N - 2) ** 3 - N ** 3
    assert gen.stencil3d(N, N, N, 7).nnz == 6 * N * N * (N - 1)
    assert gen.stencil2d(N, N, 9).nnz == (3 * N - 2) ** 2 - N ** 2
    assert gen.stencil2d(N, N, 5).nnz == 4 * N * (N - 1)
    for g in (gen.stencil3d(N, N, N, 27), gen.stencil2d(N, N, 5)):
        assert g.validate() == 0


def test_cfg2_exact_nnz():
    g = gen.config(2)
    assert g.n == 104 ** 3 and g.nnz == 28_666_136
    assert g.degrees.max() == 26 and g.degrees.min() == 7


def test_stencil_rows_natural_order():
    g = gen.stencil3d(3, 3, 3, 27)
    centre = 1 + 3 * (1 + 3 * 1)
    row = g.col_idx[g.row_ptr[centre]:g.row_ptr[centre + 1]]
    assert row.tolist() == [v for v in range(27) if v != centre]


def test_from_edges_cleans_input():
    g = gen.from_edges(5, [(0, 1), (1, 0), (2, 2), (3, 4), (4, 3), (3, 4), (0, 4)])
    assert g.validate() == 0
    assert g.row_ptr.tolist() == [0, 2, 3, 3, 4, 6]
    assert g.col_idx.tolist() == [1, 4, 0, 4, 0, 3]


def test_validate_flags():
    rp = np.array([0, 2, 3, 4], np.int64)
    assert gen.validate(rp, np.array([2, 1, 0, 0], np.int32)) & 4    # unsorted row 0
    assert gen.validate(rp, np.array([1, 1, 0, 0], np.int32)) & 8    # duplicate
    assert gen.validate(rp, np.array([0, 1, 0, 0], np.int32)) & 16   # self-loop
    assert gen.validate(rp, np.array([1, 2, 0, 7], np.int32)) & 2    # out of range
    assert gen.validate(np.array([0, 1, 1], np.int64), np.array([1], np.int32)) & 32  # asym
    assert gen.validate(np.array([0, 2, 1], np.int64), np.array([1, 0], np.int32)) & 1


@pytest.mark.parametrize("maker", [
    lambda: gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=3),
    lambda: gen.rmat(12, 8, 0.57, 0.19, 0.19, seed=3, permute=True),
    lambda: gen.er(5000, 40000, seed=9),
    lambda: gen.stencil2d(31, 17, 9),
    lambda: gen.stencil3d(6, 5, 4, 7),
])
def test_generators_satisfy_contract(maker):
    g = maker()
    assert g.validate() == 0
    assert g.row_ptr[0] == 0 and g.row_ptr[-1] == g.nnz == len(g.col_idx)


def test_rmat_permute_preserves_degree_multiset():
    a = gen.rmat(13, 8, 0.57, 0.19, 0.19, seed=2)
    b = gen.rmat(13, 8, 0.57, 0.19, 0.19, seed=2, permute=True)
    assert a.nnz == b.nnz
    assert np.array_equal(np.sort(a.degrees), np.sort(b.degrees))
    assert not np.array_equal(a.degrees, b.degrees)


def test_rmat_unpermuted_hubs_are_low_ids():
    g = gen.config(1)
    d = g.degrees
    assert int(np.argmax(d)) == 0  # quadrant a=(0,0) dominates: vertex 0 is the top hub
    assert g.validate() == 0


def _hash_rmat(threads: int) -> str:
    code = ("import hashlib;from paper_conf_ipps_licqfsty16_b200 import gen;"
            "g=gen.rmat(14,8,0.57,0.19,0.19,seed=7);"
            "print(hashlib.sha1(g.row_ptr.tobytes()+g.col_idx.tobytes()).hexdigest())")
    env = dict(os.environ, OMP_NUM_THREADS=str(threads))
    out = subprocess.run([sys.executable, "-c", code], cwd=ROOT, env=env, check=True,
                         capture_output=True, text=True)
    return out.stdout.strip()


def test_generation_independent_of_thread_count():
    assert _hash_rmat(1) == _hash_rmat(3)


def test_er_degree_distribution():
    n = 1 << 16
    g = gen.er(n, 8 * n, seed=3)
    d = g.degrees
    assert abs(g.nnz - 16 * n) < 0.005 * 16 * n      # ~no loss to loops/dups at this density
    assert abs(d.mean() - 16) < 0.1 and abs(d.var() - 16) < 1.0  # ~Poisson(16)
    assert d.max() < 50


def test_table1_rmat_er_loose():
    """rmat-er: n=1,048,576, 20,971,268 edges, min/max/avg 2/59/20.00."""
    g = gen.rmat(20, 10, 0.25, 0.25, 0.25, seed=1)
    d = g.degrees
    assert g.n == 1_048_576
    assert abs(g.nnz - 20_971_268) / 20_971_268 < 1e-3
    assert abs(d.mean() - 20.0) < 0.05 and 1 <= d.min() <= 5 and 30 <= d.max() <= 80


def test_table1_rmat_g_loose():
    """rmat-g: 20,964,268 edges, min/max/avg/var 0/899/20.00/472.81."""
    g = gen.rmat(20, 10, 0.45, 0.15, 0.15, seed=1)
    d = g.degrees
    assert abs(g.nnz - 20_964_268) / 20_964_268 < 5e-3
    assert d.min() == 0 and 500 <= d.max() <= 1300
    assert abs(d.var() - 472.81) / 472.81 < 0.2
