"""Host-side pieces of bench.py (no GPU): the byte model of the roofline,
the launch count of the plan, the kernel label, the host description and the
all-core oracle timing (the CPU baseline's second figure)."""
import os
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import bench  # noqa: E402
from paper_conf_dsn_schollbkw16_b200 import inputs as G  # noqa: E402


def test_algorithmic_bytes_csr_model():
    # A: 12 B per entry + row_ptr, x read once + y written once; the check
    # adds C as streamed and K (8 B per block)
    n, nnz, nb = 1000, 7000, 32
    plain = bench.algorithmic_bytes(n, nnz, nb, 0, check=False)
    assert plain == 12 * nnz + 4 * (n + 1) + 16 * n
    assert bench.algorithmic_bytes(n, nnz, nb, 555) == plain + 555 + 8 * nb


@pytest.mark.parametrize("info, check, want", [
    ({"stream": 1}, True, 2),                                    # k_stream + k_finish
    ({"stream": 1, "general_groups": 3}, True, 3),               # + k_general
    ({"stream": 1}, False, 1),
    ({"lean": 1, "irr_groups": 5, "general_groups": 2}, True, 4),
    ({"col_perm": 1, "hub_chunks": 9, "irr_groups": 5, "general_groups": 2}, True, 5),
])
def test_fused_launches(info, check, want):
    assert bench.fused_launches(info, check=check) == want


def test_fused_kernel_name():
    assert bench.fused_kernel_name({"stream": 1, "stream_g": 8, "stream_stages": 4}).startswith(
        "k_stream<CHECK> (G=8, 4 stages)")
    assert "k_irr" in bench.fused_kernel_name({"irr_groups": 3})
    assert bench.fused_kernel_name({"lean": 1, "lean_short": 1}) == "k_lean<CHECK, SHORT>"


def test_host_cpu():
    cores, model = bench.host_cpu()
    assert cores >= 1
    assert model is None or isinstance(model, str)


def test_oracle_all_cores_counts_replicas():
    # every logical core runs the single-thread oracle; the rate is calls/s
    from oracle import oracle as O
    A = G.laplacian_2d_5pt(16)
    x = G.uniform_vector(A.n, 42)
    enc = O.encode(A, 32)
    rate, cores, reps = bench.oracle_all_cores(A, enc, x, seconds=0.3)
    assert cores == bench.host_cpu()[0]
    assert reps >= 1 and rate > 0
