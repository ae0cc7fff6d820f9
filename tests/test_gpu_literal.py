"""The hand-worked workload results of tests/test_oracle_evaluate.py, run through the
CUDA path (C-ABI, fused and operator-at-a-time): pins the GPU side's reading of the
plan spec (tests/planspec.build_gpu_plan) to the same literals, independently of
the oracle."""
import numpy as np
import pytest

import workloads
from tests import test_oracle_evaluate as lit
from tests.planspec import run_gpu

pytestmark = pytest.mark.gpu

NPT = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "u8": np.uint8}


def gpu_rows(spec, rows, fuse):
    import torch
    ins = {}
    for name, inp in spec["inputs"].items():
        ins[name] = [torch.from_numpy(np.array([r[c] for r in rows[name]], dtype=NPT[t]).view(
            {"u32": np.int32, "u64": np.int64}.get(t, NPT[t]))).cuda() for c, t in enumerate(inp["types"])]
    got, _ = run_gpu(spec, ins, capacity=64, fuse=fuse)
    return got.types, got.rows()


CASES = {
    "c1": (workloads.c1_spec, lambda: {"R": [(0, 0), (1 << 31, 0), (5, 1 << 31), ((1 << 31) - 1, (1 << 31) - 1)]}),
    "c2": (workloads.c2_spec, lambda: {"R": [(1, -5, 2, -3), (2, 5, 3, -4), (3, -1, 4, 7), (4, -(1 << 31), 5, -(1 << 31))]}),
    "c3": (workloads.c3_spec, lambda: {"L": [(1, 5), (1, 7), (2, 1)], "R": [(1, 6), (2, 0), (3, 9)]}),
    "c5": (workloads.c5_spec, lambda: {"R": [(1, 1), (2, 5)], "S": [(1, 10), (1, 11), (2, 3)], "T": [(1, 0), (2, 9)]}),
}


@pytest.mark.parametrize("fuse", [True, False])
@pytest.mark.parametrize("name", sorted(CASES))
def test_literal_workloads_on_gpu(name, fuse):
    mk, rows = CASES[name]
    spec = mk()
    assert gpu_rows(spec, rows(), fuse) == lit.oracle_rows(spec, rows())
    expect = {"c1": [(0, 0), ((1 << 31) - 1, (1 << 31) - 1)], "c2": [(1, 2, -3), (4, 5, -(1 << 31))],
              "c3": [(1, 6)], "c5": [(2, 5, 3, 9)]}[name]
    assert gpu_rows(spec, rows(), fuse)[1] == expect


@pytest.mark.parametrize("fuse", [True, False])
def test_literal_q1_on_gpu(fuse):
    import rwgen
    D = rwgen.D_1998_09_02
    rows = {"lineitem": [(D - 1, 100, 1000, 5, 2, 0, 1), (D + 1, 100, 7, 7, 7, 0, 1),
                         (D, 200, 3000, 0, 8, 0, 1), (D - 10, 50 + 50, 500, 10, 0, 2, 0)]}
    types, got = gpu_rows(workloads.c4_spec(), rows, fuse)
    assert got == [(0, 1, 2, 300, 0, 4000, 0, 395000, 0, 42090000, 0, 5, 0),
                   (2, 0, 1, 100, 0, 500, 0, 45000, 0, 4500000, 0, 10, 0)]
