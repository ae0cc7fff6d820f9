"""GPU parity of host-streamed execution (§5.1.3): HOST
inputs run chunk by chunk with H2D / kernel / D2H overlapped on three streams.  The
result must equal the oracle element by element, row order included, for chains,
aggregates (one finalisation over every chunk) and ragged last chunks."""
import numpy as np
import pytest
import torch

import workloads
from tests.planspec import NPT, assert_same, build_gpu_plan, run_oracle
import oracle

pytestmark = pytest.mark.gpu


def run_host(spec, ins, chunk_log2, capacity=None):
    plan, ids = build_gpu_plan(spec, host_chunk_log2=chunk_log2)
    node = ids[spec["out"]]
    types = plan.node_schema(node)
    host_in = [(int(ins[k][0].numel()), [c.cpu().pin_memory() for c in ins[k]]) for k in spec["inputs"]]
    n_in = max(n for n, _ in host_in)
    cap = capacity if capacity is not None else max(n_in, 1)
    dt = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}
    outs = [torch.empty(max(cap, 1), dtype=dt[t]).pin_memory() for t in types]
    n = plan.execute_host(host_in, node, outs, cap)
    rel = oracle.Relation(types, [o[:n].numpy().view(NPT[t]) for o, t in zip(outs, types)])
    return rel, plan


@pytest.mark.parametrize("n,lg", [(100_003, 12), (4096 * 5, 12), (4096 * 5 + 1, 12), (1_000_000, 16), (3, 12)])
def test_c2_streamed(n, lg):
    spec = workloads.c2_spec()
    ins = workloads.c2_inputs(n, cfg=0xa1)
    got, plan = run_host(spec, ins, lg)
    assert_same(got, run_oracle(spec, ins))


@pytest.mark.parametrize("n", [10_001, 300_007])
def test_q1_streamed_aggregate(n):
    spec = workloads.c4_spec()
    ins = workloads.c4_inputs(n, cfg=0xa2)
    got, plan = run_host(spec, ins, 12, capacity=6)
    assert_same(got, run_oracle(spec, ins))


def test_streamed_capacity_error():
    from paper_conf_micro_wudcy12_b200 import rw
    spec = workloads.c1_spec()
    ins = workloads.c1_inputs(50_000, cfg=0xa3)
    with pytest.raises(rw.RwError) as e:
        run_host(spec, ins, 12, capacity=100)
    assert e.value.name == "RW_E_CAPACITY"
    # the plan stays usable afterwards
    got, _ = run_host(spec, ins, 12)
    assert_same(got, run_oracle(spec, ins))


def test_join_plan_is_copied_whole():
    spec = workloads.c3_spec()
    ins = workloads.c3_inputs(20_000, cfg=0xa4)
    got, _ = run_host(spec, ins, 12, capacity=400_000)
    assert_same(got, run_oracle(spec, ins))
