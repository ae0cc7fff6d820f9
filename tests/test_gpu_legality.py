"""Fusion legality pins (§4.1 Fig. 8; Fig. 14): the edge
classes and fusion decisions rw_plan_explain reports for the paper's five patterns
(a) back-to-back SELECTs: thread, fused; (b) JOIN -> JOIN on one key: CTA, fused;
(c) SELECTs feeding a JOIN: CTA, fused; (d) SELECTs sharing an input: fused by
input dependence (one launch); (e) arithmetic: thread, fused; and the kernel
dependences: an AGG output feeding anything, a JOIN on an unsorted input."""
import pytest

import workloads
from tests.planspec import build_gpu_plan, run_gpu_multi

pytestmark = pytest.mark.gpu
DEV = "cuda:0"


def explain(spec, out=None, **o):
    plan, ids = build_gpu_plan(spec, device=0, **o)
    return plan.explain(ids[out or spec["out"]]), ids


def edge(ex, a, b):
    for line in ex.splitlines():
        if f"{a}(" in line and f"-> {b}(" in line:
            return line.split(": ", 1)[1]
    raise AssertionError(f"edge {a}->{b} missing:\n{ex}")


def test_pattern_a_back_to_back_selects_thread_fused():
    ex, ids = explain(workloads.c1_spec())
    assert edge(ex, ids["s1"], ids["s2"]) == "thread dependence, fused"
    assert ex.count("group ") == 1


def test_pattern_b_join_join_cta_fused():
    ex, ids = explain(workloads.c5_spec())
    assert edge(ex, ids["rs"], ids["rst"]) == "CTA dependence, fused"
    assert edge(ex, ids["rst"], ids["s"]) == "thread dependence, fused"
    assert ex.count("group ") == 1 and "3 inputs" in ex


def test_pattern_c_selects_feeding_a_join_cta_fused():
    spec = workloads.cc_spec()
    spec["nodes"].insert(2, {"id": "fv", "op": "select", "in": "fr", "preds": [(1, "<", 7)]})
    spec["nodes"][3]["right"] = "fv"
    ex, ids = explain(spec)
    assert edge(ex, ids["fl"], ids["j"]) == "CTA dependence, fused"
    assert edge(ex, ids["fv"], ids["j"]) == "CTA dependence, fused"
    assert ex.count("group ") == 1
    assert "key SELECT" in ex and "fused into the expansion" in ex


def test_pattern_d_input_dependence_one_launch():
    spec = workloads.cd_spec(0.25, 3)
    ins = workloads.cd_inputs(20_000, device=DEV)
    _, plan = run_gpu_multi(spec, ins)
    assert plan.last_launches() == 1


def test_pattern_e_arithmetic_thread_fused():
    ex, ids = explain(workloads.c4_spec())
    assert edge(ex, ids["s"], ids["p"]) == "thread dependence, fused"
    assert edge(ex, ids["p"], ids["g"]) == "CTA dependence, fused"
    assert ex.count("group ") == 1


def test_agg_output_is_a_kernel_dependence():
    spec = workloads.c4_spec()
    spec["nodes"].append({"id": "after", "op": "select", "in": "g", "preds": [(2, ">", 0)]})
    spec["out"] = "after"
    ex, ids = explain(spec)
    assert edge(ex, ids["g"], ids["after"]) == "kernel dependence, materialised"
    assert "group 1" in ex


def test_operator_at_a_time_materialises_every_edge():
    ex, ids = explain(workloads.c2_spec(), fuse=False)
    assert edge(ex, ids["s1"], ids["p"]) == "thread dependence, materialised"
    assert ex.count("group ") == 3
