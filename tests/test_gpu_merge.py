"""GPU: the single-pass P-way merge of the key-range exchange (rw_merge_runs,
rw_pack_tuples + rw_merge_packed_runs; merge_p.cu), through the C-ABI, against a
numpy stable lexicographic sort of the concatenated runs (the merge of sorted runs
is the stable sort of their concatenation, P:196 merge path; equal tuples keep run
order, which for identical tuples is invisible, so the result is unique)."""
import numpy as np
import pytest
import torch

pytestmark = pytest.mark.gpu
DEV = "cuda:0"

NP = {"i32": np.int32, "u32": np.uint32, "i64": np.int64, "u64": np.uint64, "u8": np.uint8}
TORCH = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}


def make_runs(rng, types, lens, domain):
    """Each run sorted lexicographically on all columns (in the declared types)."""
    runs = []
    for n in lens:
        cols = []
        for t in types:
            info = np.iinfo(NP[t])
            lo = max(info.min, -domain) if info.min < 0 else 0
            hi = min(info.max, domain)
            cols.append(rng.integers(lo, hi, size=n, endpoint=True, dtype=np.int64).astype(NP[t]))
        order = np.lexsort(tuple(reversed(cols))) if n else np.zeros(0, dtype=np.int64)
        runs.append([c[order] for c in cols])
    return runs


def expected(runs, types):
    cat = [np.concatenate([r[c] for r in runs]) for c in range(len(types))]
    order = np.lexsort(tuple(reversed(cat)))
    return [c[order] for c in cat]


def to_dev(a, t):
    return torch.from_numpy(a.view(np.int32) if t == "u32" else a.view(np.int64) if t == "u64" else a).to(DEV)


def from_dev(x, t):
    return x.cpu().numpy().view(NP[t])


def run_merge(runs, types, packed):
    from paper_conf_micro_wudcy12_b200 import dist as rd
    be = rd.GpuBackend(0)
    cols = [to_dev(np.concatenate([r[c] for r in runs]), t) for c, t in enumerate(types)]
    run_off = [0]
    for r in runs:
        run_off.append(run_off[-1] + len(r[0]))
    if packed:
        buf = be.pack(cols, types)
        out = be.merge_packed(buf, types, run_off)
    else:
        out = be.merge(cols, types, run_off)
    torch.cuda.synchronize()
    return [from_dev(o, t) for o, t in zip(out, types)]


CASES = [
    (["u32", "u32"], 1 << 20),
    (["i32", "i32"], 1 << 30),
    (["i64"], 1 << 40),
    (["u64"], 1 << 62),
    (["i32", "u8", "u8"], 100),
    (["u8", "i32"], 3),          # heavy duplicates: few distinct tuples
]


@pytest.mark.parametrize("packed", [False, True])
@pytest.mark.parametrize("P", [2, 3, 8, 17, 32])
@pytest.mark.parametrize("case", range(len(CASES)))
def test_merge_single_pass_matches_stable_sort(case, P, packed):
    types, domain = CASES[case]
    rng = np.random.default_rng(1000 * case + P)
    lens = [int(x) for x in rng.integers(0, 40_000, size=P)]
    lens[P // 2] = 0                                   # an empty run
    runs = make_runs(rng, types, lens, domain)
    got = run_merge(runs, types, packed)
    for g, e in zip(got, expected(runs, types)):
        np.testing.assert_array_equal(g, e)


@pytest.mark.parametrize("packed", [False, True])
def test_merge_single_pass_all_equal_and_ragged(packed):
    """Every tuple equal (one group boundary per sample, maximal ties), tiny runs."""
    types = ["u32", "u32"]
    for lens in ([1, 1], [5, 0, 7], [4096, 4095, 1], [0, 0, 3], [12345] * 8):
        runs = [[np.full(n, 7, np.uint32), np.full(n, 9, np.uint32)] for n in lens]
        got = run_merge(runs, types, packed)
        for g, e in zip(got, expected(runs, types)):
            np.testing.assert_array_equal(g, e)


def test_merge_large_p8():
    """C5-shaped: 8 runs of 2^21 (u32 key, u32 val) rows, keys from a shared range."""
    rng = np.random.default_rng(7)
    runs = make_runs(rng, ["u32", "u32"], [1 << 21] * 8, 1 << 24)
    got = run_merge(runs, ["u32", "u32"], True)
    for g, e in zip(got, expected(runs, ["u32", "u32"])):
        np.testing.assert_array_equal(g, e)


@pytest.mark.parametrize("types", [["u32", "u32"], ["i64"], ["i32", "u8"]])
def test_packed_single_run_roundtrip(types):
    """One received run (P = 1, or the other ranks sent nothing): pack, then unpack
    through the merge kernels, is the identity."""
    rng = np.random.default_rng(11)
    runs = make_runs(rng, types, [70_001], 1 << 20)
    got = run_merge(runs, types, True)
    for g, e in zip(got, runs[0]):
        np.testing.assert_array_equal(g, e)


@pytest.mark.parametrize("types", [["i64", "i32"], ["u32", "u32"]])
def test_merge_tree_fallback(types):
    """Tuples over 8 bytes, or more than 32 runs, take the pairwise merge tree."""
    rng = np.random.default_rng(3)
    P = 2 if types == ["i64", "i32"] else 40
    runs = make_runs(rng, types, [int(x) for x in rng.integers(0, 3000, size=P)], 50)
    got = run_merge(runs, types, False)
    for g, e in zip(got, expected(runs, types)):
        np.testing.assert_array_equal(g, e)
