"""Multi-GPU sharding of fused RA chains, one process per GPU.

torch.distributed carries the collectives (NCCL over NVLink on B200; gloo in the
CPU tests); every data-path step is a kernel call made through a Backend:

* row sharding (C1, C2, C4): rank r owns rows [r*N/P, (r+1)*N/P) and runs the whole
  fused chain locally with no communication; rank-order concatenation of the outputs
  equals the single-GPU output.  An aggregate (C4) is combined exactly: each rank
  exports its groups as int64 limbs (rw_plan_agg_export), one SUM all-reduce, then
  rw_plan_agg_import recombines the 128-bit sums.
* key-range sharding (C3, C5): sampled splitters -> rw_split_by_splitters on every
  locally sorted input -> all_to_all_single of counts, then of every column ->
  rw_merge_runs (stable, by full tuple) -> the fused JOIN chain runs locally on the
  rank's key range.  Rank-order concatenation equals the single-GPU output, order
  included, because key ranges are ordered by rank and the merge restores the
  global (key, row) order inside each range.

The Backend abstraction is what lets tests/test_dist_gloo.py run the very same
orchestration on CPU with world_size 2 (its backend wraps the oracle); the product
backend, GpuBackend, has no CPU path.
"""
from __future__ import annotations

from typing import Dict, List, Sequence, Tuple

import torch
import torch.distributed as dist

STORAGE = {"i32": torch.int32, "u32": torch.int32, "i64": torch.int64, "u64": torch.int64, "u8": torch.uint8}


def row_range(n_total: int, rank: int, world: int) -> Tuple[int, int]:
    """[start, start+count) of rank's rows under an even row partition."""
    start = n_total * rank // world
    end = n_total * (rank + 1) // world
    return start, end - start


def key_values(keys: torch.Tensor, key_type: str) -> torch.Tensor:
    """Key column as int64 values that sort like the declared type (u32 stored in int32)."""
    if key_type == "u32":
        return keys.to(torch.int64) & 0xFFFFFFFF
    if key_type == "u64":
        return keys.to(torch.int64) ^ (-(1 << 63))           # order-preserving for uint64 bits
    return keys.to(torch.int64)


def from_key_values(v: torch.Tensor, key_type: str) -> torch.Tensor:
    if key_type == "u32":
        return torch.where(v >= (1 << 31), v - (1 << 32), v).to(torch.int32)
    if key_type == "u64":
        return (v ^ (-(1 << 63))).to(torch.int64)
    return v.to(STORAGE[key_type])


class Backend:
    """Kernel calls the orchestration needs."""

    device = "cpu"

    def split(self, keys, key_type: str, splitters) -> List[int]:
        raise NotImplementedError

    def merge(self, cols: Sequence[torch.Tensor], types: Sequence[str], run_off: Sequence[int]) -> List[torch.Tensor]:
        raise NotImplementedError


class GpuBackend(Backend):
    """librw kernels (rw_split_by_splitters, rw_merge_runs) on the current stream."""

    def __init__(self, device: int = 0):
        self.device = f"cuda:{device}"
        self.dev = device

    def split(self, keys, key_type, splitters):
        from . import rw
        n = int(keys.numel())
        bounds = torch.empty(max(1, len(splitters)), dtype=torch.int64, device=self.device)
        spl = from_key_values(torch.as_tensor(splitters, dtype=torch.int64), key_type).to(self.device)
        if len(splitters):
            rw.split_by_splitters(keys, n, key_type, spl, len(splitters), bounds, torch.cuda.current_stream())
        return bounds[: len(splitters)].tolist()

    def merge(self, cols, types, run_off):
        from . import rw
        total = int(run_off[-1] - run_off[0])
        outs = [torch.empty(max(total, 1), dtype=STORAGE[t], device=self.device) for t in types]
        if total:
            rw.merge_runs(list(cols), list(types), list(run_off), outs, torch.cuda.current_stream())
        return [o[:total] for o in outs]


def choose_splitters(local_keys: Sequence[Tuple[torch.Tensor, str]], world: int, samples: int = 1024,
                     group=None) -> List[int]:
    """P-1 splitters (int64 key values) from evenly spaced samples of every rank's
    locally sorted key columns, gathered with all_gather (one small collective)."""
    parts = []
    for keys, kt in local_keys:
        n = int(keys.numel())
        if n:
            pos = torch.linspace(0, n - 1, min(samples, n)).round().to(torch.int64).to(keys.device)
            parts.append(key_values(keys.index_select(0, pos), kt))
    mine = torch.cat(parts) if parts else torch.zeros(0, dtype=torch.int64, device=local_keys[0][0].device)
    # fixed-size buffer so all_gather shapes agree: buf[0] = number of samples, then the
    # samples (key values as int64; i32/i64 keys may be negative), the rest unused
    width = samples * len(local_keys)
    buf = torch.full((width + 1,), 0, dtype=torch.int64, device=mine.device)
    buf[0] = mine.numel()
    buf[1:1 + mine.numel()] = mine
    got = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(got, buf, group=group)
    allv = torch.cat([g[1:1 + int(g[0].item())] for g in got]).cpu()
    if allv.numel() == 0:
        return [0] * (world - 1)
    allv, _ = torch.sort(allv)
    idx = [(allv.numel() * (r + 1)) // world for r in range(world - 1)]
    return [int(allv[min(i, allv.numel() - 1)].item()) for i in idx]


def exchange(backend: Backend, cols: Sequence[torch.Tensor], types: Sequence[str], splitters: Sequence[int],
             world: int, group=None) -> List[torch.Tensor]:
    """Key-range redistribution of one locally sorted relation: returns this rank's
    key range of the global relation, sorted (stable, full tuple)."""
    n = int(cols[0].numel())
    bounds = backend.split(cols[0], types[0], splitters)
    cuts = [0] + [int(b) for b in bounds] + [n]
    send = [cuts[r + 1] - cuts[r] for r in range(world)]
    sc = torch.tensor(send, dtype=torch.int64, device=cols[0].device)
    rc = torch.empty_like(sc)
    dist.all_to_all_single(rc, sc, group=group)
    recv = [int(x) for x in rc.tolist()]
    out = []
    for c, t in zip(cols, types):
        o = torch.empty(max(sum(recv), 1), dtype=c.dtype, device=c.device)[: sum(recv)]
        dist.all_to_all_single(o, c.contiguous(), output_split_sizes=recv, input_split_sizes=send, group=group)
        out.append(o)
    run_off = [0]
    for r in recv:
        run_off.append(run_off[-1] + r)
    return backend.merge(out, types, run_off)


def exchange_all(backend: Backend, rels: Dict[str, List[torch.Tensor]], schema: Dict[str, List[str]],
                 world: int, samples: int = 1024, group=None) -> Dict[str, List[torch.Tensor]]:
    """Key-range shard every input relation with one shared set of splitters."""
    spl = choose_splitters([(rels[k][0], schema[k][0]) for k in rels], world, samples, group)
    return {k: exchange(backend, rels[k], schema[k], spl, world, group) for k in rels}


def allreduce_limbs(limbs: torch.Tensor, group=None) -> torch.Tensor:
    """Exact combine of exported aggregate limbs (int64 SUM; limbs are < 2^32)."""
    dist.all_reduce(limbs, op=dist.ReduceOp.SUM, group=group)
    return limbs


def run_aggregate_sharded(plan, node: int, local_inputs, capacity: int, group=None):
    """C4 on P GPUs: local fused select/arith/agg, limb export, one all-reduce, import.
    Returns (result columns, rows) identical on every rank."""
    local_cols, n_local = plan.run(local_inputs, node, capacity)
    limbs = plan.agg_export(node, local_cols, n_host=n_local)
    allreduce_limbs(limbs, group)
    types = plan.node_schema(node)
    outs = [torch.empty(capacity, dtype=STORAGE[t], device=f"cuda:{plan.device}") for t in types]
    n = plan.agg_import(node, limbs, outs, capacity)
    return [o[:n] for o in outs], n
