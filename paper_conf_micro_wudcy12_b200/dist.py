"""Multi-GPU sharding of fused RA chains, one process per GPU.

torch.distributed carries the collectives (NCCL over NVLink on B200; gloo in the
CPU tests); every data-path step is a kernel call made through a Backend:

* row sharding (C1, C2, C4): rank r owns rows [r*N/P, (r+1)*N/P) and runs the whole
  fused chain locally with no communication; rank-order concatenation of the outputs
  equals the single-GPU output.  An aggregate (C4) is combined exactly: each rank
  exports its groups as int64 limbs (rw_plan_agg_export), one SUM all-reduce, then
  rw_plan_agg_import recombines the 128-bit sums.
* key-range sharding (C3, C5): sampled splitters -> rw_split_by_splitters on every
  locally sorted input -> one all_to_all_single of every relation's counts ->
  rw_pack_tuples + one all_to_all_single per relation (issued asynchronously) ->
  rw_merge_packed_runs (single pass, stable, by full tuple) overlapping the next
  relation's transfer -> the fused JOIN chain runs locally on the rank's key range.
  Rank-order concatenation equals the single-GPU output, order included, because key ranges are ordered by rank and the merge restores the
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


def packable(types: Sequence[str]) -> bool:
    """Tuples of <= 8 bytes travel as one order-preserving u64 image (rw_pack_tuples)."""
    return sum(WIDTH[t] for t in types) <= 8


WIDTH = {"i32": 4, "u32": 4, "i64": 8, "u64": 8, "u8": 1}


class Backend:
    """Kernel calls the orchestration needs.  Splitters and bounds stay on the device."""

    device = "cpu"

    def split(self, keys, key_type: str, splitters: torch.Tensor) -> torch.Tensor:
        """int64 tensor: rows with key < splitter, per splitter (splitters = int64 key values)."""
        raise NotImplementedError

    def pack(self, cols: Sequence[torch.Tensor], types: Sequence[str]) -> torch.Tensor:
        """Order-preserving u64 tuple images (int64 storage) of tuples <= 8 bytes."""
        raise NotImplementedError

    def merge_packed(self, packed: torch.Tensor, types: Sequence[str], run_off: Sequence[int]) -> List[torch.Tensor]:
        raise NotImplementedError

    def merge(self, cols: Sequence[torch.Tensor], types: Sequence[str], run_off: Sequence[int]) -> List[torch.Tensor]:
        raise NotImplementedError


class GpuBackend(Backend):
    """librw kernels (rw_split_by_splitters, rw_pack_tuples, rw_merge_packed_runs,
    rw_merge_runs) on the current stream."""

    def __init__(self, device: int = 0):
        self.device = f"cuda:{device}"
        self.dev = device

    def split(self, keys, key_type, splitters):
        from . import rw
        n = int(keys.numel())
        ns = int(splitters.numel())
        bounds = torch.empty(max(1, ns), dtype=torch.int64, device=self.device)
        if ns:
            spl = from_key_values(splitters, key_type).to(self.device)
            rw.split_by_splitters(keys, n, key_type, spl, ns, bounds, torch.cuda.current_stream())
        return bounds[:ns]

    def pack(self, cols, types):
        from . import rw
        n = int(cols[0].numel())
        out = torch.empty(max(n, 1), dtype=torch.int64, device=self.device)
        if n:
            rw.pack_tuples(list(cols), list(types), n, out, torch.cuda.current_stream())
        return out[:n]

    def merge_packed(self, packed, types, run_off):
        from . import rw
        total = int(run_off[-1] - run_off[0])
        outs = [torch.empty(max(total, 1), dtype=STORAGE[t], device=self.device) for t in types]
        if total:
            rw.merge_packed_runs(packed, list(types), list(run_off), outs, torch.cuda.current_stream())
        return [o[:total] for o in outs]

    def merge(self, cols, types, run_off):
        from . import rw
        total = int(run_off[-1] - run_off[0])
        outs = [torch.empty(max(total, 1), dtype=STORAGE[t], device=self.device) for t in types]
        if total:
            rw.merge_runs(list(cols), list(types), list(run_off), outs, torch.cuda.current_stream())
        return [o[:total] for o in outs]


def choose_splitters(local_keys: Sequence[Tuple[torch.Tensor, str]], world: int, samples: int = 1024,
                     group=None) -> torch.Tensor:
    """P-1 splitters (int64 key values, a device tensor) from evenly spaced samples of
    every rank's locally sorted key columns, gathered with all_gather (one small
    collective); no host round trip."""
    dev = local_keys[0][0].device
    parts = []
    for keys, kt in local_keys:
        n = int(keys.numel())
        if n:
            pos = torch.linspace(0, n - 1, min(samples, n), device=dev).round().to(torch.int64)
            parts.append(key_values(keys.index_select(0, pos), kt))
    mine = torch.cat(parts) if parts else torch.zeros(0, dtype=torch.int64, device=dev)
    # fixed-size buffer so all_gather shapes agree: buf[0] = number of samples, then the
    # samples (key values as int64; i32/i64 keys may be negative), the rest unused
    width = samples * len(local_keys)
    buf = torch.zeros(width + 1, dtype=torch.int64, device=dev)
    buf[0] = mine.numel()
    buf[1:1 + mine.numel()] = mine
    got = [torch.empty_like(buf) for _ in range(world)]
    dist.all_gather(got, buf, group=group)
    allb = torch.stack(got)
    cnt = allb[:, 0]
    valid = torch.arange(width, device=dev)[None, :] < cnt[:, None]
    vals = torch.where(valid, allb[:, 1:], torch.full_like(allb[:, 1:], torch.iinfo(torch.int64).max))
    srt, _ = torch.sort(vals.flatten())
    total = cnt.sum()
    idx = (total * torch.arange(1, world, device=dev)) // world
    idx = torch.minimum(idx, torch.clamp(total - 1, min=0))
    return torch.where(total > 0, srt[idx], torch.zeros_like(idx))


def exchange_all(backend: Backend, rels: Dict[str, List[torch.Tensor]], schema: Dict[str, List[str]],
                 world: int, samples: int = 1024, group=None) -> Dict[str, List[torch.Tensor]]:
    """Key-range shard every input relation with one shared set of splitters: returns
    this rank's key range of each global relation, sorted (stable, full tuple).

    One all_to_all_single carries every relation's per-destination counts and ONE host
    read brings them back (the only host round trip: NCCL needs the split sizes).  Each
    relation whose tuples fit 8 bytes is packed into order-preserving u64 images
    (rw_pack_tuples) and sent in ONE all_to_all_single; all transfers are issued
    asynchronously before the first merge, so relation k's merge (rw_merge_packed_runs,
    one read + one write) overlaps the transfers of relations k+1, ...  Wider tuples
    fall back to one all_to_all_single per column and rw_merge_runs."""
    names = list(rels)
    spl = choose_splitters([(rels[k][0], schema[k][0]) for k in names], world, samples, group)
    dev = rels[names[0]][0].device
    send = []
    for k in names:
        n = int(rels[k][0].numel())
        b = backend.split(rels[k][0], schema[k][0], spl)
        cuts = torch.cat([torch.zeros(1, dtype=torch.int64, device=dev), b.to(torch.int64),
                          torch.full((1,), n, dtype=torch.int64, device=dev)])
        send.append(cuts[1:] - cuts[:-1])
    sc = torch.stack(send, 1).contiguous()            # [dst rank][relation]
    rc = torch.empty_like(sc)
    dist.all_to_all_single(rc, sc, group=group)       # rc: [src rank][relation]
    both = torch.stack([sc, rc]).cpu()
    pending = []
    for i, k in enumerate(names):
        s_i = [int(x) for x in both[0, :, i]]
        r_i = [int(x) for x in both[1, :, i]]
        tot = sum(r_i)
        types = schema[k]
        if packable(types):
            buf = backend.pack(rels[k], types)
            out = torch.empty(max(tot, 1), dtype=torch.int64, device=dev)[:tot]
            work = dist.all_to_all_single(out, buf, output_split_sizes=r_i, input_split_sizes=s_i,
                                          group=group, async_op=True)
            pending.append((k, types, r_i, [out], work, True))
        else:
            outs, works = [], []
            for c in rels[k]:
                o = torch.empty(max(tot, 1), dtype=c.dtype, device=dev)[:tot]
                works.append(dist.all_to_all_single(o, c.contiguous(), output_split_sizes=r_i,
                                                    input_split_sizes=s_i, group=group, async_op=True))
                outs.append(o)
            pending.append((k, types, r_i, outs, works, False))
    result = {}
    for k, types, r_i, outs, work, packed in pending:
        for w in (work if isinstance(work, list) else [work]):
            w.wait()
        run_off = [0]
        for r in r_i:
            run_off.append(run_off[-1] + r)
        result[k] = backend.merge_packed(outs[0], types, run_off) if packed else backend.merge(outs, types, run_off)
    return result


def exchange(backend: Backend, cols: Sequence[torch.Tensor], types: Sequence[str], splitters,
             world: int, group=None) -> List[torch.Tensor]:
    """Key-range redistribution of one locally sorted relation with given splitters
    (int64 key values) -- exchange_all without the splitter choice."""
    spl = torch.as_tensor(splitters, dtype=torch.int64, device=cols[0].device)
    n = int(cols[0].numel())
    dev = cols[0].device
    b = backend.split(cols[0], types[0], spl)
    cuts = torch.cat([torch.zeros(1, dtype=torch.int64, device=dev), b.to(torch.int64),
                      torch.full((1,), n, dtype=torch.int64, device=dev)])
    sc = (cuts[1:] - cuts[:-1]).contiguous()
    rc = torch.empty_like(sc)
    dist.all_to_all_single(rc, sc, group=group)
    both = torch.stack([sc, rc]).cpu()
    s_i, r_i = [int(x) for x in both[0]], [int(x) for x in both[1]]
    tot = sum(r_i)
    run_off = [0]
    for r in r_i:
        run_off.append(run_off[-1] + r)
    if packable(types):
        buf = backend.pack(cols, types)
        out = torch.empty(max(tot, 1), dtype=torch.int64, device=dev)[:tot]
        dist.all_to_all_single(out, buf, output_split_sizes=r_i, input_split_sizes=s_i, group=group)
        return backend.merge_packed(out, types, run_off)
    outs = []
    for c in cols:
        o = torch.empty(max(tot, 1), dtype=c.dtype, device=dev)[:tot]
        dist.all_to_all_single(o, c.contiguous(), output_split_sizes=r_i, input_split_sizes=s_i, group=group)
        outs.append(o)
    return backend.merge(outs, types, run_off)


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
