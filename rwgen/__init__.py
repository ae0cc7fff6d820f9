"""Seeded synthetic relation generators shared by the oracle side and the CUDA side.

This module holds NO relational-algebra arithmetic: it only produces input
columns (SURVEY.md §8(d) "Concrete synthetic inputs").  Both the tests / bench
(CUDA path) and the oracle side draw their inputs from here, so the two
implementations see bit-identical relations without sharing any method code.

Generator (stateless per row, so any rank can produce any row range):
    x(seed, i) = mix64(seed + (i + 1) * GOLDEN)  (mod 2^64)
    mix64      = the SplitMix64 finaliser (Steele, Lea, Flood 2014)
    u32        = x >> 32
    int[a, b]  = a + ((x >> 32) * (b - a + 1)) >> 32      (Lemire multiply-shift)
    unit f64   = (x >> 11) * 2^-53
Column seeds: seed_col(cfg, rel, col) = mix64(0x4B57_0000_0000_0000 | cfg<<16 | rel<<8 | col).

Implemented with torch int64 tensors (two's complement wrap on multiply) so the
same code runs on CPU (oracle inputs, tests) and on CUDA (bench inputs, no host
round trip for 8 GiB relations).  `tests/test_gen.py` pins it against a numpy
uint64 implementation.
"""
from __future__ import annotations

import math
from typing import Dict, Optional

import torch

GOLDEN = 0x9E3779B97F4A7C15
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB
SEED_TAG = 0x4B57000000000000

_MASK64 = (1 << 64) - 1


def _s64(v: int) -> int:
    """Reinterpret an unsigned 64-bit python int as a signed int64 value."""
    v &= _MASK64
    return v - (1 << 64) if v >= (1 << 63) else v


def mix64_int(z: int) -> int:
    """SplitMix64 finaliser on a python int (exact, mod 2^64)."""
    z &= _MASK64
    z = ((z ^ (z >> 30)) * M1) & _MASK64
    z = ((z ^ (z >> 27)) * M2) & _MASK64
    return z ^ (z >> 31)


def seed_col(cfg: int, rel: int, col: int) -> int:
    return mix64_int(SEED_TAG | (cfg << 16) | (rel << 8) | col)


def _lsr(z: torch.Tensor, k: int) -> torch.Tensor:
    """Logical right shift of int64 tensors holding uint64 bit patterns."""
    return (z >> k) & ((1 << (64 - k)) - 1)


def _mix64(z: torch.Tensor) -> torch.Tensor:
    z = (z ^ _lsr(z, 30)) * _s64(M1)
    z = (z ^ _lsr(z, 27)) * _s64(M2)
    return z ^ _lsr(z, 31)


def raw64(seed: int, start: int, n: int, device="cpu") -> torch.Tensor:
    """x(seed, i) for i in [start, start+n) as int64 bit patterns."""
    i = torch.arange(start + 1, start + n + 1, dtype=torch.int64, device=device)
    z = i * _s64(GOLDEN) + _s64(seed)
    return _mix64(z)


def u32(seed: int, start: int, n: int, device="cpu") -> torch.Tensor:
    """Uniform uint32 values, returned as int64 in [0, 2^32)."""
    return _lsr(raw64(seed, start, n, device), 32)


def uniform_int(seed: int, start: int, n: int, lo: int, hi: int, device="cpu") -> torch.Tensor:
    """Uniform integers in [lo, hi] (hi - lo + 1 <= 2^31), int64 tensor."""
    span = hi - lo + 1
    assert 0 < span <= (1 << 31)
    return lo + ((u32(seed, start, n, device) * span) >> 32)


def unit_f64(seed: int, start: int, n: int, device="cpu") -> torch.Tensor:
    return _lsr(raw64(seed, start, n, device), 11).to(torch.float64) * (2.0 ** -53)


def to_u32_storage(v: torch.Tensor) -> torch.Tensor:
    """int64 values in [0, 2^32) -> int32 tensor holding the same 32-bit patterns."""
    return torch.where(v >= (1 << 31), v - (1 << 32), v).to(torch.int32)


def _chunked(fn, n: int, device, chunk: int = 1 << 25, dim: int = 0):
    outs = []
    for s in range(0, n, chunk):
        outs.append(fn(s, min(chunk, n - s)))
    if not outs:
        return fn(0, 0)
    return torch.cat(outs, dim=dim) if len(outs) > 1 else outs[0]


# ----------------------------------------------------------------------------
# Relations shaped like BASELINE.json configs
# ----------------------------------------------------------------------------

def uniform_u32_relation(cfg: int, rel: int, ncols: int, start: int, n: int,
                         device="cpu") -> Dict[str, torch.Tensor]:
    """`ncols` i.i.d. uniform 32-bit columns (C1, C2).  Stored as int32 bit patterns;
    callers declare the column type (u32 for C1, i32 for C2)."""
    out = {}
    for c in range(ncols):
        sd = seed_col(cfg, rel, c)
        out[f"c{c}"] = _chunked(lambda s, m: to_u32_storage(u32(sd, start + s, m, device)), n, device)
    return out


def zipf_cdf(K: int, alpha: float = 0.5, device="cpu") -> torch.Tensor:
    """Cumulative distribution of p(r) ∝ r^-alpha, r = 1..K (float64, fixed summation order)."""
    r = torch.arange(1, K + 1, dtype=torch.float64, device=device)
    w = r.pow(-alpha)
    c = torch.cumsum(w, 0)
    return c / c[-1]


ZIPF_BIJECTION = 0x9E3779B1


def zipf_keys(seed: int, start: int, n: int, K: int, alpha: float = 0.5,
              device="cpu", cdf: Optional[torch.Tensor] = None) -> torch.Tensor:
    """Zipf(alpha) ranks mapped to u32 keys by key = rank * 0x9E3779B1 mod 2^32
    (SURVEY.md §8(c) A15).  Returned as int64 in [0, 2^32)."""
    if cdf is None:
        cdf = zipf_cdf(K, alpha, device)
    def one(s, m):
        u = unit_f64(seed, start + s, m, device)
        rank = torch.searchsorted(cdf, u, right=True).clamp_(max=K - 1) + 1
        return (rank * ZIPF_BIJECTION) & 0xFFFFFFFF
    return _chunked(one, n, device)


def sort_by_key_val(key: torch.Tensor, val: torch.Tensor):
    """Sort (u32 key, u32 val) pairs (int64 holders) by (key, val) unsigned: A6 total order."""
    comb = (key << 32) | val          # < 2^64 as unsigned; flip sign bit for signed sort
    comb = comb ^ (-(1 << 63))
    s, _ = torch.sort(comb)
    s = s ^ (-(1 << 63))
    return _lsr(s, 32), s & 0xFFFFFFFF


def zipf_join_relation(cfg: int, rel: int, n: int, K: int, device="cpu",
                       cdf: Optional[torch.Tensor] = None) -> Dict[str, torch.Tensor]:
    """C3 input: (key u32 Zipf, val u32 uniform), sorted by (key, val); int32 storage."""
    k = zipf_keys(seed_col(cfg, rel, 0), 0, n, K, device=device, cdf=cdf)
    v = u32(seed_col(cfg, rel, 1), 0, n, device)
    k, v = sort_by_key_val(k, v)
    return {"key": to_u32_storage(k), "val": to_u32_storage(v)}


def uniform_join_relation(cfg: int, rel: int, start: int, n: int, key_space: int,
                          device="cpu", sort: bool = True) -> Dict[str, torch.Tensor]:
    """C5 input: key uniform in [0, key_space), val uniform u32; optionally sorted by (key, val)."""
    k = uniform_int(seed_col(cfg, rel, 0), start, n, 0, key_space - 1, device)
    v = u32(seed_col(cfg, rel, 1), start, n, device)
    if sort:
        k, v = sort_by_key_val(k, v)
    return {"key": to_u32_storage(k), "val": to_u32_storage(v)}


def setop_relation(cfg: int, rel: int, n: int, key_space: int, nval: int, device="cpu",
                   start: int = 0) -> Dict[str, torch.Tensor]:
    """Set-operator input: rows [start, start + n) of a relation with
    key uniform in [0, key_space), val uniform in [0, nval) (small, so whole tuples
    repeat across relations), sorted by (key, val)."""
    k = uniform_int(seed_col(cfg, rel, 0), start, n, 0, key_space - 1, device)
    v = uniform_int(seed_col(cfg, rel, 1), start, n, 0, nval - 1, device)
    k, v = sort_by_key_val(k, v)
    return {"key": to_u32_storage(k), "val": to_u32_storage(v)}


# TPC-H-like lineitem (TPC-H spec §4.2.3 distributions [ext]).
# Dates are int32 days since 1970-01-01.
D_1992_01_01 = 8035
D_1998_08_02 = 10440
D_1995_06_17 = 9298
D_1998_09_02 = 10471   # Q1 cutoff: 1998-12-01 - 90 days


def lineitem(cfg: int, start: int, n: int, sf_parts: int = 200000 * 100,
             device="cpu") -> Dict[str, torch.Tensor]:
    """Columns: shipdate i32; qty, price, disc, tax i64 (DECIMAL(15,2) as cents);
    rf, ls u8 codes (rf: A=0, N=1, R=2; ls: F=0, O=1).  38 bytes/row."""
    def col(c):
        return seed_col(cfg, 0, c)

    def gen(s, m):
        o = start + s
        orderdate = uniform_int(col(0), o, m, D_1992_01_01, D_1998_08_02, device)
        shipdate = orderdate + uniform_int(col(1), o, m, 1, 121, device)
        receipt = shipdate + uniform_int(col(2), o, m, 1, 30, device)
        qty = uniform_int(col(3), o, m, 1, 50, device)
        partkey = uniform_int(col(4), o, m, 1, sf_parts, device)
        retail = 90000 + torch.remainder(partkey // 10, 20001) + 100 * torch.remainder(partkey, 1000)
        price = qty * retail                       # cents; qty is a whole number
        disc = uniform_int(col(5), o, m, 0, 10, device)
        tax = uniform_int(col(6), o, m, 0, 8, device)
        ra = uniform_int(col(7), o, m, 0, 1, device)   # R or A when received
        rf = torch.where(receipt <= D_1995_06_17, torch.where(ra == 0, 2, 0), torch.ones_like(ra))
        ls = (shipdate > D_1995_06_17).to(torch.int64)
        return torch.stack([shipdate, qty * 100, price, disc, tax, rf, ls])

    a = _chunked(gen, n, device, chunk=1 << 24, dim=1)
    return {
        "shipdate": a[0].to(torch.int32),
        "qty": a[1].contiguous(),
        "price": a[2].contiguous(),
        "disc": a[3].contiguous(),
        "tax": a[4].contiguous(),
        "rf": a[5].to(torch.uint8),
        "ls": a[6].to(torch.uint8),
    }
