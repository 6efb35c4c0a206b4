"""Chunk-sharded multi-GPU compression (not in the paper).

The paper is single-device.  Its chunks are independent, so an
array shards by chunk with no data exchange: rank r of P owns chunks
[floor(r*C/P), floor((r+1)*C/P)).  The method has exactly two exchange steps,
both tiny and latency-bound, done with torch.distributed (NCCL over NVLink on
the GPU box, gloo in the CPU tests):

  (1) NOA only, before quantizing: all-reduce MAX of [max, -min]
      so every rank derives the same global bound;
  (2) after the local encode: all-gather of the per-shard payload byte counts,
      whose exclusive prefix gives each shard's offset in the single stream
      (the cross-device analogue of the look-back concatenation).

The assembled stream  header | table_0 | ... | table_{P-1} | payload_0 | ...
is byte-identical to the single-device stream.  The per-shard work runs in the
CUDA kernels behind pfpl_minmax / pfpl_compress_shard; this module only
plans, exchanges the two small vectors and computes offsets.
"""
from __future__ import annotations

from dataclasses import dataclass

import torch
import torch.distributed as dist

CHUNK_BYTES = 16384
HEADER_BYTES = 48


def chunks_of(n: int, itemsize: int) -> int:
    cw = CHUNK_BYTES // itemsize
    return (n + cw - 1) // cw


def shard_chunks(n_total: int, itemsize: int, rank: int, world: int):
    """(first_chunk, n_chunks, e0, e1): chunk-aligned element range of `rank`."""
    cw = CHUNK_BYTES // itemsize
    C = chunks_of(n_total, itemsize)
    c0, c1 = rank * C // world, (rank + 1) * C // world
    return c0, c1 - c0, min(c0 * cw, n_total), min(c1 * cw, n_total)


@dataclass
class ShardResult:
    header: bytes          # 48-byte global header (identical on every rank)
    table: torch.Tensor    # u32 sizes of this rank's chunks (as uint8 view)
    payload: torch.Tensor  # this rank's concatenated chunk payloads (uint8)
    sizes: list            # payload bytes of every rank
    first_chunk: int
    table_offset: int      # byte offset of this rank's table slice in the stream
    payload_offset: int    # byte offset of this rank's payload in the stream
    total_bytes: int       # size of the assembled stream


def global_minmax(local_mnmx: torch.Tensor, group=None) -> torch.Tensor:
    """Exchange (1): all-reduce MAX of [max, -min] (float64, 2 values)."""
    v = torch.stack([local_mnmx[1], -local_mnmx[0]]).to(torch.float64)
    if dist.is_initialized() and dist.get_world_size(group) > 1:
        dist.all_reduce(v, op=dist.ReduceOp.MAX, group=group)
    return torch.stack([-v[1], v[0]])


def gather_sizes(payload_bytes: int, device, group=None) -> list:
    """Exchange (2): all-gather of the per-shard payload byte counts."""
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    if world == 1:
        return [int(payload_bytes)]
    mine = torch.tensor([payload_bytes], dtype=torch.int64, device=device)
    out = [torch.empty(1, dtype=torch.int64, device=device) for _ in range(world)]
    dist.all_gather(out, mine, group=group)
    return [int(v.item()) for v in out]


def plan_offsets(sizes: list, n_total: int, itemsize: int, world: int, rank: int):
    """Byte offsets of this rank's table slice and payload in the stream."""
    C = chunks_of(n_total, itemsize)
    c0 = rank * C // world
    table_off = HEADER_BYTES + 4 * c0
    payload_off = HEADER_BYTES + 4 * C + sum(sizes[:rank])
    total = HEADER_BYTES + 4 * C + sum(sizes)
    return table_off, payload_off, total


def compress_sharded(x_local: torch.Tensor, n_total: int, bound="abs", eps: float = 1e-3,
                     ms: bool = False, group=None, minmax_fn=None, shard_fn=None) -> ShardResult:
    """Compress this rank's chunk-aligned shard of a global array.

    minmax_fn / shard_fn default to the CUDA library (pfpl_minmax,
    pfpl_compress_shard); tests inject CPU stand-ins to exercise the exchange
    logic with gloo.
    """
    if minmax_fn is None or shard_fn is None:
        from . import compress_shard, minmax
        minmax_fn = minmax_fn or minmax
        shard_fn = shard_fn or (lambda x, fc, nt, b, e, m, mm: compress_shard(x, fc, nt, b, e, m, mm))
    world = dist.get_world_size(group) if dist.is_initialized() else 1
    rank = dist.get_rank(group) if dist.is_initialized() else 0
    itemsize = x_local.element_size()
    first_chunk, nch, e0, e1 = shard_chunks(n_total, itemsize, rank, world)
    if x_local.numel() != e1 - e0:
        raise ValueError(f"rank {rank} holds {x_local.numel()} elements, plan says {e1 - e0}")
    mm = None
    if str(bound).lower() == "noa":
        mm = global_minmax(minmax_fn(x_local), group)
    table, payload, header = shard_fn(x_local, first_chunk, n_total, bound, eps, ms, mm)
    sizes = gather_sizes(payload.numel(), x_local.device, group)
    toff, poff, total = plan_offsets(sizes, n_total, itemsize, world, rank)
    return ShardResult(header, table, payload, sizes, first_chunk, toff, poff, total)


def assemble_on_host(parts: list) -> bytes:
    """Concatenate gathered (header, table bytes, payload bytes) in rank order."""
    hdr = parts[0][0]
    return hdr + b"".join(p[1] for p in parts) + b"".join(p[2] for p in parts)
