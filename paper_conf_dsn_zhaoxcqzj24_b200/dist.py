"""Multi-GPU plumbing of the hot path: one process per GPU, torch.distributed
for the collectives (NCCL over NVLink on GPUs; the host-side logic is also exercised with gloo on CPU).

The path shards by run (runs are independent up to integer sums) and has one exchange step:

1. ``shard``: contiguous blocks of the ascending run list (runs alternate FIX / RND, so every rank holds
   both classes).
2. ``agree_slots``: every rank all-gathers the runs' kernel-id sequences and registers the runs it does not
   hold (``owl_register_remote_runs``), so the Myers slot assignment (A4) sees every run of a
   class in global order and slot ids agree everywhere.
3. Each rank folds its runs into partial evidences (``Context.build`` over all runs of the class: remote
   runs shape the slot table, local runs are folded).
4. ``owner_evidence``: ``owl_partition_evidence`` packs every cell by owner(attr) = mix64(attr) mod world,
   ``all_to_all_single`` moves the counts and then the cells, ``owl_absorb_evidence`` sums what arrived:
   each KS attribute now lives whole on one rank (integer sums: bit-identical to one GPU).
5. ``leak_test`` / ``diff``: each owner tests / diffs its attributes; rows are all-gathered and merged by the
   library (``owl_merge_leaks`` / ``owl_merge_diffs``) into exactly the one-GPU result.

Only argument marshalling happens here: every step on the data runs in libowl's kernels.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist


def shard(runs, world: int, rank: int) -> list:
    """Rank `rank`'s contiguous block of the ascending runs (sizes differ by at most one)."""
    runs = sorted(runs)
    q, r = divmod(len(runs), world)
    lo = rank * q + min(rank, r)
    return runs[lo: lo + q + (1 if rank < r else 0)]


def gather_sequences(local_meta: dict, group=None) -> dict:
    """local_meta: {run: (input_class, [kernel_id of each invocation in seq order])} -> the union over ranks."""
    parts = [None] * dist.get_world_size(group)
    dist.all_gather_object(parts, local_meta, group=group)
    merged = {}
    for p in parts:
        merged.update(p)
    return merged


def agree_slots(ctx, all_meta: dict, local_runs) -> None:
    """Registers every run this rank does not hold, so slot ids agree across ranks."""
    local = set(local_runs)
    remote = [r for r in sorted(all_meta) if r not in local]
    if remote:
        ctx.register_remote_runs(remote, [all_meta[r][0] for r in remote], [list(all_meta[r][1]) for r in remote])


def exchange_bytes(send: torch.Tensor, send_counts, group=None):
    """all_to_all of byte buckets: send[sum(send_counts[:k]) : +send_counts[k]] goes to rank k.  Returns the
    received bytes (rank 0's bucket first) and their sizes."""
    dev = send.device
    if send.is_cuda and dist.get_backend(group) == "gloo":  # gloo has no CUDA all-to-all (tests only)
        recv, rc = exchange_bytes(send.cpu(), send_counts, group)
        return recv.to(dev), rc
    sc = torch.tensor([int(c) for c in send_counts], dtype=torch.int64, device=dev)
    rc = torch.empty_like(sc)
    dist.all_to_all_single(rc, sc, group=group)
    recv_counts = [int(c) for c in rc.tolist()]
    recv = torch.empty(sum(recv_counts), dtype=torch.uint8, device=dev)
    dist.all_to_all_single(recv, send, output_split_sizes=recv_counts, input_split_sizes=[int(c) for c in send_counts],
                           group=group)
    return recv, recv_counts


class _DeviceBytes:
    """__cuda_array_interface__ view of a device buffer owned by libowl (no copy)."""

    def __init__(self, ptr: int, nbytes: int):
        self.__cuda_array_interface__ = {"shape": (nbytes,), "typestr": "|u1", "data": (ptr, False), "version": 2}


def owner_evidence(ctx, partial, world: int, rank: int, group=None):
    """The exchange (step 4): this rank's partial evidence -> the evidence of the attributes it owns."""
    ptr, sb = partial.partition(world)
    dev = torch.device("cuda", ctx.device)
    total = int(sum(sb))
    send = torch.as_tensor(_DeviceBytes(ptr, total), device=dev) if total else torch.empty(0, dtype=torch.uint8, device=dev)
    recv, rc = exchange_bytes(send, list(sb), group)
    return ctx.absorb(partial, recv.data_ptr() if recv.numel() else None, rc, rank), recv


def gather_rows(rows: np.ndarray, group=None) -> np.ndarray:
    parts = [None] * dist.get_world_size(group)
    dist.all_gather_object(parts, np.ascontiguousarray(rows), group=group)
    parts = [p for p in parts if p is not None and len(p)]
    return np.concatenate(parts) if parts else rows[:0].copy()


def leak_test(ctx, owned_f, owned_r, significance: float, group=None) -> np.ndarray:
    """Each owner tests its attributes; the rows are all-gathered and merged by the library
    (owl_merge_leaks: kernel rows from the replicated slot tables, CF / DF rows by alignment position, a DF
    location split across owners keeps its min-p visit, ties -> smallest j)."""
    parts = [None] * dist.get_world_size(group)
    dist.all_gather_object(parts, ctx.leak_test(owned_f, owned_r, significance), group=group)
    return ctx.merge_leaks(owned_f, owned_r, parts)


def diff(ctx, owned_a, owned_b, group=None) -> np.ndarray:
    """Each owner diffs its cells; rows all-gathered, merged into canonical order by owl_merge_diffs."""
    parts = [None] * dist.get_world_size(group)
    dist.all_gather_object(parts, ctx.diff(owned_a, owned_b), group=group)
    return ctx.merge_diffs(owned_a, owned_b, parts)
