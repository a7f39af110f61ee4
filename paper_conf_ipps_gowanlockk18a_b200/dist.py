"""Multi-GPU pieces of the path (one process per GPU, torch.distributed for the plumbing).

* ``shard_range`` / ``max_over_ranks``: the sort phase shards into independent batches
  (n_b/(n_s n_GPU) batches per stream), so ranks need no data-path
  collective; timing is the max over ranks.
* ``exchange_sorted_runs`` (the paper's NVLink-era direction P:1105-1115):
  after every rank has sorted its own shard, a splitter-based all-to-all leaves rank r with the
  r-th key range of the global order, which the library's k-way merge (K4/K5 on the GPU, H2 on
  the CPU) turns into rank r's slice of B.  The splitters come from regular samples of the
  sorted runs (positions and quantiles computed by the library: hsort_sample_positions,
  hsort_select_splitters), merged with the library's multiway merge; the partition uses the library's
  upper-bound kernel; the transfer is one ``all_to_all_single`` (NCCL over NVLink on GPUs, gloo
  on CPU in the tests).  Concatenating the ranks' results in rank order gives the global sort.

Keys are the order-preserving uint64 keys of the float64 values (the same map the kernels use);
they cross the wire as int64 bit patterns.
"""
from __future__ import annotations

import numpy as np
import torch
import torch.distributed as dist

from . import (hsort_device_merge, hsort_device_upper_bounds, hsort_host_merge,
               hsort_host_upper_bounds, hsort_sample_positions, hsort_select_splitters)


def shard_range(n: int, world: int, rank: int) -> tuple[int, int]:
    """[lo, hi) of rank's contiguous shard of n keys (sizes differ by at most one)."""
    q, r = divmod(n, world)
    lo = rank * q + min(rank, r)
    return lo, lo + q + (1 if rank < r else 0)


def max_over_ranks(x: float, group=None, device=None) -> float:
    if not dist.is_available() or not dist.is_initialized() or dist.get_world_size(group) == 1:
        return float(x)
    t = torch.tensor([float(x)], dtype=torch.float64, device=device)
    dist.all_reduce(t, op=dist.ReduceOp.MAX, group=group)
    return float(t.item())


def _as_i64(t: torch.Tensor) -> torch.Tensor:
    return t.view(torch.int64) if t.dtype == torch.uint64 else t


def choose_splitters(local_sorted: torch.Tensor, group=None, oversample: int = 64) -> np.ndarray:
    """P-1 global splitters (uint64 keys) from ``oversample * P`` regular samples per rank."""
    P = dist.get_world_size(group)
    dev = local_sorted.device
    n = local_sorted.numel()
    s = oversample * P
    if n:
        pos = torch.from_numpy(hsort_sample_positions(n, s).view(np.int64)).to(dev)
        samp = _as_i64(local_sorted)[pos]
    else:
        samp = torch.zeros(s, dtype=torch.int64, device=dev)
    cnt = torch.tensor([s if n else 0], dtype=torch.int64, device=dev)
    all_samp = [torch.empty_like(samp) for _ in range(P)]
    all_cnt = [torch.empty_like(cnt) for _ in range(P)]
    dist.all_gather(all_samp, samp, group=group)
    dist.all_gather(all_cnt, cnt, group=group)
    runs = [a.cpu().numpy().view(np.uint64)[: int(c.item())] for a, c in zip(all_samp, all_cnt)]
    runs = [r for r in runs if r.size]
    if not runs:
        return np.zeros(P - 1, dtype=np.uint64)
    off = np.cumsum([0] + [r.size for r in runs]).astype(np.uint64)
    merged = hsort_host_merge(np.concatenate(runs), off)  # sorted samples (library merge)
    return hsort_select_splitters(merged, P)  # the P-quantiles (library arithmetic)


def exchange_sorted_runs(local_sorted: torch.Tensor, group=None, oversample: int = 64,
                         out_f64: bool = False) -> torch.Tensor:
    """Globally redistribute per-rank sorted uint64 key runs and merge them.

    Returns rank r's slice of the global sort: every key k with s_r < k <= s_{r+1} (splitters
    s_0 = -inf, s_P = +inf), sorted; as uint64 keys, or float64 values if ``out_f64``.
    Equal keys never straddle ranks, so the slices concatenate to the unique global order.
    """
    P = dist.get_world_size(group)
    dev = local_sorted.device
    keys = local_sorted.contiguous()
    n = keys.numel()
    if P == 1:
        parts, sizes = [keys], [n]
    else:
        spl = choose_splitters(keys, group, oversample)
        if dev.type == "cuda":
            d_spl = torch.from_numpy(spl).to(dev)
            ub = torch.empty(P - 1, dtype=torch.uint64, device=dev)
            hsort_device_upper_bounds(keys, d_spl, ub)
            cuts = [0] + [int(v) for v in ub.cpu().numpy()] + [n]
        else:
            ub = hsort_host_upper_bounds(keys.numpy(), spl)
            cuts = [0] + [int(v) for v in ub] + [n]
        send = [cuts[r + 1] - cuts[r] for r in range(P)]
        send_t = torch.tensor(send, dtype=torch.int64, device=dev)
        recv_t = torch.empty_like(send_t)
        dist.all_to_all_single(recv_t, send_t, group=group)
        sizes = [int(v) for v in recv_t.cpu()]
        recv = torch.empty(sum(sizes), dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv, _as_i64(keys), output_split_sizes=sizes,
                               input_split_sizes=send, group=group)
        parts = [recv]
    data = parts[0].view(torch.uint64) if parts[0].dtype == torch.int64 else parts[0]
    off = np.cumsum([0] + sizes).astype(np.uint64)
    total = int(off[-1])
    if total == 0:
        return torch.empty(0, dtype=torch.float64 if out_f64 else torch.uint64, device=dev)
    if dev.type == "cuda":
        out = torch.empty(total, dtype=torch.uint64, device=dev)
        hsort_device_merge(data, off, out, out_f64)
        return out.view(torch.float64) if out_f64 else out
    merged = hsort_host_merge(data.numpy(), off, out_f64=out_f64)
    return torch.from_numpy(merged)
