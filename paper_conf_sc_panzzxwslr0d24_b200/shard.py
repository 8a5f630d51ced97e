"""Table-wise sharding across GPUs (§VII: "place different
embedding tables on multiple GPUs through heuristics ... and then use RecFlex to
optimize the embedding operations on each GPU") with the pooled-output
exchange TorchRec-style table-wise sharding needs.

  * partition: greedy LPT over features, largest first, to the least loaded
    rank (ties: lower feature id first, lower rank), by estimated device time
    (`feature_time`: distinct-row DRAM fetches at the random-access rate + L2
    re-hits + bytes at HBM rate; reading C24') or by bytes per batch
    (`feature_cost`, reading C24: E[L]*cov*(4d+4)*B + 4*d*B).
  * each rank runs its own fused RecFlex plan over ALL B samples of its
    features -> out_r [B][D_r] (row-major, so rank j's B/W-sample block is
    contiguous: no pre-permutation before the all-to-all);
  * alltoallv over NCCL: rank r sends block j (B/W x D_r) to rank j and
    receives B/W x D_i from every rank i;
  * relayout [W][B/W][D_i] -> [B/W][D_tot'] with the library's CUDA kernel
    (recflex_shard_concat).  Columns are grouped by rank (rank 0's features
    first, in their global order), i.e. a fixed permutation of the 1-GPU
    layout given by `column_order()`.
"""
from __future__ import annotations

from typing import List, Sequence

import numpy as np


def _nullcontext():
    import contextlib
    return contextlib.nullcontext()


def row_bytes(dim: int, dtype: str = 'f32') -> int:
    """Bytes one lookup gathers: the stored row (int8: codes + scale + bias)."""
    return {'f32': 4 * dim, 'f16': 2 * dim, 'bf16': 2 * dim, 'i8': dim + 8, 'fp8': dim}[dtype]


def feature_cost(feat, B: int, dtype: str = 'f32') -> float:
    """Estimated bytes per batch (reading C24): lookups x (row + ID) + pooled output."""
    el = feat.mean_len() * feat.coverage
    return el * (row_bytes(feat.dim, dtype) + 4) * B + 4.0 * feat.dim * B


# Device-time model for the partitioner (reading C24'): random row
# fetches are limited by the access rate (~40 G random accesses/s on B200 for
# rows <= 128 B, tools/gather_probe.cu), a repeated row of the batch hits L2 at
# a fraction of that cost, bytes move at HBM bandwidth, and every bag (feature,
# sample) has a fixed cost (offsets, output row, claim).  Coefficients: least
# squares over 28 measured per-rank times of sharded1000 at W = 1, 2, 4, 8
# (tools/rank_sim.py, profiles/r01_rank_sim_sharded1000_*.jsonl; rms error 4 %).
ACCESS_RATE = 44e9
HBM_BPS = 8.4e12
L2_HIT_COST = 0.33
BAG_SECONDS = 4.4e-11


def feature_time(feat, B: int, dtype: str = 'f32') -> float:
    """Estimated seconds per batch: DRAM row fetches (distinct rows of the batch,
    uniform IDs) + L2 re-hits at the access rate, plus DRAM bytes at HBM rate."""
    import math
    nnz = feat.mean_len() * feat.coverage * B
    R = float(feat.rows)
    distinct = R * (1.0 - math.exp(-nnz / R)) if R > 0 else 0.0
    rb = row_bytes(feat.dim, dtype)
    gran = max(32, (rb + 31) // 32 * 32)  # 32-byte sectors
    return ((distinct + (nnz - distinct) * L2_HIT_COST) / ACCESS_RATE
            + (distinct * gran + 4.0 * nnz + 4.0 * feat.dim * B) / HBM_BPS + BAG_SECONDS * B)


def lpt_partition(costs: Sequence[float], W: int) -> List[List[int]]:
    """Greedy longest-processing-time partition; each part sorted by feature id."""
    if W <= 0:
        raise ValueError('W must be positive')
    order = sorted(range(len(costs)), key=lambda f: (-float(costs[f]), f))
    load = [0.0] * W
    parts: List[List[int]] = [[] for _ in range(W)]
    for f in order:
        r = min(range(W), key=lambda i: (load[i], i))
        parts[r].append(f)
        load[r] += float(costs[f])
    return [sorted(p) for p in parts]


def partition_model(model, W: int, dtype: str = 'f32', cost: str = 'time') -> List[List[int]]:
    """LPT over features by estimated device time ('time', default) or bytes ('bytes', reading C24)."""
    fn = feature_time if cost == 'time' else feature_cost
    return lpt_partition([fn(f, model.batch, dtype) for f in model.features], W)


def check_parts(parts: List[List[int]], F: int, W: int) -> List[List[int]]:
    """A table-wise partition must cover every feature exactly once, W non-empty parts."""
    if len(parts) != W or any(len(p) == 0 for p in parts):
        raise ValueError(f'partition needs {W} non-empty parts')
    flat = sorted(f for p in parts for f in p)
    if flat != list(range(F)):
        raise ValueError('partition does not cover every feature exactly once')
    return [sorted(int(f) for f in p) for p in parts]


def refine_partition(parts: List[List[int]], measure, est: Sequence[float], moves: int = 8, tries: int = 6):
    """Measured refinement of a partition (tools/rebalance.py).

    `measure(parts, r)` returns rank r's measured time under `parts`; `est[f]` is the
    modelled cost of feature f.  Repeatedly: a = slowest rank, b = fastest; try moving
    one feature of a to b (candidates ordered by |est[f] * t_a / est(a) - gap/2|); accept
    the first whose two new rank times are both below t_a.  Stops after `moves`
    accepted moves or when no candidate helps.  Returns (parts, times, log); a candidate
    whose measurement raises (e.g. a schedule invalid at the new column) is skipped."""
    F = sum(len(p) for p in parts)
    W = len(parts)
    parts = check_parts(parts, F, W)
    t = [float(measure(parts, r)) for r in range(W)]
    log = [dict(step='start', ms=list(t), max=max(t), max_over_mean=max(t) * W / sum(t))]
    for _ in range(moves):
        ra = max(range(W), key=lambda r: (t[r], -r))
        rb = min(range(W), key=lambda r: (t[r], r))
        if ra == rb or len(parts[ra]) < 2:
            break
        gap = 0.5 * (t[ra] - t[rb])
        scale = t[ra] / max(sum(est[f] for f in parts[ra]), 1e-30)
        cands = sorted(parts[ra], key=lambda f: (abs(est[f] * scale - gap), f))[:tries]
        accepted = None
        for f in cands:
            trial = [list(p) for p in parts]
            trial[ra].remove(f)
            trial[rb].append(f)
            trial = check_parts(trial, F, W)
            try:
                ta, tb = float(measure(trial, ra)), float(measure(trial, rb))
            except Exception as ex:  # noqa: BLE001 -- reported in the log, candidate skipped
                log.append(dict(step='skip', feature=f, why=str(ex)[:120]))
                continue
            log.append(dict(step='try', feature=f, src=ra, dst=rb, ta=ta, tb=tb, old_max=t[ra]))
            if max(ta, tb) < t[ra]:
                accepted = (f, trial, ta, tb)
                break
        if accepted is None:
            break
        f, parts, t[ra], t[rb] = accepted
        log.append(dict(step='move', feature=f, src=ra, dst=rb, ms=list(t), max=max(t),
                        max_over_mean=max(t) * W / sum(t)))
    return parts, t, log


def model_parts(model, W: int, dtype: str = 'f32', config: str = '', tuned_dir: str = '') -> List[List[int]]:
    """The partition a run uses: the measured refinement `<tuned_dir>/<config>[_<dtype>]_w<W>_parts.json`
    (written by tools/rebalance.py together with the per-rank plans it retuned) if present,
    else the model LPT (`partition_model`)."""
    import json
    import os
    if config and tuned_dir and W > 1:
        name = f'{config}_w{W}_parts.json' if dtype == 'f32' else f'{config}_{dtype}_w{W}_parts.json'
        path = os.path.join(tuned_dir, name)
        if os.path.exists(path):
            with open(path) as fh:
                return check_parts(json.load(fh)['parts'], len(model.features), W)
    return partition_model(model, W, dtype)


def column_order(model, parts: List[List[int]]) -> np.ndarray:
    """Global column index of every column of the exchanged [B/W][D_tot'] output.

    parts[r] lists rank r's features in its LOCAL column order: the partition's
    order for plans with feature-order columns, ShardedEmbedding.column_features
    for a rank plan whose outputs follow its task order (recflex_set_column_order)."""
    col = np.cumsum([0] + model.dims)
    order = []
    for part in parts:
        for f in part:
            order.extend(range(col[f], col[f + 1]))
    return np.asarray(order, np.int64)


def shard_batch(batch, features: Sequence[int]):
    """KJT restricted to `features` (feature-major, rebased): indices, offsets."""
    B = batch.B
    offs = batch.offsets.astype(np.int64)
    idx_parts, off_parts = [], []
    pos = 0
    for f in features:
        a, b = offs[f * B], offs[(f + 1) * B]
        idx_parts.append(batch.indices[a:b])
        off_parts.append(offs[f * B:(f + 1) * B] - a + pos)
        pos += b - a
    off_parts.append(np.asarray([pos], np.int64))
    idx = np.concatenate(idx_parts) if idx_parts else np.zeros(0, np.int32)
    return idx.astype(np.int32), np.concatenate(off_parts).astype(np.int32)


def sample_slice(batch, j: int, W: int):
    """Data-parallel slice of a global KJT: all features, samples [j*B/W, (j+1)*B/W) (rebased)."""
    B, F = batch.B, batch.F
    if B % W:
        raise ValueError('B % W != 0')
    Bl = B // W
    offs = batch.offsets.astype(np.int64)
    lens = np.diff(offs).reshape(F, B)[:, j * Bl:(j + 1) * Bl]
    idx = np.concatenate([batch.indices[offs[f * B + j * Bl]:offs[f * B + (j + 1) * Bl]] for f in range(F)])
    off = np.concatenate([[0], np.cumsum(lens.reshape(-1))])
    return idx.astype(np.int32), off.astype(np.int32)


def split_sizes(B: int, W: int, dims_per_rank: Sequence[int], rank: int):
    """alltoallv element counts for rank `rank`: (input_splits, output_splits)."""
    if B % W:
        raise ValueError('table-wise exchange needs B % W == 0 (reading C23)')
    rows = B // W
    inp = [rows * dims_per_rank[rank]] * W
    out = [rows * d for d in dims_per_rank]
    return inp, out


def alltoallv(send, input_splits: Sequence[int], output_splits: Sequence[int], group=None):
    """all_to_all_single with element split sizes; returns the received flat tensor."""
    import torch
    import torch.distributed as dist
    inp, out = [int(x) for x in input_splits], [int(x) for x in output_splits]
    recv = torch.empty(sum(out), dtype=send.dtype, device=send.device)
    if send.is_cuda and dist.get_backend(group) == 'gloo':
        # test plumbing only (several ranks sharing one GPU, where NCCL refuses):
        # gloo has no CUDA all-to-all, so the exchange is staged through host memory
        r_cpu = torch.empty(sum(out), dtype=send.dtype)
        dist.all_to_all_single(r_cpu, send.reshape(-1).cpu(), output_split_sizes=out, input_split_sizes=inp,
                               group=group)
        recv.copy_(r_cpu)
        return recv
    dist.all_to_all_single(recv, send.reshape(-1), output_split_sizes=out, input_split_sizes=inp, group=group)
    return recv


def exchange(send, dims_per_rank: Sequence[int], B: int, group=None):
    """Pooled-output alltoallv: send [B][D_r] -> recv [sum_i B/W*D_i] (chunks in rank order)."""
    import torch.distributed as dist
    W = dist.get_world_size(group)
    rank = dist.get_rank(group)
    inp, out = split_sizes(B, W, dims_per_rank, rank)
    return alltoallv(send, inp, out, group)


def feature_owner(parts: List[List[int]], F: int) -> List[int]:
    """owner[f] = the rank whose part holds f (parts must cover 0..F-1 once, each sorted)."""
    owner = [-1] * F
    for r, p in enumerate(parts):
        if list(p) != sorted(p):
            raise ValueError('each part must list its features in ascending order')
        for f in p:
            if not 0 <= f < F or owner[f] != -1:
                raise ValueError(f'feature {f} out of range or owned twice')
            owner[f] = r
    if -1 in owner:
        raise ValueError('every feature needs an owner')
    return owner


def exchange_kjt(send_lengths, send_indices, dest_counts, send_length_counts: Sequence[int],
                 recv_length_counts: Sequence[int], group=None):
    """The collective half of the input distribution (layouts: include/recflex.h
    recflex_kjt_pack / recflex_kjt_unpack): the per-destination ID counts first
    (W ints), one host read of them (the alltoallv split sizes NCCL takes from
    the host), then the lengths (host-known sizes) and the IDs.
    Returns (recv_lengths, recv_indices, recv_counts list)."""
    import torch
    import torch.distributed as dist
    if len(send_length_counts) == 1:  # one rank: the send buffers are the receive buffers
        n = int(dest_counts.reshape(-1)[0].item())
        return send_lengths, send_indices[:n], [n]
    W = dist.get_world_size(group)
    recv_counts = alltoallv(dest_counts, [1] * W, [1] * W, group)
    both = torch.cat([dest_counts.reshape(-1), recv_counts]).cpu().tolist()  # the one host sync
    send_counts, rc = both[:W], both[W:]
    recv_lengths = alltoallv(send_lengths, send_length_counts, recv_length_counts, group)
    recv_indices = alltoallv(send_indices[:sum(send_counts)], send_counts, rc, group)
    return recv_lengths, recv_indices, rc


class KJTInputDist:
    """Table-wise input distribution: data-parallel local
    KJTs (all features, Bl samples per rank) -> each rank's owned features over
    all B = W*Bl samples, ready for its plan's forward.  Device passes in the
    library (recflex_kjt_pack / recflex_kjt_unpack), collective over
    torch.distributed (NCCL on GPUs)."""

    def __init__(self, parts: List[List[int]], F: int, rank: int, world: int, local_batch: int, device: int = 0):
        import torch
        from .plan import KJTDist
        self.parts, self.rank, self.world, self.local_batch = parts, rank, world, local_batch
        self.kd = KJTDist(feature_owner(parts, F), world, rank, local_batch, device)
        dev = torch.device('cuda', device)
        self.dev = dev
        self.send_lengths = torch.empty(F * local_batch, dtype=torch.int32, device=dev)
        self.dest_counts = torch.empty(world, dtype=torch.int32, device=dev)
        self.offsets_out = torch.empty(self.kd.num_owned * world * local_batch + 1, dtype=torch.int32, device=dev)
        self._send_idx = torch.empty(0, dtype=torch.int32, device=dev)

    def forward(self, indices, offsets, group=None, stream=None):
        """Returns (indices, offsets) of the owned features' global-batch KJT."""
        import torch
        if self._send_idx.numel() < indices.numel():
            self._send_idx = torch.empty(indices.numel(), dtype=torch.int32, device=self.dev)
        self.kd.pack(indices, offsets, self.send_lengths, self._send_idx, self.dest_counts, stream=stream)
        # the collectives run on torch's current stream: make it the pack kernel's stream
        with torch.cuda.stream(stream) if stream is not None else _nullcontext():
            torch.cuda.nvtx.range_push('recflex KJT all-to-all')
            rl, ri, rc = exchange_kjt(self.send_lengths, self._send_idx, self.dest_counts,
                                      self.kd.send_length_counts, self.kd.recv_length_counts, group)
            torch.cuda.nvtx.range_pop()
        idx_out = torch.empty(sum(rc), dtype=torch.int32, device=self.dev)
        self.kd.unpack(rl, ri, idx_out, self.offsets_out, stream=stream)
        return idx_out, self.offsets_out

    def close(self):
        self.kd.close()


class ShardedEmbedding:
    """One rank's slice of a table-wise sharded model: plan + exchange + relayout."""

    def __init__(self, model, rank: int, world: int, device: int = 0, parts=None, dtype: str = 'f32'):
        from .plan import Plan
        self.model = model
        self.rank, self.world = rank, world
        self.parts = parts if parts is not None else partition_model(model, world, dtype)
        self.features = self.parts[rank]
        self.dims_per_rank = [sum(model.dims[f] for f in p) for p in self.parts]
        specs = [dict(rows=model.features[f].rows, dim=model.features[f].dim, pool=model.features[f].pool,
                      mean_len=model.features[f].mean_len(), max_len=model.features[f].max_len(),
                      coverage=model.features[f].coverage, dtype=dtype) for f in self.features]
        self.plan = Plan(specs, model.batch, device)
        self.d_local = self.dims_per_rank[rank]
        self.d_tot = sum(self.dims_per_rank)

    @property
    def column_features(self) -> List[int]:
        """This rank's (global) features in the order of their local output columns."""
        cols = self.plan.columns
        return [self.features[i] for i in sorted(range(len(self.features)), key=lambda i: cols[i])]

    def forward(self, indices, offsets, B, tables, out_local=None, out=None, group=None, stream=None):
        import torch
        from .plan import shard_concat
        out_local = self.plan.forward(indices, offsets, B, tables, out=out_local, stream=stream)
        if self.world == 1:
            return out_local
        # the collective runs on torch's current stream: make it the kernel's stream
        with torch.cuda.stream(stream) if stream is not None else _nullcontext():
            torch.cuda.nvtx.range_push('recflex pooled-output all-to-all')
            recv = exchange(out_local, self.dims_per_rank, B, group)
            torch.cuda.nvtx.range_pop()
        rows = B // self.world
        if out is None:
            out = torch.empty((rows, self.d_tot), dtype=torch.float32, device=out_local.device)
        shard_concat(recv, self.dims_per_rank, rows, out, stream=stream)
        return out


class FusedShardedEmbedding(ShardedEmbedding):
    """Table-wise sharding with the pooled-output all-to-all FUSED into the
    fused kernel's store epilogue: every rank's kernel writes
    each pooled row straight into the owning rank's final [B/W][D_tot] buffer
    through CUDA-IPC-mapped peer pointers (NVLink peer stores across GPUs of a
    node; plain stores when ranks share a device), so there is no separate
    all-to-all pass and no relayout (recflex_forward_exchange).

    Per step there is no host or collective barrier: the destinations are
    double-buffered (step n writes buffer n & 1 of every rank), the kernel's
    last CTA publishes the step into every destination's flag array with a
    system-scope release, and a one-warp wait kernel on this rank's stream
    acquires all W flags before anything enqueued later runs.  The tensor
    forward() returns is valid for work enqueued on the same stream before the
    next-but-one forward() (include/recflex.h documents why); copy it to keep it
    longer.  Setup (IPC handle exchange) uses the process group once."""

    def __init__(self, model, rank: int, world: int, device: int = 0, parts=None, group=None, dtype: str = 'f32'):
        import torch
        import torch.distributed as dist
        from .plan import DeviceBuffer, ipc_handle, ipc_open
        super().__init__(model, rank, world, device, parts, dtype)
        if model.batch % world:
            raise ValueError('fused exchange needs B % W == 0 (reading C23)')
        self.group = group
        self.rows = model.batch // world
        self.col_base = sum(self.dims_per_rank[:rank])
        self.bufs = [DeviceBuffer(self.rows, self.d_tot, device) for _ in range(2)]
        self.flags = DeviceBuffer(1, world, device)  # W uint32 (4-byte cells), zeroed below
        self.flags.tensor.zero_()
        torch.cuda.synchronize(device)
        mine = (rank, [ipc_handle(b) for b in self.bufs], ipc_handle(self.flags))
        handles = [None] * world
        dist.all_gather_object(handles, mine, group=group)
        self.dst = [[0] * world, [0] * world]
        self.flag_ptrs = [0] * world
        self._opened = []
        for r, bh, fh in handles:
            if r == rank:
                for b in range(2):
                    self.dst[b][r] = self.bufs[b].ptr.value
                self.flag_ptrs[r] = self.flags.ptr.value
                continue
            for b in range(2):
                p = ipc_open(bh[b])
                self.dst[b][r] = p
                self._opened.append(p)
            p = ipc_open(fh)
            self.flag_ptrs[r] = p
            self._opened.append(p)
        dist.barrier(group=group)  # every rank's flags are zero before anyone's first step

    def forward(self, indices, offsets, B, tables, out_local=None, out=None, group=None, stream=None):
        if B != self.model.batch:
            raise ValueError('the fused exchange buffers are sized for the model batch')
        b = self.plan.forward_exchange(indices, offsets, B, tables, self.world, self.rank, self.rows, self.d_tot,
                                       self.col_base, self.dst[0], self.dst[1], self.flag_ptrs, self.flags.ptr.value,
                                       stream=stream)
        return self.bufs[b].tensor

    def close(self):
        from .plan import ipc_close
        for p in self._opened:
            ipc_close(p)
        self._opened = []
        for b in self.bufs:
            b.close()
        self.flags.close()
