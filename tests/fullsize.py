"""Helpers for full-size (BASELINE.json) parity checks: the oracle on a sample
of bags, computed chunk by chunk.

Input selection only -- the pooled values come from oracle.embedding_bag (the C
oracle).  The rows a sampled bag references are read from the TABLE INPUTS,
which the seeded generator (synth.make_table_stored, torch ops) wrote on the
device: a gather of generator output, not a product-kernel result.  (Other
tests pin the same tables through host-side regeneration; reading them back is
what makes >= 1024 sampled rows of the 82 GB heavy tables affordable.)
"""
import numpy as np
import torch

import oracle


def select_bags(batch, f, samples):
    """IDs of bags (f, s) for s in samples, concatenated in sample order, and the bag lengths."""
    B = batch.B
    offs = batch.offsets.astype(np.int64)
    starts = offs[f * B + samples]
    lens = offs[f * B + samples + 1] - starts
    total = int(lens.sum())
    if total == 0:
        return np.zeros(0, np.int32), lens
    first = np.repeat(starts - np.concatenate([[0], np.cumsum(lens)[:-1]]), lens)
    return batch.indices[first + np.arange(total)], lens


def sampled_oracle(model, batch, samples, tables, dtype='f32', chunk=None):
    """fp64 oracle rows [len(samples)][D_tot] and bag lengths [len(samples)][F].

    tables[f]: the feature's stored table on the device (rows gathered per chunk of
    samples; by default chunks hold ~1 GB of gathered rows)."""
    samples = np.asarray(samples, np.int64)
    F = batch.F
    if chunk is None:
        row_b = np.asarray([t.shape[1] * t.element_size() for t in tables], np.float64)
        offs = batch.offsets.astype(np.int64)
        per_f = (offs[np.arange(1, F + 1) * batch.B] - offs[np.arange(F) * batch.B]) / max(1, batch.B)
        per_sample = float((per_f * row_b).sum()) + 1.0
        chunk = int(max(16, min(samples.size, 1e9 / per_sample)))
    outs, lens_all = [], []
    for c0 in range(0, samples.size, chunk):
        sm = samples[c0:c0 + chunk]
        S = sm.size
        tabs, sub_idx, sub_len = [], [], []
        lens = np.zeros((S, F), np.int64)
        for f in range(F):
            ids, ln = select_bags(batch, f, sm)
            lens[:, f] = ln
            uniq, inv = np.unique(ids, return_inverse=True)
            if uniq.size == 0:
                uniq = np.zeros(1, np.int64)
            t = tables[f]
            rows = t[torch.as_tensor(uniq, dtype=torch.int64, device=t.device)].cpu()
            tabs.append(rows if dtype != 'f32' else rows.numpy())
            sub_idx.append(inv.reshape(-1).astype(np.int32))
            sub_len.append(ln)
        idx = np.concatenate(sub_idx)
        off = np.concatenate([[0], np.cumsum(np.concatenate(sub_len))]).astype(np.int32)
        out = oracle.embedding_bag(tabs, model.dims, [ft.pool for ft in model.features], idx, off, S,
                                   dtypes=[dtype] * F)
        outs.append(out)
        lens_all.append(lens)
    return np.concatenate(outs), np.concatenate(lens_all)
