"""Table-wise input distribution on the GPU: the
library's pack / unpack kernels (recflex_kjt_pack / recflex_kjt_unpack through
the C ABI) around an all-to-all, bit-exact against oracle.kjt_input_dist.

W ranks are simulated in one process on cuda:0 (the all-to-all is the slicing
NCCL would do, on the documented layouts), plus a real multi-process run over
gloo feeding the sharded forward."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

import oracle
from paper_conf_sc_panzzxwslr0d24_b200 import synth

pytestmark = pytest.mark.gpu


def _dev():
    return torch.device('cuda', 0)


def _simulate(locs, parts, F, Bl):
    """pack on every rank -> all-to-all by slicing -> unpack on every rank."""
    from paper_conf_sc_panzzxwslr0d24_b200.plan import KJTDist
    from paper_conf_sc_panzzxwslr0d24_b200.shard import feature_owner
    W = len(locs)
    owner = feature_owner(parts, F)
    kds = [KJTDist(owner, W, j, Bl) for j in range(W)]
    sends = []
    for j, (idx, off) in enumerate(locs):
        idx_d, off_d = torch.as_tensor(idx, device=_dev()), torch.as_tensor(off, device=_dev())
        sl = torch.full((F * Bl,), -7, dtype=torch.int32, device=_dev())
        si = torch.full((max(idx.size, 1),), -7, dtype=torch.int32, device=_dev())
        dc = torch.full((W,), -7, dtype=torch.int32, device=_dev())
        kds[j].pack(idx_d, off_d, sl, si, dc)
        sends.append((sl, si, dc.cpu().tolist(), kds[j].send_length_counts))
    out = []
    for r in range(W):
        rl, ri = [], []
        for sl, si, dc, lc in sends:
            a = sum(lc[:r])
            rl.append(sl[a:a + lc[r]])
            a = sum(dc[:r])
            ri.append(si[a:a + dc[r]])
        rl, ri = torch.cat(rl), torch.cat(ri)
        io = torch.full((max(ri.numel(), 1),), -7, dtype=torch.int32, device=_dev())
        oo = torch.full((kds[r].num_owned * W * Bl + 1,), -7, dtype=torch.int32, device=_dev())
        kds[r].unpack(rl, ri, io, oo)
        out.append((io[:ri.numel()].cpu().numpy(), oo.cpu().numpy()))
    torch.cuda.synchronize()
    for kd in kds:
        kd.close()
    return out


def _sample_split(idx, off, F, B, W):
    Bl = B // W
    res = []
    for j in range(W):
        lens = np.diff(off.astype(np.int64)).reshape(F, B)[:, j * Bl:(j + 1) * Bl]
        ids = np.concatenate([idx[off[f * B + j * Bl]:off[f * B + (j + 1) * Bl]] for f in range(F)])
        res.append((ids.astype(np.int32), np.concatenate([[0], np.cumsum(lens.reshape(-1))]).astype(np.int32)))
    return res


@pytest.mark.parametrize('W', [1, 2, 3, 8])
def test_kjt_dist_bitexact_vs_oracle(W):
    m = synth.make_model('medium')
    Bl = 96
    locs = [synth.make_batch(m, 40 + j, B=Bl) for j in range(W)]
    rng = np.random.default_rng(W)
    owner = rng.integers(0, W, m.F)
    if W > 1:
        owner[owner == W - 1] = 0   # the last rank owns nothing
    parts = [[f for f in range(m.F) if owner[f] == r] for r in range(W)]
    got = _simulate([(b.indices, b.offsets) for b in locs], parts, m.F, Bl)
    exp = oracle.kjt_input_dist([(b.indices, b.offsets) for b in locs], parts, Bl)
    for r in range(W):
        assert np.array_equal(got[r][0], exp[r][0]), r
        assert np.array_equal(got[r][1], exp[r][1]), r


def test_kjt_dist_edge_cases():
    """Empty features, all-empty ranks, a feature of 5000 IDs in one bag (several copy chunks), ragged tails."""
    F, W, Bl = 5, 3, 7
    rng = np.random.default_rng(3)
    locs = []
    for j in range(W):
        lens = rng.integers(0, 4, (F, Bl))
        lens[1] = 0                      # feature 1 absent everywhere
        if j == 1:
            lens[:] = 0                  # rank 1 sends nothing
        if j == 2:
            lens[3, 4] = 5000            # one long bag
        off = np.concatenate([[0], np.cumsum(lens.reshape(-1))]).astype(np.int32)
        locs.append((rng.integers(0, 1 << 30, off[-1]).astype(np.int32), off))
    parts = [[0, 3], [1, 2, 4], []]
    got = _simulate(locs, parts, F, Bl)
    exp = oracle.kjt_input_dist(locs, parts, Bl)
    for r in range(W):
        assert np.array_equal(got[r][0], exp[r][0]) and np.array_equal(got[r][1], exp[r][1])


def test_kjt_dist_full_size_sharded1000_w8():
    """BASELINE size (sharded1000, B = 16384, W = 8, LPT parts): the redistributed
    KJTs equal the global batch restricted to each rank's features."""
    from paper_conf_sc_panzzxwslr0d24_b200.shard import partition_model
    m = synth.make_model('sharded1000')
    b = synth.make_batch(m, 7)
    W, B, F = 8, b.B, m.F
    parts = partition_model(m, W)
    got = _simulate(_sample_split(b.indices, b.offsets, F, B, W), parts, F, B // W)
    for r in range(W):
        ids = np.concatenate([b.indices[b.offsets[f * B]:b.offsets[(f + 1) * B]] for f in parts[r]])
        lens = np.concatenate([np.diff(b.offsets[f * B:(f + 1) * B + 1]) for f in parts[r]])
        assert np.array_equal(got[r][0], ids)
        assert np.array_equal(got[r][1], np.concatenate([[0], np.cumsum(lens)]))


def test_kjt_dist_invalid_args():
    from paper_conf_sc_panzzxwslr0d24_b200._lib import RecflexError
    from paper_conf_sc_panzzxwslr0d24_b200.plan import KJTDist
    with pytest.raises(RecflexError):
        KJTDist([0, 2], 2, 0, 4)      # owner out of range
    with pytest.raises(RecflexError):
        KJTDist([0, 1], 2, 2, 4)      # rank out of range


def _free_port():
    s = socket.socket()
    s.bind(('127.0.0.1', 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _model():
    feats = []
    dims = [4, 8, 16, 32, 64, 128, 12, 8, 16, 32, 4, 64]
    for i, d in enumerate(dims):
        kind = 'onehot' if i % 2 == 0 else 'lognormal'
        feats.append(synth.Feature(rows=3000 + 17 * i, dim=d, pool=i % 2, kind=kind, coverage=0.8, mu=12.0,
                                   sigma=0.9, lmax=1 if kind == 'onehot' else 120, table=i))
    return synth.custom_model('kjtdist', feats, 240)


def _worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_sc_panzzxwslr0d24_b200.shard import KJTInputDist, ShardedEmbedding, partition_model
    os.environ['MASTER_ADDR'] = '127.0.0.1'
    os.environ['MASTER_PORT'] = str(port)
    dist.init_process_group('gloo', rank=rank, world_size=world)
    try:
        dev = _dev()
        m = _model()
        Bl = m.batch // world
        loc = synth.make_batch(m, 60 + rank, B=Bl)      # data-parallel input of this rank
        parts = partition_model(m, world)
        ind = KJTInputDist(parts, m.F, rank, world, Bl)
        idx, off = ind.forward(torch.from_numpy(loc.indices).to(dev), torch.from_numpy(loc.offsets).to(dev))
        sh = ShardedEmbedding(m, rank, world, device=0, parts=parts)
        tables = [synth.make_table(m.features[f].table, m.features[f].rows, m.features[f].dim, 'int', device=dev)
                  for f in sh.features]
        out = sh.forward(idx, off, m.batch, tables)
        torch.cuda.synchronize()
        q.put((rank, out.cpu().numpy(), parts))
        ind.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize('world', [2, 3])
def test_input_dist_then_sharded_forward(world):
    """Data-parallel local batches -> input dist -> table-wise forward -> output
    exchange: every rank ends with its own samples x all features, equal (bit
    for bit, integer tables) to the oracle on the concatenated global batch."""
    from paper_conf_sc_panzzxwslr0d24_b200.shard import column_order
    ctx = mp.get_context('spawn')
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    m = _model()
    Bl = m.batch // world
    locs = [synth.make_batch(m, 60 + j, B=Bl) for j in range(world)]
    tabs = [synth.make_table(f.table, f.rows, f.dim, 'int').numpy() for f in m.features]
    for rank, got, parts in res:
        b = locs[rank]
        exp = oracle.embedding_bag(tabs, m.dims, [f.pool for f in m.features], b.indices, b.offsets, Bl)
        assert np.array_equal(got, exp[:, column_order(m, parts)].astype(np.float32))


def test_input_dist_single_rank_is_identity():
    """W = 1 (no process group): pack + unpack reproduce the input KJT."""
    from paper_conf_sc_panzzxwslr0d24_b200.shard import KJTInputDist
    m = synth.make_model('industrial')
    b = synth.make_batch(m, 7, B=512)
    ind = KJTInputDist([list(range(m.F))], m.F, 0, 1, 512)
    idx, off = ind.forward(torch.from_numpy(b.indices).to(_dev()), torch.from_numpy(b.offsets).to(_dev()))
    assert np.array_equal(idx.cpu().numpy(), b.indices) and np.array_equal(off.cpu().numpy(), b.offsets)
    ind.close()
