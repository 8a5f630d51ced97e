"""Table-wise sharded forward end to end on one GPU: W ranks (processes) share
cuda:0, each runs its own fused plan over its features, the pooled outputs are
exchanged (gloo, staged through host memory -- NCCL refuses two ranks on one
device) and relayouted by the library's recflex_shard_concat kernel.  The
result must equal the 1-GPU output restricted to the rank's samples, columns
grouped by owning rank, bit for bit on integer-valued tables."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.multiprocessing as mp

pytestmark = pytest.mark.gpu


def _model():
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    feats = []
    dims = [4, 8, 16, 32, 64, 128, 12, 8, 16, 32, 4, 64]
    for i, d in enumerate(dims):
        kind = 'onehot' if i % 2 == 0 else 'lognormal'
        feats.append(synth.Feature(rows=3000 + 17 * i, dim=d, pool=i % 2, kind=kind, coverage=0.8, mu=12.0,
                                   sigma=0.9, lmax=1 if kind == 'onehot' else 120, table=i))
    return synth.custom_model('shardtest', feats, 240)


def _free_port():
    s = socket.socket()
    s.bind(('127.0.0.1', 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.shard import ShardedEmbedding, partition_model, shard_batch
    os.environ['MASTER_ADDR'] = '127.0.0.1'
    os.environ['MASTER_PORT'] = str(port)
    dist.init_process_group('gloo', rank=rank, world_size=world)
    try:
        dev = torch.device('cuda', 0)
        m = _model()
        b = synth.make_batch(m, 5)
        parts = partition_model(m, world)
        sh = ShardedEmbedding(m, rank, world, device=0, parts=parts)
        tables = [synth.make_table(m.features[f].table, m.features[f].rows, m.features[f].dim, 'int', device=dev)
                  for f in sh.features]
        idx, off = shard_batch(b, sh.features)
        out = sh.forward(torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev), b.B, tables)
        torch.cuda.synchronize()
        q.put((rank, out.cpu().numpy(), parts))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize('world', [2, 3])
def test_sharded_forward_matches_single_gpu(world):
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan
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
    b = synth.make_batch(m, 5)
    dev = torch.device('cuda', 0)
    tables = [synth.make_table(f.table, f.rows, f.dim, 'int', device=dev) for f in m.features]
    plan = Plan.from_model(m)
    full = plan.forward(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev), b.B,
                        tables).cpu().numpy()
    rows = b.B // world
    for rank, got, parts in res:
        order = column_order(m, parts)
        assert np.array_equal(got, full[rank * rows:(rank + 1) * rows][:, order])


def _worker_fused(rank, world, port, q):
    import torch.distributed as dist
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.shard import FusedShardedEmbedding, partition_model, shard_batch
    os.environ['MASTER_ADDR'] = '127.0.0.1'
    os.environ['MASTER_PORT'] = str(port)
    dist.init_process_group('gloo', rank=rank, world_size=world)
    try:
        dev = torch.device('cuda', 0)
        m = _model()
        b = synth.make_batch(m, 5)
        parts = partition_model(m, world)
        sh = FusedShardedEmbedding(m, rank, world, device=0, parts=parts)
        tables = [synth.make_table(m.features[f].table, m.features[f].rows, m.features[f].dim, 'int', device=dev)
                  for f in sh.features]
        idx, off = shard_batch(b, sh.features)
        res = []
        for _ in range(2):  # twice: the routed pointer table is cached after the first call
            out = sh.forward(torch.from_numpy(idx).to(dev), torch.from_numpy(off).to(dev), b.B, tables)
            torch.cuda.synchronize()
            res.append(out.cpu().numpy().copy())
            dist.barrier()
        q.put((rank, res, parts))
        dist.barrier()
        sh.close()
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize('world', [2, 3])
def test_fused_exchange_matches_single_gpu(world):
    """NEXT #1: the all-to-all folded into the fused kernel's store epilogue
    (peer stores through CUDA-IPC-mapped buffers)."""
    from paper_conf_sc_panzzxwslr0d24_b200 import synth
    from paper_conf_sc_panzzxwslr0d24_b200.plan import Plan
    from paper_conf_sc_panzzxwslr0d24_b200.shard import column_order
    ctx = mp.get_context('spawn')
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker_fused, args=(r, world, port, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
        assert p.exitcode == 0
    m = _model()
    b = synth.make_batch(m, 5)
    dev = torch.device('cuda', 0)
    tables = [synth.make_table(f.table, f.rows, f.dim, 'int', device=dev) for f in m.features]
    full = Plan.from_model(m).forward(torch.from_numpy(b.indices).to(dev), torch.from_numpy(b.offsets).to(dev), b.B,
                                      tables).cpu().numpy()
    rows = b.B // world
    for rank, outs, parts in res:
        exp = full[rank * rows:(rank + 1) * rows][:, column_order(m, parts)]
        for got in outs:
            assert np.array_equal(got, exp)
