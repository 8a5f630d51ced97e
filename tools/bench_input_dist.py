"""Device time of the input-distribution passes (recflex_kjt_pack / _unpack) at
BASELINE size: sharded1000, B = 16384, W ranks simulated on one GPU (rank 0's
pack of its local KJT, rank 0's unpack of what every rank sent it).

    python tools/bench_input_dist.py [--world 8] [--iters 20]

Algorithmic bytes: pack reads 2 offsets per (f, s) (4 B each, counted once:
F*Bl*4 + 4) and the local IDs, writes F*Bl lengths and the IDs; unpack reads
W*F_r*Bl lengths (twice: segment sums, then the scan) and the received IDs, writes
F_r*B offsets and the IDs."""
import argparse
import json
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from paper_conf_sc_panzzxwslr0d24_b200 import synth  # noqa: E402
from paper_conf_sc_panzzxwslr0d24_b200.plan import KJTDist, l2_flush  # noqa: E402
from paper_conf_sc_panzzxwslr0d24_b200.shard import feature_owner, partition_model  # noqa: E402


def timeit(fn, iters, flush):
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(iters)]
    for _ in range(3):
        fn()
    for a, b in ev:
        l2_flush(flush)
        a.record()
        fn()
        b.record()
    torch.cuda.synchronize()
    return float(np.median([a.elapsed_time(b) for a, b in ev]))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('--world', type=int, default=8)
    ap.add_argument('--iters', type=int, default=20)
    ap.add_argument('--config', default='sharded1000')
    a = ap.parse_args()
    dev = torch.device('cuda', 0)
    m = synth.make_model(a.config)
    W, B, F = a.world, m.batch, m.F
    Bl = B // W
    parts = partition_model(m, W)
    owner = feature_owner(parts, F)
    locs = [synth.make_batch(m, 7 + j, B=Bl) for j in range(W)]
    flush = torch.empty(512 << 20, dtype=torch.uint8, device=dev)
    kds = [KJTDist(owner, W, j, Bl) for j in range(W)]
    sends = []
    for j, b in enumerate(locs):
        idx = torch.from_numpy(b.indices).to(dev)
        off = torch.from_numpy(b.offsets).to(dev)
        sl = torch.empty(F * Bl, dtype=torch.int32, device=dev)
        si = torch.empty(idx.numel(), dtype=torch.int32, device=dev)
        dc = torch.empty(W, dtype=torch.int32, device=dev)
        kds[j].pack(idx, off, sl, si, dc)
        sends.append((idx, off, sl, si, dc))
    torch.cuda.synchronize()
    idx0, off0, sl0, si0, dc0 = sends[0]
    t_pack = timeit(lambda: kds[0].pack(idx0, off0, sl0, si0, dc0), a.iters, flush)
    pack_bytes = 4 * (F * Bl + 1) + 2 * 4 * idx0.numel() + 4 * F * Bl
    rl, ri = [], []
    for (_, _, sl, si, dc), kd in zip(sends, kds):
        lc, dcl = kd.send_length_counts, dc.cpu().tolist()
        rl.append(sl[sum(lc[:0]):sum(lc[:0]) + lc[0]])
        ri.append(si[:dcl[0]])
    rl, ri = torch.cat(rl), torch.cat(ri)
    Fr = kds[0].num_owned
    io = torch.empty(ri.numel(), dtype=torch.int32, device=dev)
    oo = torch.empty(Fr * B + 1, dtype=torch.int32, device=dev)
    t_unpack = timeit(lambda: kds[0].unpack(rl, ri, io, oo), a.iters, flush)
    unpack_bytes = 2 * 4 * rl.numel() + 2 * 4 * ri.numel() + 4 * (Fr * B + 1)
    peak = None
    try:
        peak = json.load(open(os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                           'MEASURED_PEAKS.json')))['hbm_gbs']
    except Exception:
        pass
    res = dict(what='input dist (KJT all-to-all) device passes, rank 0', config=a.config, world=W, B=B,
               local_ids=int(idx0.numel()), recv_ids=int(ri.numel()), owned_features=Fr,
               pack_ms=t_pack, pack_gbs=pack_bytes / t_pack / 1e6, unpack_ms=t_unpack,
               unpack_gbs=unpack_bytes / t_unpack / 1e6, hbm_peak_gbs=peak,
               nvlink_a2a_ms_at_900gbs=4 * max(idx0.numel(), ri.numel()) / 900e9 * 1e3)
    print(json.dumps(res))


if __name__ == '__main__':
    main()
