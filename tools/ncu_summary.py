"""Summarise an ncu --set full report of the fused kernel into profiles/.

    python tools/ncu_summary.py gpurun_out/prof_heavy.ncu-rep heavy r02 [--dtype f32] [--suffix _w2_r0]

Writes profiles/<tag>_ncu_<config>.md (human summary) and
profiles/ncu_traffic_<config>[_dtype][suffix].json (dram bytes per launch, read
by bench.py).  Algorithmic bytes (C26) and algorithmic ROW bytes are the mean
over the bench's rotating batches (seeds 7, 8, 9); sector efficiency (SURVEY
§8d) = algorithmic row bytes / (global-load sectors x 32).
"""
import argparse
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = [
    ('gpu__time_duration.sum', 'duration'),
    ('dram__bytes_read.sum', 'DRAM read'),
    ('dram__bytes_write.sum', 'DRAM write'),
    ('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'DRAM throughput % of peak'),
    ('lts__t_sector_hit_rate.pct', 'L2 hit rate'),
    ('lts__throughput.avg.pct_of_peak_sustained_elapsed', 'L2 throughput %'),
    ('l1tex__t_sector_hit_rate.pct', 'L1 hit rate'),
    ('sm__warps_active.avg.pct_of_peak_sustained_active', 'achieved occupancy %'),
    ('launch__registers_per_thread', 'registers/thread'),
    ('launch__occupancy_limit_registers', 'occupancy limit (regs, CTAs)'),
    ('launch__occupancy_limit_shared_mem', 'occupancy limit (smem, CTAs)'),
    ('launch__grid_size', 'grid'),
    ('smsp__thread_inst_executed_per_inst_executed.ratio', 'active threads / warp inst (Table II row 6)'),
    ('smsp__thread_inst_executed_pred_on_per_inst_executed.ratio', 'not-predicated-off threads / inst (Table II row 7)'),
    ('l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum', 'global load sectors'),
    ('l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum', 'global load requests'),
    ('smsp__issue_active.avg.pct_of_peak_sustained_active', 'issue active %'),
    ('l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum', 'local-memory (spill) load sectors'),
    ('l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum', 'local-memory (spill) store sectors'),
    ('l1tex__m_l1tex2xbar_write_bytes.sum', 'L1 -> L2 write bytes (stores + local evictions)'),
    ('launch__shared_mem_config_size', 'shared memory config per SM'),
]


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    launches = [dict(zip(hdr, r)) for r in rows[2:]]
    return hdr, units, launches


def num(s):
    try:
        return float(str(s).replace(',', ''))
    except ValueError:
        return None


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument('rep')
    ap.add_argument('config')
    ap.add_argument('tag')
    ap.add_argument('--alg-bytes', type=float, default=None)
    ap.add_argument('--dtype', default='f32')
    ap.add_argument('--suffix', default='', help="e.g. '_w2_r0' for a rank plan")
    a = ap.parse_args()
    row_bytes = None
    if a.alg_bytes is None:
        sys.path.insert(0, ROOT)
        from paper_conf_sc_panzzxwslr0d24_b200 import synth
        m = synth.make_model(a.config)
        al, rb = [], []
        for i in range(3):
            ab = synth.algorithmic_bytes(m, synth.make_batch(m, 7 + i), a.dtype)
            al.append(ab['total'])
            rb.append(ab.get('rows', ab['total']))
        a.alg_bytes = sum(al) / len(al)
        row_bytes = sum(rb) / len(rb)
    hdr, units, launches = raw(a.rep)
    unit = dict(zip(hdr, units))
    os.makedirs(os.path.join(ROOT, 'profiles'), exist_ok=True)
    L0 = launches[-1]
    kname = L0.get('Kernel Name', 'recflex fused kernel')
    lines = [f'# ncu --set full: `{kname}`, config `{a.config}` ({a.tag})', '',
             f'source: `{os.path.basename(a.rep)}` ({len(launches)} launch(es) profiled, '
             '`--clock-control none`, cold L2 per replay)', '']
    L = launches[-1]
    lines.append('| metric | value | unit |')
    lines.append('|---|---|---|')
    for k, name in KEYS:
        if k in L:
            lines.append(f'| {name} (`{k}`) | {L[k]} | {unit.get(k, "")} |')
    # stall breakdown
    stalls = []
    for k in hdr:
        if k.startswith('smsp__pcsamp_warps_issue_stalled_') and not k.endswith('not_issued'):
            v = num(L.get(k))
            if v:
                stalls.append((v, k.replace('smsp__pcsamp_warps_issue_stalled_', '')))
    tot = sum(v for v, _ in stalls) or 1.0
    lines += ['', '**Warp stall samples** (top 8):', '']
    for v, k in sorted(stalls, reverse=True)[:8]:
        lines.append(f'- {k}: {100 * v / tot:.1f}%')
    rd, wr = num(L.get('dram__bytes_read.sum')), num(L.get('dram__bytes_write.sum'))
    scale = {'byte': 1, 'Kbyte': 1e3, 'Mbyte': 1e6, 'Gbyte': 1e9}
    rd_b = rd * scale.get(unit.get('dram__bytes_read.sum'), 1) if rd is not None else None
    wr_b = wr * scale.get(unit.get('dram__bytes_write.sum'), 1) if wr is not None else None
    traffic = (rd_b or 0) + (wr_b or 0)
    if a.alg_bytes:
        lines += ['', f'Algorithmic bytes per launch (C26): {a.alg_bytes / 1e9:.3f} GB; DRAM traffic '
                      f'{traffic / 1e9:.3f} GB = {traffic / a.alg_bytes:.3f}x algorithmic.']
    sect = num(L.get('l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum'))
    if row_bytes and sect:
        sect *= {'sector': 1, 'Ksector': 1e3, 'Msector': 1e6, 'Gsector': 1e9}.get(
            unit.get('l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum'), 1)
        lines += [f'Sector efficiency (SURVEY §8d): algorithmic row bytes {row_bytes / 1e9:.3f} GB / '
                  f'(global-load sectors x 32 = {sect * 32 / 1e9:.3f} GB) = {row_bytes / (sect * 32):.3f} '
                  '(the global-load sectors also count the lookup-ID and offset loads).']
        loc = num(L.get('l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum'))
        if loc is not None:
            loc *= {'sector': 1, 'Ksector': 1e3, 'Msector': 1e6, 'Gsector': 1e9}.get(
                unit.get('l1tex__t_sectors_pipe_lsu_mem_local_op_ld.sum'), 1)
            lines += [f'Local-memory (spill) load sectors / global-load sectors = {loc / sect:.4f}.']
    with open(os.path.join(ROOT, 'profiles', f'{a.tag}_ncu_{a.config}.md'), 'w') as fh:
        fh.write('\n'.join(lines) + '\n')
    tname = f'ncu_traffic_{a.config}' + ('' if a.dtype == 'f32' else f'_{a.dtype}') + a.suffix + '.json'
    with open(os.path.join(ROOT, 'profiles', tname), 'w') as fh:
        json.dump({'dram_bytes_per_launch': traffic, 'dram_read_bytes': rd_b, 'dram_write_bytes': wr_b,
                   'source': os.path.basename(a.rep), 'tag': a.tag}, fh, indent=1)
    print('\n'.join(lines))


if __name__ == '__main__':
    sys.exit(main())
