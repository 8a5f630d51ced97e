"""Summarise an ncu --set full report of recflex_fused_kernel into profiles/.

    python tools/ncu_summary.py gpurun_out/prof_heavy.ncu-rep heavy r01 [--alg-bytes N]

Writes profiles/<tag>_ncu_<config>.md (human summary) and
profiles/ncu_traffic_<config>.json (dram bytes per launch, read by bench.py).
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
    a = ap.parse_args()
    hdr, units, launches = raw(a.rep)
    unit = dict(zip(hdr, units))
    os.makedirs(os.path.join(ROOT, 'profiles'), exist_ok=True)
    lines = [f'# ncu --set full: recflex_fused_kernel, config `{a.config}` ({a.tag})', '',
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
    with open(os.path.join(ROOT, 'profiles', f'{a.tag}_ncu_{a.config}.md'), 'w') as fh:
        fh.write('\n'.join(lines) + '\n')
    with open(os.path.join(ROOT, 'profiles', f'ncu_traffic_{a.config}.json'), 'w') as fh:
        json.dump({'dram_bytes_per_launch': traffic, 'dram_read_bytes': rd_b, 'dram_write_bytes': wr_b,
                   'source': os.path.basename(a.rep), 'tag': a.tag}, fh, indent=1)
    print('\n'.join(lines))


if __name__ == '__main__':
    sys.exit(main())
