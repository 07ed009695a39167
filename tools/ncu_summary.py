#!/usr/bin/env python3
"""Summarise ncu reports: key throughput/occupancy metrics and top stall reasons.
   python tools/ncu_summary.py gpurun_out/r01c_k_predict.ncu-rep [...]"""
import csv, io, subprocess, sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_bytes.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'launch__occupancy_limit_shared_mem', 'launch__occupancy_limit_registers',
        'launch__shared_mem_per_block_dynamic', 'launch__shared_mem_per_block_static',
        'launch__grid_size', 'launch__block_size', 'sm__inst_executed.sum',
        'smsp__inst_executed.avg.per_cycle_active', 'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum']


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main():
    for rep in sys.argv[1:]:
        hdr, units, vals = raw(rep)
        if not vals:
            print(rep, 'no data'); continue
        v = vals[0]
        print('==', rep, v[hdr.index('Kernel Name')] if 'Kernel Name' in hdr else '')
        for k in KEYS:
            if k in hdr:
                i = hdr.index(k); print('  %-70s %s %s' % (k, v[i], units[i]))
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith('smsp__average_warp_latency_issue_stalled_') and h.endswith('.ratio') is False:
                pass
            if h.startswith('smsp__pcsamp_warps_issue_stalled_') and not h.endswith('not_issued'):
                try:
                    stalls.append((float(v[i].replace(',', '')), h.replace('smsp__pcsamp_warps_issue_stalled_', '')))
                except ValueError:
                    pass
        tot = sum(s for s, _ in stalls) or 1
        print('  top stall reasons (pc sampling):', ', '.join('%s %.0f%%' % (n, 100 * s / tot)
                                                             for s, n in sorted(stalls, reverse=True)[:6]))


if __name__ == '__main__':
    main()
