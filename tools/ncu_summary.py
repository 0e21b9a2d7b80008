"""Summarise an ncu report (--page raw --csv) for the library's kernels."""
import csv
import io
import json
import subprocess
import sys

WANT = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'lts__t_bytes.sum',
        'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__warps_active.avg.pct_of_peak_sustained_active',
        'smsp__issue_active.avg.pct_of_peak_sustained_active',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active',
        'sm__pipe_shared_cycles_active.avg.pct_of_peak_sustained_active',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum',
        'smsp__inst_executed.sum', 'launch__registers_per_thread', 'launch__grid_size',
        'launch__block_size', 'sm__cycles_elapsed.avg.per_second',
        'smsp__average_warp_latency_issue_stalled_barrier',
        ]


def load(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True,
                         text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, units, data = rows[0], rows[1], rows[2:]
    res = []
    for r in data:
        d = {'kernel': r[h.index('Kernel Name')].split('(')[0].replace('nba::', '')}
        for w in WANT:
            if w in h:
                d[w] = (r[h.index(w)], units[h.index(w)])
        res.append(d)
    return res


if __name__ == '__main__':
    for rep in sys.argv[1:]:
        print('==', rep)
        for d in load(rep):
            print(' ', d['kernel'])
            for k, (v, u) in ((k, v) for k, v in d.items() if k != 'kernel'):
                print(f'     {k:66s} {v:>14s} {u}')
