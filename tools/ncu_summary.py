"""Summarise an ncu report (raw page) into the handful of metrics we track."""
import csv
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed',
        'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'launch__grid_size', 'launch__block_size',
        'lts__t_sector_hit_rate.pct', 'l1tex__t_sector_hit_rate.pct',
        'l1tex__throughput.avg.pct_of_peak_sustained_active',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum',
        'smsp__inst_executed_op_shared_ld.sum',
        'l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum',
        'l1tex__data_pipe_lsu_wavefronts_mem_lg.sum',
        'sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed']


def main(path):
    out = subprocess.check_output(['ncu', '-i', path, '--page', 'raw', '--csv'], text=True, stderr=subprocess.DEVNULL)
    rows = list(csv.reader(out.splitlines()))
    h, u = rows[0], rows[1]
    for v in rows[2:]:
        print('kernel:', v[h.index('Kernel Name')][:90])
        for k in KEYS:
            if k in h:
                i = h.index(k)
                print(f'  {k} = {v[i]} {u[i]}')
        st = []
        for i, k in enumerate(h):
            if k.startswith('smsp__average_warps_issue_stalled_') and k.endswith('_per_issue_active.ratio'):
                try:
                    st.append((float(v[i]), k[len('smsp__average_warps_issue_stalled_'):-len('_per_issue_active.ratio')]))
                except ValueError:
                    pass
        st.sort(reverse=True)
        print('  stalls/issue:', ', '.join(f'{n}={x:.2f}' for x, n in st[:8]))


if __name__ == '__main__':
    for p in sys.argv[1:]:
        main(p)
