"""Summarise an ncu --set full report of the count kernel (run here, no GPU).

usage: python scripts/ncu_summary.py gpurun_out/X.ncu-rep [--sass N]
Prints the headline counters (time, DRAM/L2 bytes, issue, occupancy, stalls,
shared-memory wavefronts) and optionally the N hottest SASS instructions.
"""
import csv
import io
import subprocess
import sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'dram__throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_bytes.sum',
        'lts__t_sector_hit_rate.pct', 'lts__throughput.avg.pct_of_peak_sustained_elapsed',
        'l1tex__throughput.avg.pct_of_peak_sustained_active', 'l1tex__t_sector_hit_rate.pct',
        'sm__throughput.avg.pct_of_peak_sustained_elapsed',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread',
        'launch__occupancy_limit_shared_mem', 'launch__occupancy_limit_registers',
        'launch__grid_size', 'launch__block_size', 'launch__shared_mem_per_block_dynamic',
        'sm__cycles_active.avg', 'sm__cycles_active.max', 'sm__cycles_active.min',
        'smsp__thread_inst_executed_per_inst_executed.ratio',
        'l1tex__data_pipe_lsu_wavefronts_mem_shared.sum',
        'l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum',
        'l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum',
        'l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum']


def raw(rep):
    out = subprocess.run(['ncu', '-i', rep, '--page', 'raw', '--csv'], capture_output=True,
                         text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def main():
    rep = sys.argv[1]
    hdr, units, vals = raw(rep)
    for v in vals:
        print('kernel:', v[hdr.index('Kernel Name')][:80])
        for k in KEYS:
            if k in hdr:
                print(f'  {k:60s} {v[hdr.index(k)]:>22s} {units[hdr.index(k)]}')
        st = [(h, v[i]) for i, h in enumerate(hdr)
              if h.startswith('smsp__average_warps_issue_stalled') and h.endswith('per_issue_active.ratio')]
        st.sort(key=lambda x: -float(x[1] or 0))
        for h, x in st[:8]:
            print(f'  stall {h.split("stalled_")[1].split("_per")[0]:28s} {x}')
    if '--sass' in sys.argv:
        n = int(sys.argv[sys.argv.index('--sass') + 1])
        out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'],
                             capture_output=True, text=True, check=True).stdout
        rows = list(csv.reader(io.StringIO(out)))
        h = rows[1]
        ia, isrc = h.index('Instructions Executed'), h.index('Source')
        data = [(int(r[ia] or 0), i, r[isrc]) for i, r in enumerate(rows[2:]) if len(r) > ia]
        tot = sum(d[0] for d in data)
        print('total warp instructions', tot)
        for c, i, src in data:
            if c > tot * n / 10000:
                print(f'{i:5d} {c / 1e9:7.3f}G  {src[:90]}')


if __name__ == '__main__':
    main()
