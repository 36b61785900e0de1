"""Tabulate key metrics of every kernel in an .ncu-rep (ncu -i ... --page raw --csv)."""
import csv
import subprocess
import sys

COLS = [('gpu__time_duration.sum', 'us'), ('dram__bytes_read.sum', 'rdMB'), ('dram__bytes_write.sum', 'wrMB'),
        ('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'dram%'),
        ('sm__throughput.avg.pct_of_peak_sustained_elapsed', 'sm%'), ('launch__registers_per_thread', 'regs'),
        ('sm__warps_active.avg.pct_of_peak_sustained_active', 'occ%'), ('smsp__inst_executed.sum', 'Minst'),
        ('launch__grid_size', 'grid'),
        ('smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio', 'lsb'),
        ('smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio', 'ssb'),
        ('smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio', 'bar'),
        ('smsp__average_warps_issue_stalled_wait_per_issue_active.ratio', 'wait'),
        ('smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio', 'lgthr'),
        ('smsp__average_warps_issue_stalled_mio_throttle_per_issue_active.ratio', 'mio'),
        ('smsp__issue_active.avg.pct_of_peak_sustained_active', 'issue%'),
        ('sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active', 'xu%'),       # MUFU (ex2, rcp, lg2)
        ('lts__t_requests_srcunit_tex_op_red.sum', 'L2red')]                          # global reductions (requests)


def main(path, kfilter=None):
    out = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h, u = rows[0], rows[1]
    ki = h.index('Kernel Name')
    idx = [(h.index(c) if c in h else None, n) for c, n in COLS]
    print('%-20s' % 'kernel' + ''.join('%8s' % n for _, n in idx))
    for r in rows[2:]:
        name = r[ki].split('(')[0].replace('void ', '').replace('dp::<unnamed>::', '')[:20]
        if kfilter and kfilter not in name:
            continue
        vals = []
        for i, n in idx:
            if i is None:
                vals.append('-')
                continue
            v = r[i]
            try:
                f = float(v.replace(',', ''))
                unit = u[i]
                if n == 'us' and unit in ('nsecond', 'ns'):
                    f /= 1000
                if n == 'us' and unit in ('msecond',):
                    f *= 1000
                if n in ('rdMB', 'wrMB'):
                    f = f / 1e6 if unit == 'byte' else (f / 1e3 if unit == 'Kbyte' else (f * 1e3 if unit == 'Gbyte' else f))
                if n == 'Minst':
                    f /= 1e6
                vals.append('%8.1f' % f if f < 1e5 else '%8.0f' % f)
            except ValueError:
                vals.append('%8s' % v[:8])
        print('%-20s' % name + ''.join(vals))


if __name__ == '__main__':
    main(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else None)
