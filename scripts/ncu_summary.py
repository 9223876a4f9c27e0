"""Summarise an ncu report (details page) for the profiles/ directory."""
import csv, subprocess, sys
WANT = ['Duration', 'DRAM Throughput', 'L2 Cache Throughput', 'Compute (SM) Throughput', 'Executed Ipc Active',
        'Issue Slots Busy', 'Registers Per Thread', 'Grid Size', 'Block Size', 'Achieved Occupancy',
        'Memory Throughput', 'One or More Eligible', 'SM Frequency', 'Dynamic Shared Memory Per Block']
def summary(path):
    out = subprocess.run(['ncu', '-i', path, '--page', 'details', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    mi, ui, vi, ki = h.index('Metric Name'), h.index('Metric Unit'), h.index('Metric Value'), h.index('Kernel Name')
    res = {}
    for r in rows[1:]:
        if len(r) > vi and r[mi] in WANT:
            res[r[mi]] = (r[vi], r[ui])
    return rows[1][ki] if len(rows) > 1 else '', res
def raw(path, names):
    out = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(out.splitlines()))
    h = rows[0]
    return {n: (rows[2][h.index(n)] if n in h else None) for n in names}
if __name__ == '__main__':
    for p in sys.argv[1:]:
        k, r = summary(p)
        print('==', p, k[:60])
        for n in WANT:
            if n in r: print(f'   {n:36s} {r[n][0]} {r[n][1]}')
        print('  ', raw(p, ['dram__bytes_read.sum', 'dram__bytes_write.sum', 'sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active', 'gpu__time_duration.sum']))
