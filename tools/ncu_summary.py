"""Summarise ncu --set full reports: time, DRAM bytes/throughput, L2, occupancy, top stall reasons."""
import csv, io, subprocess, sys

KEYS = ['gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed', 'lts__t_sector_hit_rate.pct',
        'lts__throughput.avg.pct_of_peak_sustained_elapsed', 'l1tex__t_sector_hit_rate.pct',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'launch__registers_per_thread', 'launch__grid_size',
        'smsp__issue_active.avg.pct_of_peak_sustained_active', 'sm__throughput.avg.pct_of_peak_sustained_elapsed']


def summary(path):
    raw = subprocess.run(['ncu', '-i', path, '--page', 'raw', '--csv'], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = dict(zip(h, r))
        lines = [f"kernel: {d.get('Kernel Name', '')[:100]}"]
        for k in KEYS:
            if k in d:
                lines.append(f"  {k} = {d[k]} {u[h.index(k)]}")
        st = [(k, float(v)) for k, v in d.items()
              if k.startswith('smsp__average_warps_issue_stalled_') and k.endswith('_per_issue_active.ratio')]
        st.sort(key=lambda t: -t[1])
        lines.append('  stalls/issue: ' + ', '.join(f"{k[34:-23]}={v:.1f}" for k, v in st[:5]))
        out.append('\n'.join(lines))
    return '\n'.join(out)


if __name__ == '__main__':
    for p in sys.argv[1:]:
        print('==', p)
        print(summary(p))
