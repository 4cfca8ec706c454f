"""Top SASS instructions by warp-stall samples from an ncu report (source page, sass view)."""
import csv, io, subprocess, sys

path = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
raw = subprocess.run(['ncu', '-i', path, '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
for i, r in enumerate(rows):
    if 'Address' in r and 'Source' in r:
        h = r
        body = rows[i + 1:]
        break
ix = {k: h.index(k) for k in h}
tot = sum(float(r[ix['Warp Stall Sampling (All Samples)']] or 0) for r in body if len(r) == len(h))
print('total samples', tot, 'instructions', len(body))
seq = [r for r in body if len(r) == len(h)]
for r in seq:
    r.append(float(r[ix['Warp Stall Sampling (All Samples)']] or 0))
mode = sys.argv[3] if len(sys.argv) > 3 else 'top'
if mode == 'all':
    for r in seq:
        print(f"{r[ix['Address']]:>6} {r[-1]:7.0f} {r[ix['Instructions Executed']]:>10} {r[ix['Source']][:90]}")
else:
    for r in sorted(seq, key=lambda r: -r[-1])[:n]:
        stalls = sorted(((k, float(r[ix[k]] or 0)) for k in h if k.startswith('stall_') and 'Not Issued' not in k),
                        key=lambda t: -t[1])[:3]
        print(f"{r[ix['Address']]:>6} {r[-1]:7.0f} {100*r[-1]/tot:5.1f}% {r[ix['Source']][:70]:70s} "
              + ' '.join(f"{k[6:]}={v:.0f}" for k, v in stalls))
