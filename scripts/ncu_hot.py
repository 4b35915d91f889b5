"""Top SASS lines of an ncu report by stall samples (needs --import-source / -lineinfo)."""
import csv, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 40
out = subprocess.run(['ncu', '-i', rep, '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True, check=True).stdout
rows = list(csv.reader(out.splitlines()))
h = rows[1]
data = rows[2:]
ia, isrc = h.index('Address'), h.index('Source')
iex, ist = h.index('Instructions Executed'), h.index('Warp Stall Sampling (All Samples)')
tot = sum(float(r[ist] or 0) for r in data)
inst = sum(float(r[iex] or 0) for r in data)
print(f'samples {tot:.0f}  instructions {inst:.3e}')
for i, r in sorted(enumerate(data), key=lambda t: -float(t[1][ist] or 0))[:top]:
    print(f'{i:5d} {float(r[ist]) / tot * 100:5.2f}% {float(r[iex] or 0) / 1e6:8.1f}M  {r[isrc][:80]}')
