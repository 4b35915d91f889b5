"""Basic-block instruction counts of the hottest kernel in an ncu report (SASS + executions)."""
import csv, subprocess, sys
out = subprocess.run(['ncu', '-i', sys.argv[1], '--page', 'source', '--csv', '--print-source', 'sass'],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(out.splitlines())); h = rows[1]; data = rows[2:]
isrc, iex, ist = h.index('Source'), h.index('Instructions Executed'), h.index('Warp Stall Sampling (All Samples)')
thr = float(sys.argv[2]) if len(sys.argv) > 2 else 1e6
blocks = []; cur = None
for r in data:
    ex = float(r[iex] or 0)
    if ex < thr:
        cur = None; continue
    if cur and abs(cur[0] - ex) < 1:
        cur[1] += 1; cur[2].append(r[isrc]); cur[3] += float(r[ist] or 0)
    else:
        cur = [ex, 1, [r[isrc]], float(r[ist] or 0)]; blocks.append(cur)
tot = sum(b[0] * b[1] for b in blocks); st = sum(b[3] for b in blocks)
for ex, n, src, s in blocks:
    print(f"{ex/1e6:7.2f}M x {n:3d} = {ex*n/1e6:8.1f}M ({ex*n/tot*100:4.1f}% inst, {s/st*100:4.1f}% stall)  {src[0][:34]} .. {src[-1][:34]}")
print('total', tot / 1e6)
