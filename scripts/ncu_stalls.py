"""Summarise an ncu report: per-kernel key metrics + top SASS stall lines."""
import csv, io, subprocess, sys
rep = sys.argv[1]
kre = sys.argv[2] if len(sys.argv) > 2 else None
top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr = rows[0]
want = ['Kernel Name', 'gpu__time_duration.sum', 'dram__bytes_read.sum', 'dram__bytes_write.sum',
        'sm__warps_active.avg.pct_of_peak_sustained_active', 'smsp__inst_executed.sum',
        'sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed',
        'smsp__issue_active.avg.pct_of_peak_sustained_active']
for r in rows[2:]:
    print({w.split('.')[0][-24:]: r[hdr.index(w)][:70] for w in want if w in hdr})
if kre:
    cmd = ["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{kre}", "--print-source", "sass"]
    src = subprocess.run(cmd, capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(src)))
    h = rows[1] if len(rows) > 1 else []
    if 'Warp Stall Sampling (All Samples)' in h:
        ia, isrc, iss = h.index('Address'), h.index('Source'), h.index('Warp Stall Sampling (All Samples)')
        data, seen = [], set()
        for r in rows[2:]:
            try:
                key = (r[ia], r[isrc])
                if key in seen:
                    continue
                seen.add(key)
                data.append((int(r[iss] or 0), r[ia], r[isrc]))
            except Exception:
                pass
        tot = sum(d[0] for d in data) or 1
        print('samples', tot)
        for sv, a, sr in sorted(data, reverse=True)[:top]:
            print(f"{sv:6d} {100*sv/tot:5.1f}% {a[-5:]} {sr[:100]}")
