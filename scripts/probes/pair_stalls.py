"""Top SASS stall lines of one kernel in an ncu report (source page), by name substring."""
import csv
import io
import subprocess
import sys

rep, want, top = sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else 40
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
for b in src.split('"Kernel Name"')[1:]:
    lines = ('"Kernel Name"' + b).splitlines()
    if want not in lines[0]:
        continue
    rows = list(csv.reader(io.StringIO("\n".join(lines[1:]))))
    h = rows[0]
    ia, isrc, iss, ie = (h.index('Address'), h.index('Source'), h.index('Warp Stall Sampling (All Samples)'),
                         h.index('Instructions Executed'))
    data = []
    for r in rows[1:]:
        try:
            data.append((int(r[iss] or 0), r[ia][-5:], r[isrc][:90], r[ie]))
        except Exception:
            pass
    tot = sum(d[0] for d in data) or 1
    print(lines[0][:150], "samples", tot)
    for d in sorted(data, reverse=True)[:top]:
        print(f"{d[0]:7d} {100 * d[0] / tot:5.1f}% {d[1]} {d[2]}  exec={d[3]}")
    break
