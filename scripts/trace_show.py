import collections
ev = []
for ln in open('gpurun_out/trace.txt'):
    f = ln.split()
    ev.append((int(f[0]), f[1], int(f[3]), int(f[5])))
# per (role, tile): stamps by event id
d = collections.defaultdict(dict)
for t, role, tile, e in ev:
    key = (role, tile)
    d[key].setdefault(e, t)
print("worker phase durations (cycles): wait_full conv wait_acc epi")
for (role, tile), st in sorted(d.items(), key=lambda x: (x[0][1], x[0][0])):
    if role.startswith('w') and all(k in st for k in range(5)):
        print(f"{role:4s} tile {tile:2d} start {st[0]:7d} wfull {st[1]-st[0]:6d} conv {st[2]-st[1]:6d} wacc {st[3]-st[2]:6d} epi {st[4]-st[3]:6d}")
    if role == 'mma' and 0 in st and 1 in st:
        print(f"mma  tile {tile:2d} waited {st[1]-st[0]:6d} at {st[1]}")
