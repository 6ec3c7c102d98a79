"""Per-source-line instruction counts and stall samples of one kernel in an ncu
report: joins ncu's SASS page (absolute addresses) with `nvdisasm -g` line info of
the matching cubin.  usage: sass_lines.py REPORT KERNEL_REGEX CUBIN [TOP]"""
import csv, io, re, subprocess, sys, collections
rep, kre, cubin = sys.argv[1:4]
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
rev = sys.argv[5] if len(sys.argv) > 5 else None      # read sources at this git revision
base_re, _, pick = kre.partition("@")          # "rowgemm@(int)2>" -> ncu filter, name filter
src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "-k", f"regex:{base_re}",
                      "--print-source", "sass"], capture_output=True, text=True).stdout
blocks = [x for x in src.split('"Kernel Name",')[1:] if pick in x.split("\n", 1)[0]]
b = blocks[0]
kname = b.split("\n", 1)[0].strip().strip('"')
rows = list(csv.reader(io.StringIO(b.split("\n", 1)[1])))
h = rows[0]
iA, iS, iI, iW = (h.index("Address"), h.index("Source"), h.index("Instructions Executed"),
                  h.index("Warp Stall Sampling (All Samples)"))
sass = []
for r in rows[1:]:
    try:
        sass.append((int(r[iA], 16), r[iS].strip(), float(r[iI] or 0), float(r[iW] or 0)))
    except (ValueError, IndexError):
        pass
base = min(a for a, *_ in sass)
# mangled-name fragment from the demangled template arguments
m = re.search(r"(\w+)<\(int\)(\d+), \(int\)(\d+)>", kname)
frag = f"{m.group(1)}ILi{m.group(2)}ELi{m.group(3)}E" if m else re.sub(r"\W.*", "", kname.split("::")[-1])
dis = subprocess.run(["nvdisasm", "-g", "-c", cubin], capture_output=True, text=True).stdout
line_of, cur_fn, cur_line = {}, None, None
for ln in dis.split("\n"):
    if ln.startswith(".text."):
        cur_fn = ln[6:].rstrip(":")
        continue
    mm = re.search(r'//## File "(.*?)", line (\d+)', ln)
    if mm:
        cur_line = (mm.group(1), int(mm.group(2)))
        continue
    mo = re.search(r"/\*([0-9a-f]{4,})\*/", ln)
    if mo and cur_fn and frag in cur_fn:
        line_of[int(mo.group(1), 16)] = cur_line
agg = collections.defaultdict(lambda: [0.0, 0.0])
tot_i = tot_w = 0.0
for a, s, n, w in sass:
    l = line_of.get(a - base)
    agg[l][0] += n
    agg[l][1] += w
    tot_i += n
    tot_w += w
cache = {}
def text(fl):
    if not fl:
        return "?"
    f, l = fl
    if f not in cache:
        try:
            if rev and "/root/repo/" in f:
                rel = f.split("/root/repo/", 1)[1]
                cache[f] = subprocess.run(["git", "show", f"{rev}:{rel}"], capture_output=True,
                                          text=True).stdout.split("\n")
            else:
                cache[f] = open(f).read().split("\n")
        except OSError:
            cache[f] = []
    ls = cache[f]
    return f"{f.rsplit('/', 1)[-1]}:{l}: " + (ls[l - 1].strip()[:80] if l <= len(ls) else "?")
print(kname, f"instructions {tot_i:.0f}, stall samples {tot_w:.0f}, mapped lines {len(line_of)}")
for fl, (n, w) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{100*n/tot_i:5.1f}% inst {100*w/max(tot_w,1):5.1f}% stall  {text(fl)}")
