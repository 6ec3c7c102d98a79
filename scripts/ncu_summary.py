"""Summarise ncu captures of one round into profiles/ (run on the GPU box or here).

    python scripts/ncu_summary.py TAG launches.csv  [REP:TITLE:TRAFFIC_JSON ...]

* launches.csv (ncu --metrics gpu__time_duration.sum,dram__bytes_*.sum --csv): per-launch
  list -> profiles/TAG_launches.csv + a class table (share of time, DRAM bytes / launch);
* each REP.ncu-rep (ncu --set full): per kernel class, DRAM bytes / launch, DRAM %, tensor
  pipe %, issue active %, registers -> profiles/TRAFFIC_JSON and a section of
  profiles/TAG_ncu_summary.md.
"""
import collections
import csv
import io
import json
import os
import subprocess
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.environ.get("PROFILES_OUT", os.path.join(ROOT, "profiles"))


def kname(full):
    import re
    m = re.search(r"rowgemm_pair_kernel<(?:\(int\))?(\d+)[,>]", full)
    if m:
        return ["node_tc", "edge_tc", "gate_tc"][int(m.group(1))]
    m = re.search(r"rowgemm(?:_bf16)?_kernel<(?:\(int\))?(\d+), (?:\(int\))?(\d+)", full)
    if m:
        return ["node_tc", "edge_tc", "gate_tc", "plain_tc", "gatebwd_tc", "edgebwd_tc",
                "gateagg_tc"][int(m.group(2))]
    for k in ("gate_bwd_stream", "edge_bwd_small", "node_bwd", "wgrad_tc", "multi_reduce",
              "split_reduce", "gather_segsum", "edge_small", "broadcast_dh", "head_bwd_graph",
              "head_bwd_reduce", "adam", "wimage", "readout_head", "attn_bwd_q", "attn_bwd_kv",
              "ln_bwd", "colsum", "col_reduce", "mask_dA", "dec_tail_bwd", "dec_pool_bwd",
              "dec_seed_grads", "gph_attn", "gph_ln", "set_decoder_pool", "set_decoder_prep",
              "set_decoder_kernel", "synth", "wgrad_skinny", "wgrad_partial", "row_exp",
              "gather_hubs", "hub_partial", "hub_merge", "small_forward", "edge_gate", "edgegate"):
        if k in full:
            return k
    return full[:40]


def launches(tag, path):
    txt = open(path).read()
    rows = list(csv.reader(io.StringIO(txt[txt.index('"ID"'):])))
    hdr = rows[0]
    iK, iM, iV, iID = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value"), hdr.index("ID")
    iU = hdr.index("Metric Unit") if "Metric Unit" in hdr else None
    to_base = {"nsecond": 1.0, "ns": 1.0, "usecond": 1e3, "us": 1e3, "msecond": 1e6, "ms": 1e6,
               "second": 1e9, "s": 1e9, "byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
    per = collections.OrderedDict()
    for r in rows[1:]:
        if len(r) <= max(iK, iM, iV, iID):
            continue
        d = per.setdefault(r[iID], {"kernel": r[iK]})
        sc = to_base.get(r[iU], 1.0) if iU is not None else 1.0      # times -> ns, bytes -> B
        d[r[iM]] = float(r[iV].replace(",", "")) * sc
    with open(os.path.join(OUT, f"{tag}_launches.csv"), "w") as f:
        f.write("id,kernel,class,gpu_time_ns,dram_read_bytes,dram_write_bytes\n")
        for i, d in per.items():
            f.write(f"{i},\"{d['kernel'][:80]}\",{kname(d['kernel'])},{d.get('gpu__time_duration.sum', 0):.0f},"
                    f"{d.get('dram__bytes_read.sum', 0):.0f},{d.get('dram__bytes_write.sum', 0):.0f}\n")
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
    for d in per.values():
        a = agg[kname(d["kernel"])]
        a[0] += 1
        a[1] += d.get("gpu__time_duration.sum", 0)
        a[2] += d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
    tot = sum(a[1] for a in agg.values()) or 1
    dram = any(a[2] > 0 for a in agg.values())
    if dram:
        lines = ["| class | launches | total µs | share of time | mean DRAM MB / launch |", "|---|---|---|---|---|"]
    else:
        lines = ["| class | launches | total µs | share of time |", "|---|---|---|---|"]
    for k, a in sorted(agg.items(), key=lambda x: -x[1][1]):
        row = f"| {k} | {a[0]} | {a[1] / 1e3:.1f} | {100 * a[1] / tot:.1f} % |"
        lines.append(row + (f" {a[2] / a[0] / 1e6:.1f} |" if dram else ""))
    return "\n".join(lines)


def capture(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr = rows[0]

    def g(r, k):
        try:
            return float(r[hdr.index(k)].replace(",", ""))
        except Exception:
            return None
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(rows[1][hdr.index("dram__bytes_read.sum")], 1)
    tunit = rows[1][hdr.index("gpu__time_duration.sum")]
    tscale = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3,
              "second": 1e6, "s": 1e6}[tunit]
    acc = collections.defaultdict(list)
    for r in rows[2:]:
        acc[kname(r[hdr.index("Kernel Name")])].append({
            "time_us": (g(r, "gpu__time_duration.sum") or 0) * tscale,
            "dram": ((g(r, "dram__bytes_read.sum") or 0) + (g(r, "dram__bytes_write.sum") or 0)) * scale,
            "dram_pct": g(r, "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed") or 0,
            "tensor": g(r, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed") or 0,
            "issue": g(r, "smsp__issue_active.avg.pct_of_peak_sustained_active") or 0,
            "regs": g(r, "launch__registers_per_thread") or 0})
    out = {}
    for k, lst in acc.items():
        n = len(lst)
        out[k] = {"dram_bytes_per_launch": sum(x["dram"] for x in lst) / n, "launches_captured": n,
                  "mean_time_us_under_ncu": sum(x["time_us"] for x in lst) / n,
                  "dram_throughput_pct": sum(x["dram_pct"] for x in lst) / n,
                  "tensor_pipe_pct": sum(x["tensor"] for x in lst) / n,
                  "issue_active_pct": sum(x["issue"] for x in lst) / n, "registers": lst[0]["regs"]}
    return out


def main():
    tag, lpath = sys.argv[1], sys.argv[2]
    os.makedirs(OUT, exist_ok=True)
    md = [f"# {tag}: ncu evidence (serialised, cold-cache replays; --clock-control none)\n"]
    if os.path.exists(lpath) and '"ID"' in open(lpath).read():
        md += [f"## launch list ({os.path.basename(lpath)})\n", launches(tag, lpath), ""]
    for spec in sys.argv[3:]:
        rep, title, tj = spec.split(":", 2)
        if not os.path.exists(rep):
            continue
        t = capture(rep)
        for v in t.values():
            v["source"] = f"profiles/{tag}: {title}"
        json.dump(t, open(os.path.join(OUT, tj), "w"), indent=1)
        md += [f"## {title}\n", "| kernel | launches | us/launch | DRAM MB/launch | DRAM % | tensor pipe % | issue active % | regs |",
               "|---|---|---|---|---|---|---|---|"]
        for k, v in sorted(t.items(), key=lambda x: -x[1]["mean_time_us_under_ncu"] * x[1]["launches_captured"]):
            md.append(f"| {k} | {v['launches_captured']} | {v['mean_time_us_under_ncu']:.1f} | "
                      f"{v['dram_bytes_per_launch'] / 1e6:.1f} | {v['dram_throughput_pct']:.1f} | "
                      f"{v['tensor_pipe_pct']:.1f} | {v['issue_active_pct']:.1f} | {v['registers']:.0f} |")
        md.append("")
    open(os.path.join(OUT, f"{tag}_ncu_summary.md"), "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
