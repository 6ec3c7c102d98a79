"""Summarise gpurun_out ncu captures into profiles/ (launch list, traffic.json, summary)."""
import csv, io, json, os, re, subprocess, sys, collections
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
out = os.environ.get("PROFILES_OUT", os.path.join(ROOT, "profiles"))
os.makedirs(out, exist_ok=True)

def kname(full):
    m = re.search(r"rowgemm(?:_bf16)?_kernel<(?:\(int\))?(\d+), (?:\(int\))?(\d+)", full)
    if m:
        return ["node_tc", "edge_tc", "gate_tc", "plain_tc", "gatebwd_tc", "edgebwd_tc",
                "gateagg_tc"][int(m.group(2))]
    for k, v in [("synth_kernel", "synthesize"), ("set_decoder_pool", "set_decoder_pool"),
                 ("gph_attn", "gph_attn"), ("gph_ln", "gph_ln"), ("set_decoder_prep", "set_decoder_prep"),
                 ("set_decoder_kernel", "set_decoder"), ("gather_segsoftmax", "gather_segsoftmax"),
                 ("edgegate", "edge_gate_tc"), ("edge_small", "edge_small"), ("wgrad_tc", "wgrad_tc"), ("wimage", "wimage"),
                 ("split_reduce", "split_reduce"), ("agg_fixup", "agg_fixup"),
                 ("wgrad_skinny", "wgrad_skinny"), ("gather_segsum", "gather_segsum"),
                 ("readout_head", "readout_head"), ("permute_rows", "permute_e0"),
                 ("node_gemm_kernel", "node_gemm"), ("edge_fwd_kernel", "edge_fwd"),
                 ("edge_bwd_m", "edge_bwd_m"), ("edge_bwd_e", "edge_bwd_e"), ("node_bwd", "node_bwd"),
                 ("wgrad_partial", "wgrad_partial"), ("wgrad_reduce", "wgrad_reduce"),
                 ("head_bwd_graph", "head_bwd_graph"), ("head_bwd_reduce", "head_bwd_reduce"),
                 ("broadcast_dh", "broadcast_dh"), ("adam", "adam")]:
        if k in full:
            return v
    return full[:40]

# 1) launch list
lp = os.path.join(ROOT, "gpurun_out", "launches.csv")
if os.path.exists(lp):
    txt = open(lp).read()
    rows = list(csv.reader(io.StringIO(txt[txt.index('"ID"'):])))
    hdr = rows[0]
    iK, iM, iV = hdr.index("Kernel Name"), hdr.index("Metric Name"), hdr.index("Metric Value")
    iID = hdr.index("ID")
    per = collections.OrderedDict()
    for r in rows[1:]:
        d = per.setdefault(r[iID], {"kernel": r[iK]})
        d[r[iM]] = float(r[iV].replace(",", ""))
    with open(os.path.join(out, f"{tag}_launches.csv"), "w") as f:
        f.write("id,kernel,class,gpu_time_ns,dram_read_bytes,dram_write_bytes\n")
        for i, d in per.items():
            f.write(f"{i},\"{d['kernel'][:80]}\",{kname(d['kernel'])},{d.get('gpu__time_duration.sum',0):.0f},"
                    f"{d.get('dram__bytes_read.sum',0):.0f},{d.get('dram__bytes_write.sum',0):.0f}\n")
    agg = collections.defaultdict(lambda: [0, 0.0, 0.0])
    for d in per.values():
        a = agg[kname(d["kernel"])]
        a[0] += 1
        a[1] += d.get("gpu__time_duration.sum", 0)
        a[2] += d.get("dram__bytes_read.sum", 0) + d.get("dram__bytes_write.sum", 0)
    tot = sum(a[1] for a in agg.values())
    print("launch list: class, launches, share of time, mean dram bytes/launch")
    for k, a in sorted(agg.items(), key=lambda x: -x[1][1]):
        print(f"  {k:16s} {a[0]:4d} {100*a[1]/tot:6.1f}% {a[2]/a[0]/1e6:9.1f} MB")

# 2) full capture -> traffic per launch for the hot kernels
def capture(reps):
 traffic = {}
 for rep, drv in reps:
  fp = os.path.join(ROOT, "gpurun_out", rep + ".ncu-rep")
  if os.path.exists(fp):
      raw = subprocess.run(["ncu", "-i", fp, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
      rows = list(csv.reader(io.StringIO(raw)))
      hdr = rows[0]
      def g(r, k):
          try:
              return float(r[hdr.index(k)].replace(",", ""))
          except Exception:
              return None
      acc = collections.defaultdict(list)
      for r in rows[2:]:
          k = kname(r[hdr.index("Kernel Name")])
          unit_r = rows[1][hdr.index("dram__bytes_read.sum")]
          scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(unit_r, 1)
          acc[k].append({
              "time_us": g(r, "gpu__time_duration.sum"),
              "dram_bytes": (g(r, "dram__bytes_read.sum") + g(r, "dram__bytes_write.sum")) * scale,
              "dram_pct": g(r, "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"),
              "tensor_pct": g(r, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed"),
              "issue_pct": g(r, "smsp__issue_active.avg.pct_of_peak_sustained_active"),
              "regs": g(r, "launch__registers_per_thread"),
          })
      for k, lst in acc.items():
          n = len(lst)
          traffic[k] = {"dram_bytes_per_launch": sum(x["dram_bytes"] for x in lst) / n,
                        "launches_captured": n,
                        "mean_time_us_under_ncu": sum(x["time_us"] or 0 for x in lst) / n,
                        "dram_throughput_pct": sum(x["dram_pct"] or 0 for x in lst) / n,
                        "tensor_pipe_pct": sum(x["tensor_pct"] or 0 for x in lst) / n,
                        "issue_active_pct": sum(x["issue_pct"] or 0 for x in lst) / n,
                        "registers": lst[0]["regs"],
                        "source": f"profiles/{tag}: ncu --set full, {drv}"}
  # (end of one capture)
 return traffic

traffic = capture((("prof_full", "scripts/prof_driver.py (CFG2 inference)"),
                   ("prof_train", "scripts/prof_driver.py --train (CFG2 training)")))
traffic_bf = capture((("prof_bf16", "scripts/prof_driver.py --bf16 (CFG2 inference, OCCU_BF16)"),))
traffic_nx = capture((("prof_next", "scripts/prof_driver.py --graphormer 2 --decoder (CFG2 inference, NEXT-2/3)"),))
if traffic_nx:
    json.dump(traffic_nx, open(os.path.join(out, "traffic_next.json"), "w"), indent=1)
json.dump(traffic, open(os.path.join(out, "traffic.json"), "w"), indent=1)
if traffic_bf:
    json.dump(traffic_bf, open(os.path.join(out, "traffic_bf16.json"), "w"), indent=1)
with open(os.path.join(out, f"{tag}_ncu_summary.md"), "w") as f:
  for title, traffic in (("OCCU_FP32 (inference + training)", traffic), ("OCCU_BF16 inference", traffic_bf),
                         ("NEXT-2/3/4 kernels: Graphormer x2 + decoder readout + on-device synthesis, OCCU_FP32 inference", traffic_nx)):
    if not traffic:
        continue
    f.write(f"# {tag}: ncu --set full --clock-control none (serialised, cold-cache replays), {title}\n\n")
    f.write("| kernel | launches | us/launch (ncu) | DRAM MB/launch | DRAM % peak | tensor pipe % | issue active % | regs |\n")
    f.write("|---|---|---|---|---|---|---|---|\n")
    for k, t in traffic.items():
        f.write(f"| {k} | {t['launches_captured']} | {t['mean_time_us_under_ncu']:.1f} | "
                f"{t['dram_bytes_per_launch']/1e6:.1f} | {t['dram_throughput_pct']:.1f} | "
                f"{t['tensor_pipe_pct']:.1f} | {t['issue_active_pct']:.1f} | {t['registers']:.0f} |\n")
print(open(os.path.join(out, f"{tag}_ncu_summary.md")).read())
