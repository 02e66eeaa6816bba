"""Summarise a round's ncu captures (gpurun_out/prof_<tag>/) into profiles/:
  <tag>_launch_shares.csv   per-kernel share of the bench step (ncu launch list; cold-cache, serialised)
  <tag>_kernel_traffic.json dram bytes read+write per launch, duration, dram %, occupancy per kernel
  <tag>_ncu_summary.txt     the same as text
"""
import csv
import json
import os
import subprocess
import sys
from collections import defaultdict

tag = sys.argv[1] if len(sys.argv) > 1 else "r2"
src = f"gpurun_out/prof_{tag}"
os.makedirs("profiles", exist_ok=True)


def short(name):
    for k, v in (("sort_hist_kernel", "fcm_sort_hist"), ("sort_scan_kernel", "fcm_sort_scan"),
                 ("sort_scatter_kernel", "fcm_sort_scatter"), ("sort_ghist_kernel", "fcm_sort_ghist"),
                 ("sort_onesweep_kernel", "fcm_sort_scatter")):
        if k in name:
            return v
    for k in ("speed_encode_kernel<unsigned int>", "speed_encode_kernel<unsigned long>",
              "speed_decode_kernel<unsigned int>", "speed_decode_kernel<unsigned long>",
              "spratio_encode_kernel", "spratio_decode_kernel", "dpratio_encode_kernel", "dpratio_decode_kernel",
              "fcm_hash_kernel", "fcm_match_kernel", "dp_find_roots_kernel", "dp_gather_roots_kernel", "fcm_verify_kernel",
              "dp_walk_nodes_kernel", "dp_gather_leaves_kernel", "dp_gather_nodes_kernel",
              "fcm_carry_merge_kernel", "fcm_summary_kernel", "DeviceRadixSortOnesweepKernel", "DeviceRadixSortHistogramKernel",
              "DeviceRadixSortExclusiveSumKernel", "write_header_kernel"):
        if k in name:
            return (k.replace("_kernel<unsigned int>", "_u32").replace("_kernel<unsigned long>", "_u64")
                    .replace("_kernel", ""))
    if "spratio_encode" in name or "spratio_decode" in name:
        return "spratio_encode" if "encode" in name else "spratio_decode"
    return None


# 1. launch list shares
rows = [r for r in csv.reader(open(os.path.join(src, "launches.csv"))) if len(r) > 10]
h = rows[0]
ki, vi = h.index("Kernel Name"), h.index("Metric Value")
tot = defaultdict(float)
cnt = defaultdict(int)
for r in rows[1:]:
    s = short(r[ki])
    if s:
        tot[s] += float(r[vi].replace(",", ""))
        cnt[s] += 1
allsum = sum(tot.values())
with open(f"profiles/{tag}_launch_shares.csv", "w") as f:
    f.write("kernel,launches,total_ns,share_of_library_time\n")
    for k, v in sorted(tot.items(), key=lambda kv: -kv[1]):
        f.write(f"{k},{cnt[k]},{v:.0f},{v / allsum:.4f}\n")

# 2. full-set captures: traffic per launch
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed.sum.pct_of_peak_sustained_elapsed", "launch__registers_per_thread", "launch__grid_size",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_st.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_st.sum",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active"]
UNIT = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1, "us": 1e-6, "ms": 1e-3, "ns": 1e-9, "s": 1.0,
        "usecond": 1e-6, "msecond": 1e-3, "nsecond": 1e-9}
traffic = {}
lines = []
for fn in sorted(os.listdir(src)):
    if not fn.endswith(".ncu-rep"):
        continue
    out = subprocess.run(["ncu", "-i", os.path.join(src, fn), "--page", "raw", "--csv"], capture_output=True,
                         text=True).stdout
    rr = list(csv.reader(out.splitlines()))
    if len(rr) < 3:
        continue
    hh, uu = rr[0], rr[1]
    ix = {x: i for i, x in enumerate(hh)}
    for r in rr[2:]:
        s = short(r[ix["Kernel Name"]])
        if not s:
            continue
        vals = {}
        for k in KEYS:
            if k in ix:
                v = float(r[ix[k]].replace(",", "") or 0)
                vals[k] = v * UNIT.get(uu[ix[k]], 1)
        b = vals.get("dram__bytes_read.sum", 0) + vals.get("dram__bytes_write.sum", 0)
        e = traffic.setdefault(f"{fn[5:-8]}:{s}", {"launches": 0, "dram_bytes": 0.0, "seconds": 0.0})
        e["launches"] += 1
        e["dram_bytes"] += b
        e["seconds"] += vals.get("gpu__time_duration.sum", 0)
        e["dram_pct"] = vals.get("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed")
        e["warps_active_pct"] = vals.get("sm__warps_active.avg.pct_of_peak_sustained_active")
        e["issue_pct"] = vals.get("sm__inst_executed.sum.pct_of_peak_sustained_elapsed")
        e["registers"] = vals.get("launch__registers_per_thread")
        e["grid"] = vals.get("launch__grid_size")
        # LSU global sectors per request (TMA bulk copies bypass the LSU: 0 requests → None)
        for op in ("ld", "st"):
            req = vals.get(f"l1tex__t_requests_pipe_lsu_mem_global_op_{op}.sum", 0)
            sec = vals.get(f"l1tex__t_sectors_pipe_lsu_mem_global_op_{op}.sum", 0)
            e[f"{op}_sectors_per_request"] = sec / req if req else None
        e["alu_pipe_pct"] = vals.get("sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active")
for k, e in traffic.items():
    e["dram_bytes_per_launch"] = e["dram_bytes"] / e["launches"]
    e["seconds_per_launch"] = e["seconds"] / e["launches"]
    lines.append(f"{k:55s} launches={e['launches']} dram/launch={e['dram_bytes_per_launch'] / 1e6:9.2f} MB "
                 f"t/launch={e['seconds_per_launch'] * 1e6:9.1f} us dram%={e['dram_pct']:.1f} "
                 f"warps_active%={e['warps_active_pct']:.1f} issue%={e['issue_pct']:.1f} regs={e['registers']:.0f} "
                 f"alu%={(e.get('alu_pipe_pct') or 0):.1f} "
                 f"ld_sec/req={'-' if e.get('ld_sectors_per_request') is None else format(e['ld_sectors_per_request'], '.1f')} "
                 f"st_sec/req={'-' if e.get('st_sectors_per_request') is None else format(e['st_sectors_per_request'], '.1f')}")
json.dump(traffic, open(f"profiles/{tag}_kernel_traffic.json", "w"), indent=1)
with open(f"profiles/{tag}_ncu_summary.txt", "w") as f:
    f.write("# ncu --set full, one capture per kernel family on the bench workload (cold cache, serialised)\n")
    f.write("\n".join(lines) + "\n\n# launch shares of the bench command (ncu launch list)\n")
    f.write(open(f"profiles/{tag}_launch_shares.csv").read())
print(open(f"profiles/{tag}_ncu_summary.txt").read())
