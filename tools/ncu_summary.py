"""Summarise an ncu --set full capture of the fused kernel (no GPU needed):
  python tools/ncu_summary.py gpurun_out/prof_X.ncu-rep CONFIG_NAME [traffic.json] > ..._summary.md
Also merges the kernel's DRAM traffic per launch into traffic.json (default profiles/traffic.json)."""
import csv, io, json, os, subprocess, sys

rep, cfg = sys.argv[1], sys.argv[2]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
hdr, units, vals = rows[0], rows[1], rows[2]
get = lambda k: (vals[hdr.index(k)], units[hdr.index(k)]) if k in hdr else (None, None)
keys = ["Kernel Name", "gpu__time_duration.sum", "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "dram__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_st.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum",
        "sm__warps_active.avg.pct_of_peak_sustained_active",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
        "l1tex__m_xbar2l1tex_read_bytes.sum.pct_of_peak_sustained_elapsed",
        "lts__t_sectors_srcunit_tex_op_red.sum"]
print(f"# ncu --set full summary: {cfg} ({os.path.basename(rep)})\n")
print("| metric | value | unit |\n|---|---|---|")
for k in keys:
    v, u = get(k)
    if v is not None:
        print(f"| {k} | {v[:120]} | {u} |")
stalls = [(k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""), float(vals[i]))
          for i, k in enumerate(hdr) if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("per_issue_active.ratio")
          and vals[i] not in ("", None)]
stalls.sort(key=lambda t: -t[1])
print("\nTop warp stall reasons (warps per issue-active cycle):\n")
for k, v in stalls[:8]:
    print(f"- {k}: {v:.2f}")
rd, _ = get("dram__bytes_read.sum"); wr, u = get("dram__bytes_write.sum")
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
traffic = (float(rd) + float(wr)) * scale
path = sys.argv[3] if len(sys.argv) > 3 else os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))),
                                                         "profiles", "traffic.json")
d = json.load(open(path)) if os.path.exists(path) else {}
d[cfg] = traffic
json.dump(d, open(path, "w"), indent=1, sort_keys=True)
print(f"\nDRAM traffic per launch (read + write): {traffic/1e6:.1f} MB -> profiles/traffic.json[{cfg}]")
