# summarize a k_update_tc ncu capture: SOL, stalls, top SASS lines
import csv, subprocess, sys
rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(raw.splitlines())); h = r[0]; d = dict(zip(h, r[2]))
for k in ["gpu__time_duration.sum", "sm__cycles_elapsed.avg", "smsp__issue_active.avg.pct_of_peak_sustained_active",
          "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed" ,
          "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
          "dram__bytes_read.sum", "dram__bytes_write.sum", "smsp__cycles_active.avg"]:
    print(f"{k:75s} {d.get(k)}")
for k in h:
    if "tensor" in k and "pct" in k and d.get(k) not in (None, "", "0"):
        print(f"{k:75s} {d.get(k)}")
st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): float(v or 0) for k, v in d.items()
      if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
tot = sum(st.values())
print("stalls:", ", ".join(f"{k}={v/tot:.3f}" for k, v in sorted(st.items(), key=lambda x: -x[1])[:8]))
sass = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"], capture_output=True, text=True).stdout
rows = list(csv.reader(sass.splitlines())); h = rows[1]; data = [dict(zip(h, x)) for x in rows[2:]]
tot = sum(float(x["Warp Stall Sampling (All Samples)"] or 0) for x in data)
idx = sorted(range(len(data)), key=lambda i: -float(data[i]["Warp Stall Sampling (All Samples)"] or 0))[:int(sys.argv[2]) if len(sys.argv) > 2 else 25]
for i in sorted(idx):
    x = data[i]
    print(i, f"{float(x['Warp Stall Sampling (All Samples)'])/tot:.3f}", x["Source"][:80], x["Instructions Executed"])
