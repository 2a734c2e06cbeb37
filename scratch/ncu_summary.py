import csv, subprocess, sys
rep = sys.argv[1]
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(out.splitlines())); h = r[0]
for row in r[2:]:
    d = dict(zip(h, row))
    print("kernel:", d.get("Kernel Name", "")[:60], "dur(ns):", d.get("gpu__time_duration.sum"))
    keys = ["sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__inst_executed.sum", "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
            "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__occupancy_limit_registers",
            "launch__occupancy_limit_shared_mem", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smsp__warps_eligible.avg.per_cycle_active"]
    for k in keys:
        print(f"  {k:70s} {d.get(k)}")
    st = {k.replace("smsp__pcsamp_warps_issue_stalled_", ""): v for k, v in d.items()
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")}
    tot = sum(float(v) for v in st.values() if v)
    print("  stalls:", ", ".join(f"{k}={float(v)/tot:.2f}" for k, v in sorted(st.items(), key=lambda x: -float(x[1] or 0))[:8]))
