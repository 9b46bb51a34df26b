"""Print the headline metrics + stall breakdown + hottest SASS lines of an ncu report (per launch)."""
import csv, io, subprocess, sys

rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 25
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units = rows[0], rows[1]
keys = ["Kernel Name", "gpu__time_duration.sum", "launch__grid_size", "launch__registers_per_thread",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "l1tex__throughput.avg.pct_of_peak_sustained_active", "smsp__inst_executed.sum", "dram__bytes_read.sum",
        "lts__t_sector_hit_rate.pct"]
for r in rows[2:]:
    d = dict(zip(h, r))
    print("----")
    for k in keys:
        print(f"  {k:60s} {d.get(k, '?')[:90]}")
    st = [(k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", ""), float(v))
          for k, v in d.items() if k.startswith("smsp__average_warps_issue_stalled_") and v not in ("", "0")]
    st.sort(key=lambda x: -x[1])
    print("  stalls/issue:", ", ".join(f"{k}={v:.2f}" for k, v in st[:8]))
if top:
    src = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    lines = list(csv.reader(io.StringIO(src)))
    hdr = None
    block = []
    for r in lines:
        if r and r[0] == "Address":
            hdr = r
            continue
        if hdr and len(r) == len(hdr):
            block.append(r)
    if hdr:
        iss = hdr.index("Warp Stall Sampling (All Samples)")
        isrc = hdr.index("Source")
        iex = hdr.index("Instructions Executed")
        tot = sum(int(r[iss]) for r in block) or 1
        print(f"---- hottest SASS ({len(block)} instructions, {tot} samples)")
        for r in sorted(block, key=lambda r: -int(r[iss]))[:top]:
            print(f"  {100*int(r[iss])/tot:5.1f}% {int(r[iex]):>11}  {r[isrc].strip()}")
