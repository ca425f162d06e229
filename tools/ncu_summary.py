"""Summarise an ncu report (read here, no GPU): key SOL/pipe/stall metrics + top stall SASS."""
import collections
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.avg.per_cycle_active",
        "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
        "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum", "dram__bytes_read.sum",
        "dram__bytes_write.sum", "dram__bytes_read.sum.per_second", "lts__t_bytes.sum",
        "smsp__inst_executed.sum", "launch__grid_size", "sm__cycles_elapsed.avg"]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return {h: (v, u) for h, u, v in zip(r[0], r[1], r[2])}


def main(rep, top=25):
    d = raw(rep)
    print(f"== {rep}")
    for k in KEYS:
        if k in d:
            print(f"  {k:62s} {d[k][0]:>16s} {d[k][1]}")
    st = []
    for k, (v, u) in d.items():
        if "average_warps_issue_stalled" in k and k.endswith("per_issue_active.ratio"):
            try:
                st.append((float(v), k.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", "")))
            except ValueError:
                pass
    print("  stalls (warps per issue): " + ", ".join(f"{n}={v:.2f}" for v, n in sorted(st, reverse=True)[:8]))
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h = rows[1]
    data = [dict(zip(h, r)) for r in rows[2:] if len(r) == len(h)]
    tot = sum(float(x["Warp Stall Sampling (All Samples)"] or 0) for x in data) or 1
    mix = collections.Counter()
    for x in data:
        src = x["Source"].split()
        if not src:
            continue
        op = src[1] if src[0].startswith("@") else src[0]
        mix[op.split(".")[0]] += int(x["Instructions Executed"] or 0)
    T = sum(mix.values()) or 1
    print("  SASS mix (executed): " + ", ".join(f"{k} {v / T * 100:.1f}%" for k, v in mix.most_common(14)))
    print("  top stall instructions:")
    for x in sorted(data, key=lambda x: -float(x["Warp Stall Sampling (All Samples)"] or 0))[:top]:
        print(f"    {x['Address'][-5:]} {float(x['Warp Stall Sampling (All Samples)'] or 0) / tot * 100:5.1f}%  {x['Source'][:80]}")


if __name__ == "__main__":
    main(sys.argv[1], int(sys.argv[2]) if len(sys.argv) > 2 else 25)
