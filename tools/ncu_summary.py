"""Summarise an ncu report: key throughput metrics, stall reasons and the SASS opcode mix."""
import collections
import csv
import io
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__grid_size",
        "sm__inst_executed_pipe_alu.sum.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_fma.sum.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.sum.pct_of_peak_sustained_active", "sm__inst_executed.sum",
        "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "smsp__average_warps_issue_stalled_", "smsp__pcsamp_warps_issue_stalled_"]


def raw(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2]


def main(rep):
    h, u, v = raw(rep)
    print("==", rep)
    stalls = []
    for i, name in enumerate(h):
        if any(name.startswith(k) for k in KEYS[:14]) and not name.endswith("per_second"):
            print(f"  {name} = {v[i]} {u[i]}")
        if name.startswith("smsp__average_warps_issue_stalled_") and name.endswith("_per_issue_active.ratio"):
            try:
                stalls.append((float(v[i]), name.replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", "")))
            except ValueError:
                pass
    print("  stalls per issue:", ", ".join(f"{n}={x:.2f}" for x, n in sorted(stalls, reverse=True)[:8]))
    src = subprocess.check_output(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                                  stderr=subprocess.DEVNULL).decode()
    rows = list(csv.reader(io.StringIO(src)))
    hdr = rows[1]
    ie, sc = hdr.index("Instructions Executed"), hdr.index("Source")
    cnt = collections.Counter()
    tot = 0
    for r in rows[2:]:
        try:
            n = int(r[ie])
        except (ValueError, IndexError):
            continue
        toks = r[sc].split()
        if not toks:
            continue
        op = toks[1] if toks[0].startswith("@") else toks[0]
        cnt[op.split(".")[0]] += n
        tot += n
    print(f"  warp instructions {tot:.4g}; mix:", ", ".join(f"{k} {c/tot*100:.1f}%" for k, c in cnt.most_common(16)))
    return tot


if __name__ == "__main__":
    for rep in sys.argv[1:]:
        main(rep)
