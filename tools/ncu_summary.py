"""Summarise an ncu report (raw page) into a small JSON for profiles/ (run here, no GPU needed)."""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "duration_s": "gpu__time_duration.sum",
    "registers_per_thread": "launch__registers_per_thread",
    "grid": "launch__grid_size",
    "block": "launch__block_size",
    "occupancy_limit_registers": "launch__occupancy_limit_registers",
    "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "fmaheavy_pipe_pct_elapsed": "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "fma_pipe_pct_active": "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "alu_pipe_pct_active": "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "inst_executed": "smsp__inst_executed.sum",
    "dram_read_bytes": "dram__bytes_read.sum",
    "dram_write_bytes": "dram__bytes_write.sum",
    "sm_clock_hz": "sm__cycles_elapsed.avg.per_second",
    "warps_eligible_per_cycle": "smsp__warps_eligible.avg.per_cycle_active",
    "stall_wait": "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
    "stall_math_pipe_throttle": "smsp__average_warps_issue_stalled_math_pipe_throttle_per_issue_active.ratio",
    "stall_dispatch": "smsp__average_warps_issue_stalled_dispatch_stall_per_issue_active.ratio",
    "stall_not_selected": "smsp__average_warps_issue_stalled_not_selected_per_issue_active.ratio",
    "stall_short_scoreboard": "smsp__average_warps_issue_stalled_short_scoreboard_per_issue_active.ratio",
    "stall_long_scoreboard": "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "local_load_inst": "smsp__sass_inst_executed_op_local_ld.sum",
    "fmaheavy_pipe_pct_active": "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_active",
    "alu_inst_pct_active": "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
    "stall_barrier": "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "warps_active_per_scheduler": "smsp__warps_active.avg.per_cycle_active",
    "dram_throughput_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k, m in KEYS.items():
            if m in hdr:
                v = r[hdr.index(m)]
                u = units[hdr.index(m)]
                try:
                    x = float(v.replace(",", ""))
                except ValueError:
                    x = v
                scale = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1, "s": 1, "ms": 1e-3, "us": 1e-6,
                         "ns": 1e-9, "Ghz": 1e9, "Mhz": 1e6, "hz": 1}.get(u, 1)
                d[k] = x * scale if isinstance(x, float) else x
        res.append(d)
    return res


def sass_mix(rep, kernel_regex):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k",
                          "regex:" + kernel_regex], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = rows[1]
    ia, isrc = hdr.index("Instructions Executed"), hdr.index("Source")
    cnt, total = {}, 0
    for r in rows[2:]:
        try:
            n = int(r[ia])
        except (ValueError, IndexError):
            continue
        toks = r[isrc].split()
        if not toks:
            continue
        op = toks[1] if toks[0].startswith("@") else toks[0]
        cnt[op] = cnt.get(op, 0) + n
        total += n
    top = sorted(cnt.items(), key=lambda kv: -kv[1])[:14]
    return {op: round(100.0 * n / total, 2) for op, n in top}


if __name__ == "__main__":
    rep = sys.argv[1]
    res = raw(rep)
    if len(sys.argv) > 2:
        res.append({"sass_mix_pct_of_warp_instructions": sass_mix(rep, sys.argv[2])})
    print(json.dumps(res, indent=1))
