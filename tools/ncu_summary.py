"""Summarise an ncu report into the JSON kept under profiles/ (tool).

    python tools/ncu_summary.py gpurun_out/prof_fill.ncu-rep profiles/r01_fill_ncu.json
Needs the `ncu` CLI (present in the build container and on the GPU box).
"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "launch__block_size",
    "launch__grid_size", "launch__registers_per_thread", "launch__occupancy_limit_registers",
    "launch__occupancy_limit_shared_mem", "launch__shared_mem_per_block_static",
    "sm__cycles_elapsed.avg.per_second", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "lts__t_sector_hit_rate.pct",
    "smsp__inst_executed.sum", "sm__cycles_elapsed.avg", "smsp__inst_executed_op_shared_ld.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared_op_ld.sum",
    "l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum",
]
STALLS = "smsp__pcsamp_warps_issue_stalled_"


def main(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], check=True,
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    head, units, vals = rows[0], rows[1], rows[2]
    res = {}
    for i, k in enumerate(head):
        if k in KEYS or k.startswith(STALLS):
            v = vals[i]
            try:
                v = float(v.replace(",", ""))
            except ValueError:
                pass
            res[k] = {"value": v, "unit": units[i]}
    res["_source"] = {"report": rep, "command": "ncu --set full --clock-control none "
                      "--import-source on (one launch)"}
    with open(out, "w") as f:
        json.dump(res, f, indent=1)
    print(json.dumps({k: res[k]["value"] for k in res if not k.startswith(("_", STALLS))},
                     indent=0))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
