"""Summarise an ncu report: per kernel duration, IPC, occupancy, DRAM bytes,
registers and the top warp-stall reasons (reads `ncu -i X --page raw --csv`).

    python tools/ncu_summary.py gpurun_out/p_x.ncu-rep [--json out.json]
"""
import csv
import io
import json
import subprocess
import sys

METRICS = {
    "dur_us": "gpu__time_duration.sum",
    "ipc": "sm__inst_executed.avg.per_cycle_active",
    "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "dram_read": "dram__bytes_read.sum",
    "dram_write": "dram__bytes_write.sum",
    "regs": "launch__registers_per_thread",
    "grid": "launch__grid_size",
    "block": "launch__block_size",
    "smem_dyn": "launch__shared_mem_per_block_dynamic",
    "fp64_pipe_pct": "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active",
    "dmma_pipe_pct": "sm__inst_executed_pipe_tensor_subpipe_dmma.avg.pct_of_peak_sustained_active",
    "tensor_pipe_pct": "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "fp64_pipe_realtime_pct": "TPC.TriageCompute.sm__pipe_fp64_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "dfma_thread_inst_x2": "derived__sm__sass_thread_inst_executed_op_dfma_pred_on_x2",
    "inst_executed": "inst_executed",
    "l2_hit": "lts__t_sector_hit_rate.pct",
}
_TIME = {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3, "second": 1e6, "s": 1e6}
_BYTES = {"byte": 1, "B": 1, "Kbyte": 1e3, "KB": 1e3, "Mbyte": 1e6, "MB": 1e6, "Gbyte": 1e9, "GB": 1e9}


def load(path):
    out = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        u = dict(zip(hdr, units))
        rec = {"kernel": d.get("Kernel Name", "")[:60]}
        for k, m in METRICS.items():
            v = d.get(m, "")
            try:
                x = float(v.replace(",", ""))
            except ValueError:
                continue
            unit = u.get(m, "")
            if k == "dur_us":        # always microseconds, whatever unit ncu printed
                x = x * _TIME.get(unit, 1.0)
            if k.startswith("dram_"):
                x = x * _BYTES.get(unit, 1)
            rec[k] = x
        st = [(k.replace("smsp__pcsamp_warps_issue_stalled_", ""), float(v.replace(",", "")))
              for k, v in d.items()
              if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued")
              and v.replace(",", "").replace(".", "").isdigit()]
        tot = sum(v for _, v in st) or 1.0
        rec["stalls"] = {k: round(100 * v / tot, 1) for k, v in sorted(st, key=lambda kv: -kv[1])[:6]}
        res.append(rec)
    return res


if __name__ == "__main__":
    recs = load(sys.argv[1])
    for r in recs:
        print(r["kernel"][:40], {k: (round(v, 3) if isinstance(v, float) else v) for k, v in r.items()
                                 if k not in ("kernel", "stalls")})
        print("    stalls", r["stalls"])
    if "--json" in sys.argv:
        with open(sys.argv[sys.argv.index("--json") + 1], "w") as f:
            json.dump(recs, f, indent=1)
