"""Summarise an ncu report of the EP kernel (development + profiles/ aid).

python tools/ncu_summary.py gpurun_out/<tag>_prof.ncu-rep [--json out.json]
"""
import csv, io, json, subprocess, sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "sm__cycles_elapsed.avg": "cycles",
    "sm__cycles_elapsed.avg.per_second": "sm_clock",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active": "fp64_pipe_pct",
    "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active": "fp64_inst_pct",
    "sm__issue_active.avg.pct_of_peak_sustained_elapsed": "issue_active_pct",
    "sm__inst_executed.sum": "inst_executed",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active": "alu_pct",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active": "fma_pct",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active": "xu_pct",
    "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active": "lsu_pct",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed": "smem_wavefront_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
    "launch__registers_per_thread": "registers",
    "launch__block_size": "block",
    "launch__grid_size": "grid",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "sm__sass_thread_inst_executed_op_dfma_pred_on.sum": "dfma_thread",
    "sm__sass_thread_inst_executed_op_dmul_pred_on.sum": "dmul_thread",
    "sm__sass_thread_inst_executed_op_dadd_pred_on.sum": "dadd_thread",
    "smsp__thread_inst_executed_per_inst_executed.ratio": "threads_per_inst",
}
STALL = "smsp__average_warps_issue_stalled_"


def to_float(v):
    try:
        return float(v.replace(",", ""))
    except Exception:
        return None


def main():
    rep = sys.argv[1]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        if "ep_kernel" not in " ".join(r):
            continue
        d = {"kernel": next((x for x in r if "ep_kernel" in x), "")}
        stalls = {}
        for h, u, v in zip(hdr, units, r):
            if h in KEYS:
                f = to_float(v)
                d[KEYS[h]] = f if f is not None else v
                if u:
                    d[KEYS[h] + "_unit"] = u
            if h.startswith(STALL) and h.endswith("_per_issue_active.ratio"):
                f = to_float(v)
                if f and f > 0.05:
                    stalls[h[len(STALL):-len("_per_issue_active.ratio")]] = round(f, 3)
        d["stalls_per_issue"] = dict(sorted(stalls.items(), key=lambda kv: -kv[1]))
        out.append(d)
    js = json.dumps(out, indent=1)
    print(js)
    if "--json" in sys.argv:
        open(sys.argv[sys.argv.index("--json") + 1], "w").write(js)


if __name__ == "__main__":
    main()
