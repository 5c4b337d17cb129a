"""Summarise an ncu --set full report: per kernel launch duration, throughputs,
occupancy, DRAM bytes and the top warp-stall reasons (B200_PROFILING.md)."""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h = rows[0]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
        "launch__registers_per_thread", "launch__grid_size", "lts__t_sector_hit_rate.pct",
        "smsp__thread_inst_executed_per_inst_executed.ratio", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum", "smsp__inst_executed_op_branch.sum",
        "smsp__branch_targets_threads_divergent.sum", "lts__t_sectors_srcunit_tex_op_read.sum"]
idx = {w: h.index(w) for w in want if w in h}
stall = [i for i, c in enumerate(h) if c.startswith("smsp__average_warps_issue_stalled_") and c.endswith("_per_issue_active.ratio")]
ki = h.index("Kernel Name")
for r in rows[2:]:
    if len(r) < len(h):
        continue
    name = r[ki].split("(")[0].split("::")[-1]
    d = {w: r[i] for w, i in idx.items()}
    st = sorted(((float(r[i].replace(",", "") or 0), h[i].replace("smsp__average_warps_issue_stalled_", "").replace("_per_issue_active.ratio", "")) for i in stall), reverse=True)[:4]
    print(f"{name}: dur={d.get('gpu__time_duration.sum')} dramR={d.get('dram__bytes_read.sum')} dramW={d.get('dram__bytes_write.sum')} "
          f"dram%={d.get('dram__throughput.avg.pct_of_peak_sustained_elapsed')} l2%={d.get('lts__throughput.avg.pct_of_peak_sustained_elapsed')} "
          f"sm%={d.get('sm__throughput.avg.pct_of_peak_sustained_elapsed')} warps%={d.get('sm__warps_active.avg.pct_of_peak_sustained_active')} "
          f"regs={d.get('launch__registers_per_thread')} grid={d.get('launch__grid_size')} l2hit={d.get('lts__t_sector_hit_rate.pct')} "
          f"simt={d.get('smsp__thread_inst_executed_per_inst_executed.ratio')}")
    def num(k):
        try:
            return float(d.get(k, "").replace(",", ""))
        except ValueError:
            return None
    sec, req = num("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"), num("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")
    print(f"    dram%(gpu)={d.get('gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed')} "
          f"ld sectors/request={sec / req if sec and req else None} "
          f"atom requests={d.get('l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum')} "
          f"branches={d.get('smsp__inst_executed_op_branch.sum')} "
          f"divergent branch targets={d.get('smsp__branch_targets_threads_divergent.sum')} "
          f"L2 read sectors from L1={d.get('lts__t_sectors_srcunit_tex_op_read.sum')}")
    print("    stalls:", ", ".join(f"{n}={v:.1f}" for v, n in st))
