"""Summarise an ncu report (run here, no GPU needed): python scripts/ncu_summary.py rep.ncu-rep"""
import csv
import subprocess
import sys

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "sm__throughput.avg.pct",
        "smsp__issue_active.avg.pct", "launch__registers_per_thread", "sm__warps_active.avg.pct",
        "lts__throughput.avg.pct", "smsp__inst_executed.sum", "launch__grid_size", "launch__occupancy_limit",
        "l1tex__t_requests_pipe_lsu_mem_global_op_atom.sum", "lts__t_sectors_srcunit_tex_op_read.sum",
        "dram__throughput.avg.pct", "lts__t_sector_hit_rate.pct", "lts__t_sector_op_read_hit_rate.pct",
        "lts__t_sector_op_atom_hit_rate.pct", "lts__t_sectors_op_atom.sum", "lts__t_requests_op_atom.sum",
        "l1tex__t_sector_hit_rate.pct", "lts__t_sectors.sum", "dram__bytes.sum.per_second"]


def main(path):
    out = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True, stderr=subprocess.DEVNULL)
    rows = list(csv.reader(out.splitlines()))
    h, units, vals = rows[0], rows[1], rows[2]
    for name, u, v in zip(h, units, vals):
        if any(name.startswith(k) for k in WANT) and "peak_sustained_active" not in name[:0]:
            print(f"{name:70s} {v:>16s} {u}")
    print("-- stalls (warps per issue) --")
    for name, v in zip(h, vals):
        if "smsp__average_warps_issue_stalled" in name and name.endswith("per_issue_active.ratio"):
            try:
                if float(v) > 0.15:
                    print(f"{name.replace('smsp__average_warps_issue_stalled_', ''):60s} {v}")
            except ValueError:
                pass


if __name__ == "__main__":
    main(sys.argv[1])
