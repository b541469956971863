"""Summarise an ncu report (raw page) into the metrics this project tracks."""
import csv
import subprocess
import sys

WANT = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__t_sectors_srcunit_tex_op_read.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
        "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_sector_hit_rate.pct",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "lts__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__warp_issue_stalled_long_scoreboard_per_warp_active.pct",
        "smsp__warp_issue_stalled_lg_throttle_per_warp_active.pct",
        "lts__t_sectors_op_atom.sum", "lts__t_sectors_op_red.sum", "lts__t_sectors_op_write.sum"]


STALL_PREFIX = "smsp__average_warps_issue_stalled_"
STALL_SUFFIX = "_per_issue_active.ratio"


def main(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(raw.splitlines()))
    hdr, units, data = rows[0], rows[1], rows[2:]
    for r in data:
        print(r[hdr.index("Kernel Name")][:70])
        for w in WANT:
            if w in hdr:
                print(f"    {w:75s} {r[hdr.index(w)]:>22s} {units[hdr.index(w)]}")
        # stall breakdown: cycles between issues by reason (the dependent-load chain
        # shows up as long_scoreboard), largest first
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith(STALL_PREFIX) and h.endswith(STALL_SUFFIX):
                try:
                    stalls.append((float(r[i].replace(",", "")), h[len(STALL_PREFIX):-len(STALL_SUFFIX)]))
                except ValueError:
                    pass
        tot = sum(v for v, _ in stalls) or 1.0
        print("    stall cycles per issued instruction (share):")
        for v, name in sorted(stalls, reverse=True)[:6]:
            print(f"        {name:30s} {v:8.2f}  ({100 * v / tot:4.1f}%)")


if __name__ == "__main__":
    main(sys.argv[1])
