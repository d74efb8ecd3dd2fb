"""Summarise an ncu report (raw page) for the kernels of interest: time, DRAM bytes, L2
atomic/reduction sectors, sectors per request, warp efficiency, top stall reasons."""
import csv
import re
import subprocess
import sys

KEYS = [
    ("gpu__time_duration.sum", "duration"),
    ("dram__bytes_read.sum", "dram_read"),
    ("dram__bytes_write.sum", "dram_write"),
    ("dram__throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct"),
    ("lts__throughput.avg.pct_of_peak_sustained_elapsed", "lts_pct"),
    ("lts__t_sectors_op_red.sum", "lts_red_sectors"),
    ("lts__t_sectors_op_atom.sum", "lts_atom_sectors"),
    ("lts__t_sectors_op_read.sum", "lts_read_sectors"),
    ("lts__t_sectors_op_write.sum", "lts_write_sectors"),
    ("lts__t_sector_hit_rate.pct", "l2_hit_pct"),
    ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1_ld_sectors"),
    ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "l1_ld_requests"),
    ("smsp__thread_inst_executed_per_inst_executed.ratio", "threads_per_inst"),
    ("sm__warps_active.avg.pct_of_peak_sustained_active", "occupancy_pct"),
    ("launch__registers_per_thread", "regs"),
    ("smsp__inst_executed.sum", "inst"),
]
STALL = re.compile(r"smsp__pcsamp_warps_issue_stalled_(\w+)$")


def load(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(out.splitlines()))
    return r[0], r[1], r[2:]


def summarize(rep, pattern=""):
    hdr, units, rows = load(rep)
    ki = hdr.index("Kernel Name")
    res = []
    for row in rows:
        if pattern and not re.search(pattern, row[ki]):
            continue
        d = {"kernel": row[ki][:80]}
        for k, short in KEYS:
            if k in hdr:
                v = row[hdr.index(k)].replace(",", "")
                try:
                    d[short] = float(v)
                except ValueError:
                    d[short] = v
                d[short + "_unit"] = units[hdr.index(k)]
        stalls = {}
        for i, h in enumerate(hdr):
            mm = STALL.match(h)
            if mm and not h.endswith("_not_issued"):
                try:
                    stalls[mm.group(1)] = float(row[i].replace(",", ""))
                except ValueError:
                    pass
        tot = sum(stalls.values()) or 1.0
        d["top_stalls"] = {k: round(100 * v / tot, 1) for k, v in sorted(stalls.items(), key=lambda x: -x[1])[:6]}
        res.append(d)
    return res


if __name__ == "__main__":
    import json
    for d in summarize(sys.argv[1], sys.argv[2] if len(sys.argv) > 2 else ""):
        print(json.dumps(d))
