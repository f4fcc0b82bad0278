"""Summarise an ncu report (raw page) into the metrics we track (run here, no GPU)."""
import csv
import io
import json
import subprocess
import sys

KEYS = {
    "gpu__time_duration.sum": "duration",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "lts__t_sectors_srcunit_tex_op_red.sum": "l2_red_sectors",
    "lts__t_sector_hit_rate.pct": "l2_hit_pct",
    "l1tex__t_sector_hit_rate.pct": "l1_hit_pct",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum": "smem_wavefronts",
    "l1tex__data_pipe_lsu_wavefronts.sum": "lsu_wavefronts",
    "smsp__inst_executed.sum": "warp_inst",
    "sm__cycles_elapsed.avg": "sm_cycles",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "occupancy_pct",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "l1tex__throughput.avg.pct_of_peak_sustained_active": "l1tex_pct",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_pct",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed": "dram_pct",
    "launch__registers_per_thread": "regs",
    "launch__shared_mem_per_block_dynamic": "smem_dyn",
    "launch__block_size": "block",
    "launch__grid_size": "grid",
    "lts__t_bytes.sum": "l2_bytes",
    "l1tex__m_xbar2l1tex_read_bytes.sum": "l2_to_l1_bytes",
}


def summarise(rep):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        rec = {"kernel": d.get("Kernel Name", "")[:80]}
        for k, name in KEYS.items():
            if k in d:
                v = d[k].replace(",", "")
                try:
                    v = float(v)
                except ValueError:
                    pass
                rec[name] = v
                rec[name + "_unit"] = units[hdr.index(k)]
        stalls = {}
        for k in hdr:
            if k.startswith("smsp__average_warps_issue_stalled_") and k.endswith("_per_issue_active.ratio"):
                try:
                    v = float(d[k].replace(",", ""))
                except ValueError:
                    continue
                if v > 0.05:
                    stalls[k[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]] = round(v, 3)
        rec["stalls"] = stalls
        out.append(rec)
    return out


if __name__ == "__main__":
    for rec in summarise(sys.argv[1]):
        print(json.dumps(rec))
