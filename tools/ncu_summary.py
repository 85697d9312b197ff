"""Summarise ncu raw CSV exports (tools/profile.sh) into one JSON for profiles/:
python tools/ncu_summary.py TAG > profiles/TAG_ncu_summary.json"""
import csv
import json
import sys

KEYS = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "smsp__issue_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread", "launch__grid_size",
        "launch__block_size", "smsp__inst_executed.sum",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum",
        # sector accounting (north_star: "sector-per-request counters").  The stream
        # loads are TMA bulk copies (UBLKCP), not LSU loads, so the LSU
        # sectors/request pair below counts only the report phase's few LDGs;
        # the L2 / DRAM sector counts are the meaningful efficiency measure.
        "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum",
        "lts__t_sectors_srcunit_tex_op_read.sum", "lts__t_sectors_op_read.sum", "lts__t_requests_op_read.sum",
        "dram__sectors_read.sum", "lts__t_sector_hit_rate.pct"]


def one(path):
    rows = list(csv.reader(open(path)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {k: (vals[hdr.index(k)] + (" " + units[hdr.index(k)] if units[hdr.index(k)] else "")).strip()
            for k in KEYS if k in hdr}


def main():
    tag = sys.argv[1]
    out = {"tag": tag, "gpu": "NVIDIA B200", "note": "ncu --set full --clock-control none; one launch each, "
           "cold-cache, serialised (shares of a step, not bench numbers)"}
    for name in ("k1_c4", "k2_c4", "k1_c2a", "k1_c2b", "k1_c3", "k1_c5"):
        try:
            out[name] = one(f"gpurun_out/{tag}_{name}_raw.csv")
        except (OSError, IndexError):
            continue
        k = out[name]
        try:  # derived: DRAM bytes / L2 read sectors vs 32-byte sectors of DRAM reads
            num = lambda s: float(s.split()[0].replace(",", ""))
            if "dram__sectors_read.sum" in k and "lts__t_sectors_srcunit_tex_op_read.sum" in k:
                # ~1.0: every 32-byte sector the SMs read through L2 came from DRAM exactly once
                k["derived_l2_tex_read_sectors_per_dram_read_sector"] = round(
                    num(k["lts__t_sectors_srcunit_tex_op_read.sum"]) / max(num(k["dram__sectors_read.sum"]), 1), 5)
                k["derived_dram_read_bytes_from_sectors"] = int(32 * num(k["dram__sectors_read.sum"]))
            if "lts__t_sectors_op_read.sum" in k and "lts__t_requests_op_read.sum" in k:
                k["derived_l2_sectors_per_request"] = round(
                    num(k["lts__t_sectors_op_read.sum"]) / max(num(k["lts__t_requests_op_read.sum"]), 1), 3)
            k["lsu_sectors_per_request_note"] = ("N/A for the stream: operands arrive by cp.async.bulk (UBLKCP, "
                                                 "TMA), which issues no LSU global loads; see the L2/DRAM sectors")
        except (ValueError, IndexError):
            pass
    try:  # per call: K1 (with the fused report phase), + K2 when it was a separate launch
        ks = [out[k] for k in ("k1_c4", "k2_c4") if k in out]
        b = lambda s: float(s.split()[0]) * {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1}[s.split()[1]]
        out["c4_dram_bytes_per_launch"] = int(sum(b(k[m]) for k in ks
                                                  for m in ("dram__bytes_read.sum", "dram__bytes_write.sum")))
    except (KeyError, ValueError, IndexError):
        pass
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
