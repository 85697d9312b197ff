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
        "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]


def one(path):
    rows = list(csv.reader(open(path)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {k: (vals[hdr.index(k)] + (" " + units[hdr.index(k)] if units[hdr.index(k)] else "")).strip()
            for k in KEYS if k in hdr}


def main():
    tag = sys.argv[1]
    out = {"tag": tag, "gpu": "NVIDIA B200", "note": "ncu --set full --clock-control none; one launch each, "
           "cold-cache, serialised (shares of a step, not bench numbers)"}
    for name in ("k1_c4", "k2_c4", "k1_c2a"):
        try:
            out[name] = one(f"gpurun_out/{tag}_{name}_raw.csv")
        except (OSError, IndexError):
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
