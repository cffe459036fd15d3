"""Summarise ncu reports (run on the dev box): profiles/ncu_summary.json + markdown table.

    python scripts/summarize_ncu.py r01
"""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
        "launch__grid_size", "launch__block_size", "launch__occupancy_limit_registers",
        "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
        "smsp__average_warps_issue_stalled_lg_throttle_per_issue_active.ratio",
        "l1tex__t_sectors_pipe_lsu_mem_local_op_st.sum", "lts__t_bytes.sum"]
SCALE = {"Gbyte": 1e9, "Mbyte": 1e6, "Kbyte": 1e3, "byte": 1.0, "Tbyte": 1e12}


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    h, u, v = rows[0], rows[1], rows[2]
    d = {}
    for i, k in enumerate(h):
        if k in KEYS:
            val = v[i].replace(",", "")
            try:
                x = float(val)
            except ValueError:
                continue
            if u[i] in SCALE:
                x *= SCALE[u[i]]
                d[k] = {"value": x, "unit": "byte"}
            else:
                d[k] = {"value": x, "unit": u[i]}
    return d


def main():
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    res = {}
    import glob
    reps = sorted(glob.glob(os.path.join(ROOT, "gpurun_out", f"prof_*_{tag}.ncu-rep")))
    for rep in reps:
        name = os.path.basename(rep)[len("prof_"):-len(f"_{tag}.ncu-rep")]
        key = name if name.startswith("acc") else "allreduce_loopback_" + name
        d = raw(rep)
        t = d["gpu__time_duration.sum"]["value"]
        t_s = t * 1e-6 if d["gpu__time_duration.sum"]["unit"] == "us" else t * 1e-9 if d["gpu__time_duration.sum"]["unit"] == "ns" else t * 1e-3
        rd, wr = d["dram__bytes_read.sum"]["value"], d["dram__bytes_write.sum"]["value"]
        res[key] = {"report": os.path.basename(rep), "tag": tag,
                    "dram_bytes_per_launch": int(rd + wr), "dram_read": int(rd), "dram_write": int(wr),
                    "duration_s_ncu": t_s, "dram_gbs_ncu": (rd + wr) / t_s / 1e9,
                    "metrics": {k: v["value"] for k, v in d.items()}}
    path = os.path.join(ROOT, "profiles", "ncu_summary.json" if tag == "r01" else f"ncu_summary_{tag}.json")
    json.dump(res, open(path, "w"), indent=1)
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main()
