"""Summarise an ncu --set full report (read with `ncu -i ... --page raw --csv`)
into a small JSON kept under profiles/ (the .ncu-rep itself stays in gpurun_out/).

    python tools/ncu_summary.py gpurun_out/prof.ncu-rep profiles/r01_ncu_sampler.json
"""
import csv
import io
import json
import subprocess
import sys

METRICS = {
    "gpu__time_duration.sum": "duration_ms",
    "dram__bytes_read.sum": "dram_read",
    "dram__bytes_write.sum": "dram_write",
    "lts__t_bytes.sum": "l2_bytes",
    "sm__cycles_active.avg": "sm_active_cycles",
    "sm__cycles_elapsed.avg": "sm_elapsed_cycles",
    "smsp__issue_active.avg.pct_of_peak_sustained_active": "issue_active_pct",
    "sm__warps_active.avg.per_cycle_active": "warps_active_per_sm",
    "smsp__inst_executed.sum": "warp_instructions",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active": "fma_pipe_pct",
    "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active": "alu_pipe_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "sm__maximum_warps_per_active_cycle_pct": "theoretical_occupancy_pct",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "achieved_occupancy_pct",
}


def to_bytes(v, unit):
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}
    return v * scale.get(unit, 1)


def main(rep, out):
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    head, units = rows[0], rows[1]
    launches = []
    for r in rows[2:]:
        d = {"kernel": r[head.index("Kernel Name")][:120]}
        for m, k in METRICS.items():
            if m in head:
                i = head.index(m)
                try:
                    v = float(r[i].replace(",", ""))
                except ValueError:
                    continue
                u = units[i]
                if k.startswith("dram") or k == "l2_bytes":
                    v = to_bytes(v, u)
                if k == "duration_ms":
                    v = v / 1e6 if u in ("nsecond", "ns") else (v / 1e3 if u in ("usecond", "us") else v)
                d[k] = v
        if "dram_read" in d and "dram_write" in d:
            d["dram_bytes"] = d["dram_read"] + d["dram_write"]
        launches.append(d)
    json.dump({"report": rep, "launches": launches}, open(out, "w"), indent=1)
    print(json.dumps(launches, indent=1)[:3000])


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2])
