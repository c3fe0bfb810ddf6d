"""Per-kernel ncu counters the north_star asks every design choice to be evidenced by (instructions per
event, atomic traffic, achieved DRAM GB/s), normalised per unit of work, as JSON.
usage: ncu_counters.py report.ncu-rep name=units [name=units ...] > out.json
(`name` is a substring of the kernel name; `units` the events that one launch of it processes)."""
import csv
import io
import json
import subprocess
import sys

M = {
    "time_ms": ("gpu__time_duration.sum", 1e-6),          # ncu reports ns here; scaled below by unit
    "warp_inst": ("smsp__inst_executed.sum", 1),
    "issue_active_pct": ("smsp__issue_active.avg.pct_of_peak_sustained_active", 1),
    "dram_read_bytes": ("dram__bytes_read.sum", 1),
    "dram_write_bytes": ("dram__bytes_write.sum", 1),
    "shared_atomic_wavefronts": ("l1tex__data_pipe_lsu_wavefronts_mem_shared_op_atom.sum", 1),
    "global_atomic_sectors": ("l1tex__m_l1tex2xbar_write_sectors_mem_global_op_atom.sum", 1),
    "global_red_sectors": ("l1tex__m_l1tex2xbar_write_sectors_mem_global_op_red.sum", 1),
}
SCALE = {"ns": 1e-6, "us": 1e-3, "ms": 1.0, "s": 1e3, "byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9,
         "inst": 1, "%": 1, "": 1, "sector": 1}


def main(rep, specs):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    res = {}
    for row in data:
        name = row[hdr.index("Kernel Name")]
        for spec in specs:
            key, n = spec.split("=")
            if key not in name or key in res:
                continue
            d = {"kernel": name[:90], "units_per_launch": float(n)}
            for k, (metric, _) in M.items():
                if metric not in hdr:
                    continue
                i = hdr.index(metric)
                v = float(row[i].replace(",", "") or 0) * SCALE.get(units[i], 1)
                d[k] = v
            u = float(n)
            d["warp_inst_per_unit"] = d["warp_inst"] / u
            d["dram_bytes_per_unit"] = (d["dram_read_bytes"] + d["dram_write_bytes"]) / u
            d["dram_gbs"] = (d["dram_read_bytes"] + d["dram_write_bytes"]) / (d["time_ms"] * 1e-3) / 1e9
            d["shared_atomic_wavefronts_per_unit"] = d.get("shared_atomic_wavefronts", 0) / u
            d["global_atomic_sectors_per_unit"] = (d.get("global_atomic_sectors", 0) + d.get("global_red_sectors", 0)) / u
            res[key] = d
    print(json.dumps(res, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2:])
