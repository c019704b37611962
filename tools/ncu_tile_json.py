"""Write profiles/dgemm_tile_ncu.json (the numbers bench.py's roofline.traffic reads) from an
ncu --set full capture of one grouped dgemm_tma_kernel launch.
usage: python tools/ncu_tile_json.py report.ncu-rep T tasks_per_launch "command"."""
import csv
import io
import json
import subprocess
import sys

rep, T, tasks, cmd = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), sys.argv[4]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(raw)))
h, units, v = rows[0], rows[1], rows[2]
get = {n: (v[i], units[i]) for i, n in enumerate(h)}


def num(name, scale_to=None):
    val, unit = get[name]
    x = float(val.replace(",", ""))
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "msecond": 1e-3, "usecond": 1e-6, "nsecond": 1e-9,
            "second": 1.0, "ms": 1e-3, "us": 1e-6, "ns": 1e-9, "s": 1.0}
    return x * mult.get(unit, 1.0) if scale_to else x


rd, wr = num("dram__bytes_read.sum", True), num("dram__bytes_write.sum", True)
out = {
    "kernel": get["Kernel Name"][0] if "Kernel Name" in get else "dgemm_tma_kernel",
    "tile": T, "tasks_per_launch": tasks, "grid": int(num("launch__grid_size")),
    "block": int(num("launch__block_size")),
    "duration_ms_ncu": num("gpu__time_duration.sum", True) * 1e3,
    "dram_bytes_read": rd, "dram_bytes_write": wr, "dram_bytes_per_launch": rd + wr,
    "algorithmic_bytes_per_launch": 4 * 8 * T * T * tasks,
    "algorithmic_flops_per_launch": 2 * T ** 3 * tasks,
    "dmma_pipe_active_pct": num("sm__pipe_tensor_subpipe_dmma_cycles_active.avg.pct_of_peak_sustained_active"),
    "l2_hit_pct": num("lts__t_sector_hit_rate.pct"),
    "registers": int(num("launch__registers_per_thread")),
    "source": cmd,
}
print(json.dumps(out, indent=1))
