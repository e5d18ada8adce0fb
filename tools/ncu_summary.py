"""Summarise an `ncu --set full` report into the JSON kept under profiles/.
usage: python tools/ncu_summary.py report.ncu-rep [kernel-index] > summary.json"""
import csv
import io
import json
import subprocess
import sys

KEYS = [
    "Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "launch__grid_size", "launch__block_size", "launch__registers_per_thread",
    "launch__shared_mem_per_block_dynamic", "launch__occupancy_limit_shared_mem",
    "launch__occupancy_limit_registers", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "lts__t_sector_hit_rate.pct", "lts__t_sectors_srcunit_tex_op_read.sum",
    "lts__t_sectors_srcunit_tex_op_write.sum", "smsp__inst_executed.sum",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "sm__cycles_elapsed.avg",
    "gpc__cycles_elapsed.avg.per_second", "dram__cycles_elapsed.avg.per_second",
]
UNIT_SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}


def main():
    rep = sys.argv[1]
    idx = int(sys.argv[2]) if len(sys.argv) > 2 else 0
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True, check=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    head, units, row = rows[0], rows[1], rows[2 + idx]
    get = {h: (u, v) for h, u, v in zip(head, units, row)}
    s = {}
    for k in KEYS:
        if k in get:
            u, v = get[k]
            s[k] = f"{v} {u}".strip()
    # stall breakdown from the warp-state samples (share of all samples)
    pre = "smsp__pcsamp_warps_issue_stalled_"
    st = {h[len(pre):]: float(v.replace(",", "")) for h, (u, v) in get.items()
          if h.startswith(pre) and not h.endswith("_not_issued") and v not in ("", "n/a")}
    tot = sum(st.values())
    if tot:
        s["stall_reasons_pct"] = {k: round(100 * v / tot, 1)
                                  for k, v in sorted(st.items(), key=lambda kv: -kv[1])[:8]}
    # DRAM bytes per launch, and the achieved rate
    def val(k):
        u, v = get[k]
        return float(v.replace(",", "")) * UNIT_SCALE.get(u, 1)
    t_u, t_v = get["gpu__time_duration.sum"]
    t = float(t_v.replace(",", "")) * {"ns": 1e-9, "us": 1e-6, "ms": 1e-3, "s": 1}[t_u]
    dram = val("dram__bytes_read.sum") + val("dram__bytes_write.sum")
    s["dram_bytes_per_launch"] = int(dram)
    s["dram_gbs"] = round(dram / t / 1e9, 1)
    json.dump(s, sys.stdout, indent=1)
    print()


if __name__ == "__main__":
    main()
