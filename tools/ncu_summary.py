"""Summarise an ncu --set full report of the MAC kernel into profiles/ncu_summary.json
(the bench's roofline.traffic comes from here) and print the key counters.

    python tools/ncu_summary.py gpurun_out/<rep>.ncu-rep <key> [launches.csv]
key: e.g. mac_tc_pair_bf16 (bench.py looks up "mac_<kernel>_<math>")."""
import csv, io, json, os, subprocess, sys

WANT = {
    "gpu__time_duration.sum": "duration_ns",
    "dram__bytes_read.sum": "dram_bytes_read",
    "dram__bytes_write.sum": "dram_bytes_write",
    "sm__cycles_elapsed.avg": "sm_cycles_elapsed",
    "sm__cycles_active.avg": "sm_cycles_active",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed": "tensor_pipe_pct",
    "sm__inst_executed_pipe_tensor_subpipe_hmma.avg.pct_of_peak_sustained_active": "hmma_inst_pct",
    "lts__t_bytes.sum": "l2_bytes",
    "lts__throughput.avg.pct_of_peak_sustained_elapsed": "l2_throughput_pct",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed": "dram_throughput_pct",
    "launch__registers_per_thread": "registers",
    "launch__grid_size": "grid",
    "launch__block_size": "block",
    "smsp__cycles_active.avg": "smsp_cycles_active",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed": "sm_throughput_pct",
    "gpc__cycles_elapsed.avg.per_second": "gpc_hz",
    "lts__t_sectors_srcunit_tex_op_write.sum": "l2_write_sectors",
    "lts__t_sectors_srcunit_tex_op_read.sum": "l2_read_sectors",
    "smsp__inst_executed.sum": "inst_executed",
    "sm__warps_active.avg.pct_of_peak_sustained_active": "warps_active_pct",
}
UNIT = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ns": 1, "us": 1e3, "ms": 1e6, "Ghz": 1e9, "Mhz": 1e6}


def main():
    rep, key = sys.argv[1], sys.argv[2]
    raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units = rows[0], rows[1]
    out = {}
    for row in rows[2:3]:
        out["kernel"] = row[hdr.index("Kernel Name")][:120]
        for m, k in WANT.items():
            if m in hdr:
                i = hdr.index(m)
                try:
                    v = float(row[i].replace(",", ""))
                except ValueError:
                    continue
                out[k] = v * UNIT.get(units[i], 1)
    path = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "ncu_summary.json")
    allsum = json.load(open(path)) if os.path.exists(path) else {}
    out["source"] = os.path.basename(rep)
    allsum[key] = out
    json.dump(allsum, open(path, "w"), indent=1, sort_keys=True)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main()
