"""Summarise an ncu report: key throughput / traffic / stall metrics as JSON."""
import csv
import io
import json
import subprocess
import sys

KEYS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
        "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
        "lts__t_sectors_srcunit_tex.avg.pct_of_peak_sustained_elapsed",
        "l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum",
        "l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum",
        "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__cycles_active.avg", "sm__cycles_active.max",
        "sm__cycles_active.min", "launch__registers_per_thread", "launch__grid_size",
        "smsp__inst_executed.sum", "sm__inst_executed_pipe_tensor.sum"]


def summarize(path):
    out = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(out)))
    h, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {}
        for k in KEYS:
            for i, name in enumerate(h):
                if name == k or name.startswith(k.replace(".sum", "").replace(".avg", "") + "_realtime") and False:
                    d[k] = (r[i], units[i])
        tensor = [(n, r[i], units[i]) for i, n in enumerate(h) if "pipe_tensor" in n and "pct" in n]
        d["_tensor_pcts"] = tensor[:6]
        d["_kernel"] = r[h.index("Kernel Name")] if "Kernel Name" in h else ""
        res.append(d)
    return res


if __name__ == "__main__":
    for p in sys.argv[1:]:
        print(p)
        print(json.dumps(summarize(p), indent=1))
