"""Summarise ncu captures in gpurun_out/ into profiles/ (tracked): per-kernel metrics JSON,
the launch list of a bench run, and the DRAM traffic per launch that bench.py reports."""
import csv
import io
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
OUT = os.path.join(ROOT, "gpurun_out")
PROF = os.path.join(ROOT, "profiles")
METRICS = {
    "duration_ms": ("gpu__time_duration.sum", 1e-3, "us->ms"),
    "dram_read_GB": ("dram__bytes_read.sum", None, None),
    "dram_write_GB": ("dram__bytes_write.sum", None, None),
    "dram_throughput_pct": ("dram__throughput.avg.pct_of_peak_sustained_elapsed", None, None),
    "l2_hit_pct": ("lts__t_sector_hit_rate.pct", None, None),
    "l2_tex_throughput_pct": ("lts__t_sectors_srcunit_tex.avg.pct_of_peak_sustained_elapsed", None, None),
    "tma_load_GB": ("l1tex__m_xbar2l1tex_read_bytes_mem_global_op_tma_ld.sum", None, None),
    "tma_store_GB": ("l1tex__m_l1tex2xbar_write_bytes_mem_global_op_tma_st.sum", None, None),
    "tensor_pipe_active_pct": ("sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_elapsed", None, None),
    "fma_pipe_active_pct": ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", None, None),
    "sm_throughput_pct": ("sm__throughput.avg.pct_of_peak_sustained_elapsed", None, None),
    "sm_active_cycles_avg": ("sm__cycles_active.avg", None, None),
    "sm_active_cycles_max": ("sm__cycles_active.max", None, None),
    "registers_per_thread": ("launch__registers_per_thread", None, None),
    "grid": ("launch__grid_size", None, None),
    "block": ("launch__block_size", None, None),
    "smem_dynamic_per_block": ("launch__shared_mem_per_block_dynamic", None, None),
}
SCALE = {"Gbyte": 1.0, "Mbyte": 1e-3, "Kbyte": 1e-6, "byte": 1e-9, "Tbyte": 1e3, "ms": 1.0, "us": 1e-3, "usecond": 1e-3,
         "msecond": 1.0, "nsecond": 1e-6}


def summarize(path):
    out = subprocess.check_output(["ncu", "-i", path, "--page", "raw", "--csv"], text=True)
    rows = list(csv.reader(io.StringIO(out)))
    h, units, vals = rows[0], rows[1], rows[2]
    d = {"kernel": vals[h.index("Kernel Name")] if "Kernel Name" in h else ""}
    for key, (metric, _, _) in METRICS.items():
        if metric in h:
            i = h.index(metric)
            v = vals[i].replace(",", "")
            try:
                x = float(v)
            except ValueError:
                d[key] = v
                continue
            u = units[i]
            if key.endswith("_GB"):
                x *= SCALE.get(u, 1.0)
            if key == "duration_ms":
                x *= SCALE.get(u, 1.0)
            d[key] = round(x, 4)
    return d


def launches(path):
    """Kernel -> (count, total ms, share) from an ncu --metrics gpu__time_duration.sum CSV."""
    txt = open(path).read()
    txt = txt[txt.index('"ID"'):] if '"ID"' in txt else txt
    rows = list(csv.DictReader(io.StringIO(txt)))
    agg = {}
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        name = r["Kernel Name"].split("(")[0]
        v = float(r["Metric Value"].replace(",", ""))
        unit = r.get("Metric Unit", "")
        ms = v * {"nsecond": 1e-6, "usecond": 1e-3, "msecond": 1.0, "ns": 1e-6, "us": 1e-3, "ms": 1.0}.get(unit, 1e-6)
        c, t = agg.get(name, (0, 0.0))
        agg[name] = (c + 1, t + ms)
    tot = sum(t for _, t in agg.values())
    return {k: {"launches": c, "total_ms": round(t, 4), "share": round(t / tot, 4)} for k, (c, t) in
            sorted(agg.items(), key=lambda kv: -kv[1][1])}


if __name__ == "__main__":
    tag = sys.argv[1] if len(sys.argv) > 1 else "r01"
    os.makedirs(PROF, exist_ok=True)
    res = {}
    for cfg in ("C5", "C4", "C4single", "C2", "C3", "C3i", "C1"):
        p = os.path.join(OUT, f"prof_{cfg}.ncu-rep")
        if os.path.exists(p):
            res[cfg] = summarize(p)
    lf = os.path.join(OUT, "launches_c5.csv")
    if os.path.exists(lf):
        res["launch_list_bench_C5"] = launches(lf)
    with open(os.path.join(PROF, f"ncu_{tag}.json"), "w") as f:
        json.dump(res, f, indent=1)
    traffic = {cfg: {"dram_bytes_per_launch": int((v["dram_read_GB"] + v["dram_write_GB"]) * 1e9),
                     "source": f"profiles/ncu_{tag}.json (ncu --set full, one launch, cold)"}
               for cfg, v in res.items() if isinstance(v, dict) and "dram_read_GB" in v and cfg in ("C5", "C4", "C2", "C3")}
    with open(os.path.join(PROF, "ncu_traffic.json"), "w") as f:
        json.dump(traffic, f, indent=1)
    print(json.dumps(res, indent=1))
