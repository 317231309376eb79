"""Reduce the ncu captures of tools/prof_traffic.sh to the per-config summaries
bench.py reads (profiles/ncu_cfg{3,4,5}_summary.json: traffic per launch of the
dominant kernel, FP64-pipe and issue utilisation).  usage: python tools/mk_summaries.py [round]"""
import csv
import json
import sys

R = sys.argv[1] if len(sys.argv) > 1 else "r2"


SCALE = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12, "ns": 1e-6, "us": 1e-3, "usecond": 1e-3,
         "ms": 1, "msecond": 1, "s": 1e3, "second": 1e3, "nsecond": 1e-6}


def raw(path):
    """{metric: value in bytes / ms / plain} from an `ncu --page raw --csv` export"""
    rows = list(csv.reader(open(path)))
    h, u, v = rows[0], rows[1], rows[2]
    out = {}
    for i, k in enumerate(h):
        try:
            out[k] = float(v[i].replace(",", "")) * SCALE.get(u[i], 1)
        except ValueError:
            out[k] = v[i]
    return out


def f(d, k):
    x = d.get(k)
    return x if isinstance(x, float) else None


def summary(d, kernel, cfg, periods, n_inst, note):
    rd = f(d, "dram__bytes_read.sum")
    wr = f(d, "dram__bytes_write.sum")
    return {"kernel": kernel, "config": cfg, "periods": periods, "n_inst": n_inst,
            "dram_bytes_per_launch": (rd or 0) + (wr or 0), "gpu_time_ms": f(d, "gpu__time_duration.sum"),
            "fp64_pipe_pct": f(d, "sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active"),
            "issue_active_pct": f(d, "smsp__issue_active.avg.pct_of_peak_sustained_active"),
            "warps_active_per_sm": f(d, "sm__warps_active.avg.per_cycle_active"),
            "registers": f(d, "launch__registers_per_thread"), "note": note,
            "source": f"ncu --set full --clock-control none ({R}, tools/prof_traffic.sh; profiles/{R}_ncu_cfg{cfg}_raw.csv)"}


if __name__ == "__main__":
    import shutil
    for name, cfg, kern, periods, n, note in [
            ("prof_cfg3c", 3, "k_simulate<9,3,4,32,0,0,1> (chunked schedule)", 1000, 65536, "one launch = one bench step"),
            ("prof_cfg4", 4, "k_period<9,2,4> (one period of 1,048,576 servers)", 1000, 1048576,
             "per k_period launch (one per period; independent of the run length); algorithmic 1936 B x 1,048,576 = 2.030 GB")]:
        d = raw(f"gpurun_out/{name}_raw.csv")
        shutil.copy(f"gpurun_out/{name}_raw.csv", f"profiles/{R}_ncu_cfg{cfg}_raw.csv")
        json.dump(summary(d, kern, cfg, periods, n, note), open(f"profiles/ncu_cfg{cfg}_summary.json", "w"), indent=1)
    rows = list(csv.DictReader(l for l in open("gpurun_out/prof_cfg5_metrics.csv") if not l.startswith("==")))
    m = {r["Metric Name"]: r["Metric Value"].replace(",", "") for r in rows}
    unit = {r["Metric Name"]: r["Metric Unit"] for r in rows}
    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "ms": 1, "us": 1e-3, "ns": 1e-6, "s": 1e3, "%": 1}
    val = lambda k: float(m[k]) * scale.get(unit[k], 1)  # noqa: E731
    shutil.copy("gpurun_out/prof_cfg5_metrics.csv", f"profiles/{R}_ncu_cfg5_metrics.csv")
    json.dump({"kernel": "k_simulate<4,2,4,128> (cfg 5)", "config": 5, "periods": 2000, "n_inst": 8388608,
               "dram_bytes_per_launch": val("dram__bytes_read.sum") + val("dram__bytes_write.sum"),
               "gpu_time_ms": val("gpu__time_duration.sum"),
               "fp64_pipe_pct": val("sm__inst_executed_pipe_fp64.avg.pct_of_peak_sustained_active"),
               "source": f"ncu --metrics ({R}, tools/prof_traffic.sh; profiles/{R}_ncu_cfg5_metrics.csv)"},
              open("profiles/ncu_cfg5_summary.json", "w"), indent=1)
    print(open("profiles/ncu_cfg3_summary.json").read())
