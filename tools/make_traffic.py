"""Build profiles/traffic.json: measured DRAM bytes / algorithmic bytes per SpMV format, from ncu
--set full captures (cold, one launch) on configs[3] (3D 27-pt 128^3 fp64) and configs[2] (R-MAT 2^22
fp32).  bench.py scales the dominant format's ratio by its algorithmic bytes per launch."""
import csv, io, json, subprocess, sys

CAPS = {  # format -> (ncu report, algorithmic bytes of that SpMV)
    "CSR": ("gpurun_out/ncu_r01_csr_st3d27.ncu-rep", 710.9e6, "k_spmv_csr_stream<double> on configs[3]"),
    "COO": ("gpurun_out/ncu_r01_coo_st3d27.ncu-rep", 925.4e6, "k_spmv_coo<double> on configs[3]"),
    "ELL": ("gpurun_out/ncu_r01_ell_st3d27.ncu-rep", 713.0e6, "k_spmv_ell<double> on configs[3]"),
    "HYB": ("gpurun_out/ncu_r01_ell_st3d27.ncu-rep", 713.0e6, "k_spmv_ell<double> (HYB of configs[3] has no COO part)"),
    "DIA": ("gpurun_out/ncu_r01_dia_st3d27.ncu-rep", 486.5e6, "k_spmv_dia<double,1> on configs[3]"),
    "COO_rmat": ("gpurun_out/ncu_r01_coo_rmat22.ncu-rep", 816.5e6, "k_spmv_coo<float> on configs[2]"),
    "CSR_rmat": ("gpurun_out/ncu_r01_merge_rmat22.ncu-rep", 572.3e6, "k_spmv_csr_merge<float> on configs[2]"),
}


def metrics(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    h, u = rows[0], rows[1]
    d = dict(zip(h, rows[2]))
    scale = {"Mbyte": 1e6, "Gbyte": 1e9, "Kbyte": 1e3, "byte": 1.0}
    b = lambda k: float(d[k].replace(",", "")) * scale[u[h.index(k)]]
    t = float(d["gpu__time_duration.sum"].replace(",", "")) * (1e-3 if u[h.index("gpu__time_duration.sum")] == "ns" else 1.0)
    return b("dram__bytes_read.sum") + b("dram__bytes_write.sum"), t, float(d["gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed"])


out = {}
for fmt, (path, model, what) in CAPS.items():
    dram, t_us, pct = metrics(path)
    out[fmt] = {"dram_bytes": dram, "algorithmic_bytes": model, "ratio": dram / model, "kernel": what,
                "ncu_time_us": t_us, "dram_pct_of_peak": pct}
json.dump(out, open(sys.argv[1] if len(sys.argv) > 1 else "profiles/traffic.json", "w"), indent=1)
for k, v in out.items():
    print(f"{k:9s} ratio {v['ratio']:.3f}  {v['ncu_time_us']:8.1f} us  dram {v['dram_pct_of_peak']:.1f}%  {v['kernel']}")
