"""One-line-per-capture summary of `ncu --page raw --csv` exports (duration, DRAM bytes / throughput, cache
hit rates, occupancy, issue activity, top stall reasons per issue).  python tools/ncu_raw_summary.py *.raw.csv"""
import csv
import sys

KEYS = [("gpu__time_duration.sum", "dur_us", None), ("dram__bytes_read.sum", "dram_rd_MB", None),
        ("dram__bytes_write.sum", "dram_wr_MB", None),
        ("gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed", "dram_pct", 1),
        ("lts__t_sector_hit_rate.pct", "l2_hit", 1), ("l1tex__t_sector_hit_rate.pct", "l1_hit", 1),
        ("sm__warps_active.avg.pct_of_peak_sustained_active", "warps_act", 1),
        ("smsp__issue_active.avg.pct_of_peak_sustained_active", "issue_act", 1),
        ("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "smem_wf", 1),
        ("lts__t_sectors_srcunit_tex.sum", "l2_sect_M", 1e-6),
        ("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum", "ld_req_M", 1e-6),
        ("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum", "ld_sect_M", 1e-6),
        ("l1tex__data_pipe_lsu_wavefronts_mem_lg.sum", "lg_wf_M", 1e-6),
        ("sm__cycles_elapsed.avg", "cycles", 1),
        ("launch__registers_per_thread", "regs", 1), ("launch__grid_size", "grid", 1)]


UNIT = {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3, "byte": 1e-6,
        "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}  # -> us / MB


def conv(v):
    try:
        return float(v.replace(",", ""))
    except ValueError:
        return None


def main():
    for path in sys.argv[1:]:
        rows = list(csv.reader(open(path)))
        if len(rows) < 3:
            print(path, "empty")
            continue
        hdr, units, data = rows[0], rows[1], rows[2:]
        idx = {h: i for i, h in enumerate(hdr)}
        for d in data:
            out = {"capture": path.split("/")[-1].replace(".raw.csv", ""), "kernel": d[idx["Kernel Name"]][:60]}
            for k, name, sc in KEYS:
                if k in idx and conv(d[idx[k]]) is not None:
                    f = sc if sc is not None else UNIT.get(units[idx[k]], 1.0)
                    out[name] = round(conv(d[idx[k]]) * f, 3)
            st = []
            for h, i in idx.items():
                if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                    v = conv(d[i])
                    if v:
                        st.append((v, h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
            st.sort(reverse=True)
            out["stalls"] = " ".join(f"{n}={v:.2f}" for v, n in st[:5])
            print(out)


if __name__ == "__main__":
    main()
