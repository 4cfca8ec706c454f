"""One line per ncu gate capture (tools/r2_gate.sh: gate_<name>.csv, `ncu --csv --metrics ...` of one launch):
kernel, duration, dram__throughput % of ncu's nominal peak, DRAM MB read / written, L2 / L1 hit rates, L2
sectors requested by the SMs.   python tools/gate_summary.py gpurun_out/r2gate > profiles/r02/ncu_gate_tma.txt"""
import csv
import glob
import io
import os
import sys


def main():
    d = sys.argv[1]
    for path in sorted(glob.glob(os.path.join(d, "gate_*.csv"))):
        name = os.path.basename(path)[5:-4]
        txt = open(path, errors="replace").read()
        i = txt.find('"ID"')
        if i < 0:
            print(f"{name:16s} (no capture)")
            continue
        rows = list(csv.DictReader(io.StringIO(txt[i:])))
        m = {r["Metric Name"]: (r["Metric Value"], r["Metric Unit"]) for r in rows}
        kern = rows[0]["Kernel Name"][:48] if rows else "?"

        def val(k, scale=1.0):
            v, u = m.get(k, ("nan", ""))
            v = float(str(v).replace(",", ""))
            if u in ("Kbyte", "KB"):
                v *= 1e-3
            elif u in ("Gbyte", "GB"):
                v *= 1e3
            elif u in ("byte",):
                v *= 1e-6
            elif u in ("msecond", "ms"):
                v *= 1e3
            elif u in ("nsecond", "ns"):
                v *= 1e-3
            return v * scale
        print(f"{name:16s} {kern:48s} t={val('gpu__time_duration.sum'):8.1f}us "
              f"dram__throughput={val('dram__throughput.avg.pct_of_peak_sustained_elapsed'):6.2f}% "
              f"dram_read={val('dram__bytes_read.sum'):8.1f}MB write={val('dram__bytes_write.sum'):6.1f}MB "
              f"l2_hit={val('lts__t_sector_hit_rate.pct'):5.2f}% l1_hit={val('l1tex__t_sector_hit_rate.pct'):5.2f}% "
              f"l2_sectors={val('lts__t_sectors_srcunit_tex.sum') / 1e6:7.2f}M "
              f"warps_active={val('sm__warps_active.avg.pct_of_peak_sustained_active'):5.1f}%")


if __name__ == "__main__":
    main()
