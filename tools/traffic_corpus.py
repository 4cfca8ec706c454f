"""Measured DRAM traffic per SpMV launch on the bench workload itself (corpus-200), per format.

Input: an ncu CSV (--metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,
lts__t_sectors_srcunit_tex.sum
--cache-control none -k regex:"k_spmv|k_zero") of `bench.py --steps 1 --warmup 0 --reps R
--race-warmup W --dump D`, and that dump.  The SpMV launches come in race order (matrix by matrix,
formats CSR..DIA, W + R calls each); each call's kernels are predicted from the matrix's features
(CSR variant, HYB one-launch rule) and checked by name.  The LAST call of every (matrix, format) runs
right after an identical call, as in the race's back-to-back reps, and with --cache-control none the
L2 holds what that call left: its DRAM bytes are the hot-rep traffic the race sees.

  python tools/traffic_corpus.py launches.csv dump.jsonl W+R [out.json]
"""
import csv
import json
import sys
from collections import defaultdict

NAMES = ["CSR", "COO", "ELL", "HYB", "DIA"]


def hyb_rowwise(f, z):
    o = f["nnz_max"] - f["hyb_k"]
    return f["hyb_coo"] > 0 and (o <= 32 or (z < (1 << 20) and o <= 64))


def kernels_of(fmt, f, z):
    if fmt == 0:
        if f["csr_variant"] in (3, 4, 5) and z == 0:
            return ["k_zero"]
        return {2: ["k_spmv_csr_stream"], 3: ["k_zero_rows", "k_spmv_csr_tile"],
                4: ["k_zero_rows", "k_spmv_csr_tile"], 5: ["k_zero", "k_spmv_csr_tile"],
                1: ["k_spmv_csr_merge", "k_spmv_csr_merge_fixup"], 0: ["k_spmv_csr_vector"]}[f["csr_variant"]]
    if fmt == 1:
        return ["k_zero", "k_spmv_coo"]
    if fmt == 2:
        return ["k_spmv_ell"]
    if fmt == 3:
        if f["hyb_k"] == 0:
            return ["k_zero", "k_spmv_coo"]
        if f["hyb_coo"] == 0 or hyb_rowwise(f, z):
            return ["k_spmv_ell"]
        return ["k_zero", "k_spmv_ell", "k_spmv_coo"]  # overlapped parts
    return ["k_spmv_dia"]


def load_launches(path):
    rows = list(csv.reader([l for l in open(path) if l.startswith('"')]))
    h = rows[0]
    ik, iid, im, iv = h.index("Kernel Name"), h.index("ID"), h.index("Metric Name"), h.index("Metric Value")
    per = defaultdict(dict)
    order = []
    for r in rows[1:]:
        if len(r) <= iv:
            continue
        key = int(r[iid])
        if key not in per:
            order.append(key)
            per[key]["name"] = r[ik]
        per[key][r[im]] = float(r[iv].replace(",", ""))
    return [per[k] for k in order]


def main(csv_path, dump_path, calls, out=None):
    launches = load_launches(csv_path)
    dump = [json.loads(l) for l in open(dump_path)]
    pos = 0
    acc = {f: defaultdict(float) for f in range(5)}
    for d in dump:
        f_, L, z = d["features"], d["race"], d["nnz"]
        for fmt in range(5):
            if L["status"][fmt] != 0:
                continue
            ks = kernels_of(fmt, f_, z)
            for c in range(calls):
                last = c == calls - 1
                for k in ks:
                    got = launches[pos]["name"]
                    if not got.split("(")[0].replace("void ", "").split("::")[-1].startswith(k):
                        raise SystemExit(f"launch {pos}: expected {k} for matrix {d['id']} {NAMES[fmt]}, got {got[:80]}")
                    if last:
                        a = acc[fmt]
                        a["dram"] += launches[pos].get("dram__bytes_read.sum", 0) + launches[pos].get("dram__bytes_write.sum", 0)
                        a["ns"] += launches[pos].get("gpu__time_duration.sum", 0)
                        a["l2s"] += launches[pos].get("lts__t_sectors_srcunit_tex.sum", 0)
                    pos += 1
            acc[fmt]["alg"] += L["bytes"][fmt]
            acc[fmt]["n"] += 1
    res = {}
    for fmt in range(5):
        a = acc[fmt]
        if not a["n"]:
            continue
        res[NAMES[fmt]] = {"launches": int(a["n"]), "dram_bytes_per_launch": a["dram"] / a["n"],
                           "algorithmic_bytes_per_launch": a["alg"] / a["n"], "ratio": a["dram"] / a["alg"],
                           "ncu_us_per_launch": a["ns"] / a["n"] / 1e3,
                           "l2_sectors_per_launch": a["l2s"] / a["n"],
                           "kernel": "+".join(sorted({k for d in dump for k in kernels_of(fmt, d["features"], d["nnz"])}))}
    res["_source"] = {"csv": csv_path, "dump": dump_path, "calls_per_format": calls, "launches_parsed": pos,
                      "launches_in_csv": len(launches),
                      "note": "last of W+R back-to-back calls per (matrix, format), ncu --cache-control none: "
                              "the hot-rep DRAM traffic of the race; per launch = averaged over the corpus; "
                              "l2_sectors = lts__t_sectors_srcunit_tex.sum (32 B sectors the SMs requested from L2)"}
    s = json.dumps(res, indent=1)
    print(s)
    if out:
        open(out, "w").write(s + "\n")


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]), sys.argv[4] if len(sys.argv) > 4 else None)
