"""Summarise an ncu --set full capture exported as CSV (raw + details pages)."""
import csv
import json
import sys


def load_raw(path):
    rows = list(csv.reader(open(path)))
    hdr, units, vals = rows[0], rows[1], rows[2]
    return {h: (v, u) for h, u, v in zip(hdr, units, vals)}


def num(x):
    try:
        return float(str(x).replace(",", ""))
    except Exception:
        return None


def main(raw_path, details_path, nq=None):
    d = load_raw(raw_path)
    keys = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "smsp__inst_executed.sum",
            "sm__warps_active.avg.pct_of_peak_sustained_active", "launch__registers_per_thread",
            "launch__grid_size", "launch__block_size", "smsp__average_warp_latency_per_inst_issued.ratio",
            "lts__t_sectors_srcunit_tex_op_read.sum", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum"]
    out = {}
    for k in keys:
        if k in d:
            out[k] = {"value": d[k][0], "unit": d[k][1]}
    st = [(h.replace("smsp__pcsamp_warps_issue_stalled_", ""), num(v)) for h, (v, u) in d.items()
          if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued") and num(v)]
    tot = sum(v for _, v in st)
    out["stall_pct"] = {h: round(100 * v / tot, 1) for h, v in sorted(st, key=lambda x: -x[1])[:10]}
    # dram bytes in bytes
    def to_bytes(k):
        v, u = d[k]
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        return num(v) * scale
    if "dram__bytes_read.sum" in d:
        tr = to_bytes("dram__bytes_read.sum") + to_bytes("dram__bytes_write.sum")
        out["dram_bytes_total"] = tr
        if nq:
            out["dram_bytes_per_query"] = tr / nq
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1], sys.argv[2], int(sys.argv[3]) if len(sys.argv) > 3 else None)
