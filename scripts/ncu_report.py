"""Summarise an `ncu --set full` capture of the search kernel (run HERE on the
.ncu-rep brought back from the GPU box): key counters, DRAM bytes per query,
stall breakdown and the top stalled SASS instructions -> a markdown file under
profiles/, plus the traffic JSON bench.py reads for `roofline.traffic`.

usage: python scripts/ncu_report.py gpurun_out/prof_op.ncu-rep --nq 10000 \
          --out profiles/round1_c2_op_ncu.md --traffic profiles/traffic_C2.json \
          --params itopk=12,width=8,ctas_per_query=4,threads_per_cta=512,slots=32,visited_mode=1
"""
import argparse
import csv
import io
import json
import subprocess


def ncu_csv(rep, page, extra=()):
    out = subprocess.run(["ncu", "-i", rep, "--page", page, "--csv", *extra], capture_output=True, text=True,
                         check=True).stdout
    return list(csv.reader(io.StringIO(out)))


def num(x):
    try:
        return float(str(x).replace(",", ""))
    except Exception:
        return None


def to_bytes(v, u):
    return num(v) * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6, "GB": 1e9}.get(u, 1)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("rep")
    ap.add_argument("--nq", type=int, required=True, help="queries served by the captured launch")
    ap.add_argument("--out", required=True)
    ap.add_argument("--traffic")
    ap.add_argument("--params", default="")
    ap.add_argument("--title", default="search kernel")
    a = ap.parse_args()
    rows = ncu_csv(a.rep, "raw")
    hdr, units, vals = rows[0], rows[1], rows[2]
    d = {h: (v, u) for h, u, v in zip(hdr, units, vals)}
    keys = ["Kernel Name", "gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum",
            "dram__throughput.avg.pct_of_peak_sustained_elapsed", "lts__t_sector_hit_rate.pct",
            "sm__throughput.avg.pct_of_peak_sustained_elapsed", "sm__warps_active.avg.pct_of_peak_sustained_active",
            "launch__registers_per_thread", "launch__grid_size", "launch__block_size",
            "launch__shared_mem_per_block_dynamic", "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
            "smsp__inst_executed.sum"]
    lines = [f"# ncu --set full: {a.title}", "", f"source: `{a.rep}` (ncu --set full --clock-control none, "
             f"kernel replay; per-launch numbers are cold-cache and serialised)", "", "| metric | value | unit |",
             "|---|---|---|"]
    for k in keys:
        if k in d:
            lines.append(f"| {k} | {d[k][0]} | {d[k][1]} |")
    rd = to_bytes(*d["dram__bytes_read.sum"]) if "dram__bytes_read.sum" in d else None
    wr = to_bytes(*d["dram__bytes_write.sum"]) if "dram__bytes_write.sum" in d else None
    traffic = (rd or 0) + (wr or 0)
    lines += ["", f"DRAM traffic per launch: {traffic / 1e6:.1f} MB = {traffic / a.nq / 1e6:.3f} MB per query "
              f"({a.nq} queries)"]
    st = [(h.replace("smsp__pcsamp_warps_issue_stalled_", ""), num(v)) for h, (v, u) in d.items()
          if h.startswith("smsp__pcsamp_warps_issue_stalled_") and not h.endswith("not_issued") and num(v)]
    tot = sum(v for _, v in st) or 1
    lines += ["", "Warp-stall samples (kernel-wide): " + ", ".join(
        f"{h} {100 * v / tot:.1f}%" for h, v in sorted(st, key=lambda x: -x[1])[:8])]
    try:
        src = ncu_csv(a.rep, "source", ["--print-source", "sass"])
        shdr, data = src[1], src[2:]
        ci = {h: i for i, h in enumerate(shdr)}
        S = ci["Warp Stall Sampling (All Samples)"]
        tot2 = sum(num(r[S]) or 0 for r in data) or 1
        sc = [h for h in shdr if h.startswith("stall_") and "(Not Issued)" not in h]
        lines += ["", "Top stalled SASS instructions:", "", "| share | instruction | top reasons |", "|---|---|---|"]
        for r in sorted(data, key=lambda r: -(num(r[S]) or 0))[:15]:
            rs = sorted(((h[6:], num(r[ci[h]]) or 0) for h in sc), key=lambda x: -x[1])[:2]
            lines.append(f"| {100 * (num(r[S]) or 0) / tot2:.1f}% | `{r[ci['Source']][:60]}` | "
                         + ", ".join(f"{n} {100 * v / max(1, num(r[S]) or 1):.0f}%" for n, v in rs if v) + " |")
    except Exception as e:  # source page needs -lineinfo / --import-source
        lines += ["", f"(source page unavailable: {e})"]
    open(a.out, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))
    if a.traffic:
        params = {}
        for kv in filter(None, a.params.split(",")):
            k, v = kv.split("=")
            params[k] = int(v)
        json.dump({"source": f"ncu --set full capture {a.rep} -> {a.out}", "queries": a.nq,
                   "dram_bytes_per_launch_per_query": traffic / a.nq, "params": params}, open(a.traffic, "w"),
                  indent=1)


if __name__ == "__main__":
    main()
