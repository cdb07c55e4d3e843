"""Summarise tools/lever_ab.sh captures into profiles/<tag>_levers.md: per variant the
counters SURVEY 8(d) names, normalised per query (m from the bench line)."""
import csv
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
M = {"c2": 1 << 24, "c3": 1 << 26, "c5": 1 << 26}


def parse(path):
    txt = open(path).read()
    i = txt.find('"ID"')
    if i < 0:
        return None
    rows = list(csv.DictReader(io.StringIO(txt[i:])))
    d = {}
    for r in rows:
        d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
        d["kernel"] = r["Kernel Name"].split("(")[0]
    return d


def main(src, tag):
    out = ["| variant | kernel | time ms | DRAM B/q | L2 read sectors/q | L2 hit % | L1 hit % | "
           "global sectors/request | LSU pipe % | smem wavefronts/q | long-scoreboard stall/issue |",
           "|---|---|---|---|---|---|---|---|---|---|---|"]
    for f in sorted(os.listdir(src)):
        if not (f.startswith("ab_") and f.endswith(".csv")):
            continue
        d = parse(os.path.join(src, f))
        if not d:
            continue
        v = f[3:-4]
        m = M[v.split("_")[0]]
        g = lambda k: d.get(k, float("nan"))
        out.append("| %s | %s | %.3f | %.1f | %.2f | %.1f | %.1f | %.2f | %.1f | %.2f | %.1f |" % (
            v, d["kernel"].replace("void unnamed>::", ""), g("gpu__time_duration.sum") / 1e6,
            (g("dram__bytes_read.sum") + g("dram__bytes_write.sum")) / m,
            g("lts__t_sectors_srcunit_tex_op_read.sum") / m, g("lts__t_sector_hit_rate.pct"),
            g("l1tex__t_sector_hit_rate.pct"),
            g("l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum") / max(1.0, g("l1tex__t_requests_pipe_lsu_mem_global_op_ld.sum")),
            g("l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed"),
            g("l1tex__data_pipe_lsu_wavefronts_mem_shared.sum") / m,
            g("smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio")))
        dst = os.path.join(ROOT, "profiles", f"{tag}_ab_{v}.csv")
        open(dst, "w").write(open(os.path.join(src, f)).read())
    txt = "\n".join(out) + "\n"
    open(os.path.join(ROOT, "profiles", f"{tag}_levers.md"), "w").write(
        "# Design levers A/B (ncu single pass, --cache-control none, one steady-state launch each)\n\n"
        "Source: tools/lever_ab.sh; raw CSVs beside this file.  Per-query figures divide by the\n"
        "config's batch (c2 2^24, c3/c5 2^26).  Units: the ncu DRAM byte counters are in the CSV's units.\n\n"
        + txt)
    print(txt)


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out"),
         sys.argv[2] if len(sys.argv) > 2 else "r01")
