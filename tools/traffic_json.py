"""Collect the steady-state single-pass ncu CSVs (tools/steady_traffic.sh) into
profiles/traffic.json: DRAM bytes per launch of each config's dominant kernel."""
import csv
import io
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def parse(path):
    txt = open(path).read()
    i = txt.find('"ID"')
    if i < 0:
        return None
    rows = list(csv.DictReader(io.StringIO(txt[i:])))
    by = {}
    for r in rows:
        by.setdefault(r["ID"], {})[r["Metric Name"]] = r["Metric Value"]
        by[r["ID"]]["kernel"] = r["Kernel Name"].split("(")[0]
    last = by[sorted(by, key=int)[-1]]
    rd, wr = float(last["dram__bytes_read.sum"]), float(last["dram__bytes_write.sum"])
    return {"dram_bytes_per_launch": int(rd + wr), "dram_read": int(rd), "dram_write": int(wr),
            "l2_hit_pct": float(last.get("lts__t_sector_hit_rate.pct", "nan")),
            "duration_ns_under_ncu": int(float(last["gpu__time_duration.sum"])),
            "kernel": last["kernel"],
            "source": f"ncu single-pass --cache-control none, steady state (profiles/{os.path.basename(path)})"}


def main(src_dir, tag):
    out = {}
    for c in ("c1", "c2", "c3", "c4", "c5"):
        p = os.path.join(src_dir, f"steady_{c}.csv")
        if os.path.exists(p):
            d = parse(p)
            if d:
                dst = os.path.join(ROOT, "profiles", f"{tag}_steady_{c}.csv")
                open(dst, "w").write(open(p).read())
                d["source"] = f"ncu single-pass --cache-control none, steady state (profiles/{tag}_steady_{c}.csv)"
                out[c] = d
    json.dump(out, open(os.path.join(ROOT, "profiles", "traffic.json"), "w"), indent=1)
    print(json.dumps(out, indent=1))


if __name__ == "__main__":
    main(sys.argv[1] if len(sys.argv) > 1 else os.path.join(ROOT, "gpurun_out"),
         sys.argv[2] if len(sys.argv) > 2 else "r01")
