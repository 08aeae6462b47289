"""Summarise ncu reports / launch lists into profiles/ (markdown + JSON).  Tool code.

usage: python tools/ncu_summarize.py OUT_PREFIX report1.ncu-rep [report2 ...] [--launch list.csv]
"""
import csv
import io
import json
import os
import subprocess
import sys

KEYS = [
    "gpu__time_duration.sum",
    "gpc__cycles_elapsed.max",
    "gpc__cycles_elapsed.avg.per_second",
    "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
    "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "dram__bytes_read.sum",
    "dram__bytes_write.sum",
    "dram__throughput.avg.pct_of_peak_sustained_elapsed",
    "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "lts__t_sector_hit_rate.pct",
    "l1tex__data_pipe_tc_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "launch__registers_per_thread",
    "launch__grid_size",
    "launch__block_size",
    "launch__cluster_dim_x",
    "smsp__inst_executed.sum",
    "sm__warps_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed",
    "l1tex__lsu_writeback_active.avg.pct_of_peak_sustained_elapsed",
]


def raw(rep):
    out = subprocess.check_output(["ncu", "-i", rep, "--page", "raw", "--csv"], stderr=subprocess.DEVNULL).decode()
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {}
        for h, u, v in zip(hdr, units, r):
            d[h] = (v, u)
        res.append(d)
    return res


def to_bytes(v, u):
    try:
        x = float(v.replace(",", ""))
    except ValueError:
        return None
    mult = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, None)
    return x * mult if mult else x


def summarize(rep):
    out = []
    for d in raw(rep):
        name = d.get("Kernel Name", ("?", ""))[0]
        s = {"kernel": name[:140], "report": os.path.basename(rep)}
        for k in KEYS:
            h = k if k in d else next((x for x in d if x.endswith("." + k)), None)
            if h is not None:
                s[k] = d[h][0] + (" " + d[h][1] if d[h][1] else "")
        rb = to_bytes(*d["dram__bytes_read.sum"]) if "dram__bytes_read.sum" in d else None
        wb = to_bytes(*d["dram__bytes_write.sum"]) if "dram__bytes_write.sum" in d else None
        if rb is not None and wb is not None:
            s["dram_bytes_total"] = rb + wb
        out.append(s)
    return out


def launch_list(path, first=None):
    """Per-kernel totals of an ncu launch list; `first` = only the first N launches (the
    bench's headline warm-up + timed steps come first)."""
    rows = [r for r in csv.reader(open(path)) if len(r) > 10]
    hdr = rows[0]
    ik, iv, iu = hdr.index("Kernel Name"), hdr.index("Metric Value"), hdr.index("Metric Unit")
    agg = {}
    for r in rows[1:1 + first if first else None]:
        k = r[ik].split("(")[0][:80]
        ns = float(r[iv].replace(",", "")) * (1e3 if r[iu] == "usecond" else 1e6 if r[iu] == "msecond" else 1)
        a = agg.setdefault(k, [0, 0.0])
        a[0] += 1
        a[1] += ns
    tot = sum(v[1] for v in agg.values())
    return [{"kernel": k, "launches": v[0], "total_ms": v[1] / 1e6, "share": v[1] / tot}
            for k, v in sorted(agg.items(), key=lambda kv: -kv[1][1])]


def bench_summary(out, cfg, shape, gemm_rep, split_rep, label):
    """profiles/ncu_summary.json for bench.py: the DRAM bytes of the bench's own GEMM launch
    (identified by its configuration and shape: bench.py uses the number only when both
    match its launch) and of its split launches."""
    g = [k for k in summarize(gemm_rep) if "egemm_tc_kernel" in k["kernel"]][0]
    sp = [k for k in summarize(split_rep) if "split" in k["kernel"]] if split_rep != "-" else []
    doc = {"source": "%s (ncu --set full --clock-control none, one launch; tools/prof_all.sh)" % label,
           "gemm_kernel": g["kernel"], "gemm_config": cfg, "gemm_shape": shape,
           "gemm_dram_bytes_per_launch": g.get("dram_bytes_total"),
           "gemm_profiled": {k: g.get(k) for k in ("gpu__time_duration.sum", "gpc__cycles_elapsed.avg.per_second",
                                                    "sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
                                                    "lts__t_sector_hit_rate.pct")},
           "split_dram_bytes_per_step": sum(k.get("dram_bytes_total") or 0 for k in sp) if sp else None,
           "split_kernels": [k["kernel"][:60] for k in sp]}
    json.dump(doc, open(out, "w"), indent=1)
    print("wrote", out)


def main():
    args = sys.argv[1:]
    if args and args[0] == "--bench-summary":
        # --bench-summary OUT.json "cg bn sep kc fused" "M N K" gemm.ncu-rep split.ncu-rep|- LABEL
        _, out, cfg, shape, grep, srep, label = args[:7]
        bench_summary(out, [int(v) for v in cfg.split()], [int(v) for v in shape.split()], grep, srep, label)
        return
    prefix = args.pop(0)
    launch, head = None, None
    if "--launch" in args:
        i = args.index("--launch")
        launch = args[i + 1]
        del args[i:i + 2]
    if "--headline" in args:
        i = args.index("--headline")
        head = int(args[i + 1])
        del args[i:i + 2]
    res = {"kernels": []}
    for rep in args:
        res["kernels"] += summarize(rep)
    if launch:
        res["launch_list"] = launch_list(launch)
        if head:
            res["headline_launches"] = launch_list(launch, head)
    json.dump(res, open(prefix + ".json", "w"), indent=1)
    with open(prefix + ".md", "w") as f:
        for s in res["kernels"]:
            f.write("### %s (%s)\n\n| metric | value |\n|---|---|\n" % (s["kernel"], s["report"]))
            for k, v in s.items():
                if k not in ("kernel", "report"):
                    f.write("| %s | %s |\n" % (k, v))
            f.write("\n")
        if launch:
            f.write("### launch list (ncu gpu__time_duration, cold-cache, serialised)\n\n")
            f.write("| kernel | launches | total ms | share |\n|---|---|---|---|\n")
            for r in res["launch_list"]:
                f.write("| %s | %d | %.3f | %.3f |\n" % (r["kernel"], r["launches"], r["total_ms"], r["share"]))
            if head:
                f.write("\n### headline step only (first %d launches: warm-up + timed steps)\n\n" % head)
                f.write("| kernel | launches | total ms | share |\n|---|---|---|---|\n")
                for r in res["headline_launches"]:
                    f.write("| %s | %d | %.3f | %.3f |\n" % (r["kernel"], r["launches"], r["total_ms"],
                                                          r["share"]))
    print("wrote", prefix + ".json", prefix + ".md")


if __name__ == "__main__":
    main()
