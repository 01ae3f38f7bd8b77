"""Copy one evidence run (tools/round_evidence.sh output dir) into profiles/ (tracked).

    python tools/collect_evidence.py /path/to/gpurun_out [--round r01]

Writes profiles/<round>_bench_c2.json, _bench_reference_c2.json, _bench_allconfigs.jsonl,
_ncu_summary.md (table of the dominant kernel per config from the --set full captures),
ncu_traffic.json (dram read+write per launch, read by bench.py), _launches_c2_bench.csv +
summary, _pytest_gpu.txt, _sanitize_*.txt, _cta_trace.txt, _ncu_raw_<cfg>.csv.
"""
import csv
import glob
import json
import os
import shutil
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
PROF = os.path.join(ROOT, "profiles")
CFG_N = {"c2": 128, "c3": 256, "c3h": 256, "c4": 128, "c5": 512}


def last_json(path):
    with open(path) as f:
        lines = [x for x in f.read().strip().splitlines() if x.startswith("{")]
    return json.loads(lines[-1]) if lines else None


def raw_metrics(path):
    rows = list(csv.reader(open(path)))
    hdr, units = rows[0], rows[1]
    out = []
    for vals in rows[2:]:
        out.append({h: (vals[i], units[i]) for i, h in enumerate(hdr)})
    return out


def num(d, k):
    v = d.get(k, ("nan", ""))[0].replace(",", "")
    try:
        return float(v)
    except ValueError:
        return float("nan")


def to_bytes(d, k):
    v, u = d.get(k, ("nan", ""))
    v = float(v.replace(",", ""))
    return v * {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)


def to_us(d, k):
    v, u = d.get(k, ("nan", ""))
    v = float(v.replace(",", ""))
    return v * {"ns": 1e-3, "us": 1.0, "usecond": 1.0, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3}.get(u, 1)


def main():
    src = sys.argv[1]
    rnd = sys.argv[sys.argv.index("--round") + 1] if "--round" in sys.argv else "r01"
    p = lambda name: os.path.join(PROF, f"{rnd}_{name}")
    # bench lines
    if os.path.exists(os.path.join(src, "ev_bench_default.json")):
        shutil.copy(os.path.join(src, "ev_bench_default.json"), p("bench_c2.json"))
    if os.path.exists(os.path.join(src, "ev_bench_reference.json")):
        shutil.copy(os.path.join(src, "ev_bench_reference.json"), p("bench_reference_c2.json"))
    lines = []
    for c in ("default", "c3", "c3h", "c4", "c5"):
        f = os.path.join(src, f"ev_bench_{c}.json")
        if os.path.exists(f) and last_json(f):
            lines.append(json.dumps(last_json(f)))
    if lines:
        open(p("bench_allconfigs.jsonl"), "w").write("\n".join(lines) + "\n")
    # ncu --set full summaries
    rows, traffic = [], {"_source": f"dram__bytes_read.sum + dram__bytes_write.sum per launch of the dominant "
                                    f"SpMM kernel, ncu --set full (profiles/{rnd}_ncu_summary.md)"}
    for c in CFG_N:
        f = os.path.join(src, f"ev_raw_{c}.csv")
        if not os.path.exists(f):
            continue
        shutil.copy(f, p(f"ncu_raw_{c}.csv"))
        for d in raw_metrics(f):
            name = d.get("Kernel Name", ("?", ""))[0]
            rd, wr = to_bytes(d, "dram__bytes_read.sum"), to_bytes(d, "dram__bytes_write.sum")
            dur = to_us(d, "gpu__time_duration.sum")
            stalls = sorted(((num(d, h), h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")])
                             for h in d if h.startswith("smsp__average_warps_issue_stalled_")
                             and h.endswith("_per_issue_active.ratio")), reverse=True)[:3]
            rows.append((c, CFG_N[c], name.split("(")[0].replace("void ", ""), int(num(d, "launch__registers_per_thread")),
                         num(d, "sm__warps_active.avg.per_cycle_active"), dur, rd / 1e9, wr / 1e9,
                         (rd + wr) / (dur * 1e-6) / 1e9, num(d, "lts__t_sector_hit_rate.pct"),
                         num(d, "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active"),
                         num(d, "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum"),
                         num(d, "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"),
                         ", ".join(f"{n} {v:.2f}" for v, n in stalls)))
            traffic[f"{c}_N{CFG_N[c]}"] = int(rd + wr)
    if rows:
        md = [f"# {rnd} -- ncu --set full of the dominant kernel, one launch per config", "",
              "`ncu --set full --clock-control none --import-source on -k regex:k_spmm -s 3 -c 1` on "
              "`python bench.py --config <c> --steps 3 --warmup 3 --minimal` (tools/round_evidence.sh).  Times under "
              "ncu are cold-cache and serialised: rates come from bench.py; these give traffic, hit rates, "
              "occupancy and stalls.  Raw pages: `" + rnd + "_ncu_raw_<cfg>.csv`.", "",
              "| config | N | kernel | regs | warps/SM | duration us | DRAM read GB | DRAM write GB | DRAM GB/s | "
              "L2 hit % | tensor pipe % | smem bank conflicts / wavefronts | top stalls (per issue) |",
              "|---|---|---|---|---|---|---|---|---|---|---|---|---|"]
        for r in rows:
            md.append(f"| {r[0]} | {r[1]} | `{r[2]}` | {r[3]} | {r[4]:.1f} | {r[5]:.1f} | {r[6]:.3f} | {r[7]:.3f} | "
                      f"{r[8]:.0f} | {r[9]:.1f} | {r[10]:.1f} | {r[11]:.0f} / {r[12]:.0f} | {r[13]} |")
        open(p("ncu_summary.md"), "w").write("\n".join(md) + "\n")
        json.dump(traffic, open(os.path.join(PROF, "ncu_traffic.json"), "w"), indent=1)
    # launch list
    f = os.path.join(src, "ev_launches_c2.csv")
    if os.path.exists(f):
        shutil.copy(f, p("launches_c2_bench.csv"))
        out = subprocess.run([sys.executable, os.path.join(ROOT, "tools", "launch_share.py"), f],
                             capture_output=True, text=True).stdout
        open(p("launches_c2_bench_summary.txt"), "w").write(out)
    # logs
    for name, dst in (("ev_pytest_gpu.log", "pytest_gpu.txt"), ("ev_sanitize_memcheck.log", "sanitize_memcheck.txt"),
                      ("ev_sanitize_racecheck.log", "sanitize_racecheck.txt"),
                      ("ev_sanitize_synccheck.log", "sanitize_synccheck.txt")):
        f = os.path.join(src, name)
        if os.path.exists(f):
            txt = open(f).read().splitlines()
            open(p(dst), "w").write("\n".join(txt[-40:]) + "\n")
    tr = []
    for c in CFG_N:
        f = os.path.join(src, f"ev_trace_{c}.txt")
        if os.path.exists(f):
            tr.append(open(f).read().strip())
    if tr:
        open(p("cta_trace.txt"), "w").write("\n\n".join(tr) + "\n")
    print("\n".join(sorted(glob.glob(os.path.join(PROF, f"{rnd}_*")))))


if __name__ == "__main__":
    main()
