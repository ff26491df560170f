"""Summarise .ncu-rep files: per kernel launch, the metrics the roofline and
the RMT cost attribution need.  usage: ncu_summary.py FILE.ncu-rep ... [--json OUT]"""
import csv, io, json, subprocess, sys

KEYS = {
    "time_us": ("gpu__time_duration.sum", 1e-3),
    "dram_read_MB": ("dram__bytes_read.sum", None),
    "dram_write_MB": ("dram__bytes_write.sum", None),
    "dram_pct": ("dram__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "lts_pct": ("lts__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "l1tex_pct": ("l1tex__throughput.avg.pct_of_peak_sustained_active", 1),
    "sm_pct": ("sm__throughput.avg.pct_of_peak_sustained_elapsed", 1),
    "issue_pct": ("smsp__issue_active.avg.pct_of_peak_sustained_active", 1),
    "warps_active_pct": ("sm__warps_active.avg.pct_of_peak_sustained_active", 1),
    "regs": ("launch__registers_per_thread", 1),
    "block": ("launch__block_size", 1),
    "grid": ("launch__grid_size", 1),
    "smem_ld_conflicts": ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_ld.sum", 1),
    "smem_st_conflicts": ("l1tex__data_bank_conflicts_pipe_lsu_mem_shared_op_st.sum", 1),
    "inst_executed": ("smsp__inst_executed.sum", 1),
    "alu_pct": ("sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active", 1),
    "fma_pct": ("sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", 1),
    "lsu_pct": ("sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", 1),
}
STALLS = ["long_scoreboard", "short_scoreboard", "barrier", "lg_throttle", "mio_throttle", "membar", "wait",
          "math_pipe_throttle", "not_selected", "selected", "branch_resolving", "sleeping", "drain", "tex_throttle",
          "no_instruction", "dispatch_stall", "misc"]


def to_float(s):
    try:
        return float(s.replace(",", ""))
    except Exception:
        return None


def summarize(path):
    raw = subprocess.run(["ncu", "-i", path, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(raw)))
    hdr, units, data = rows[0], rows[1], rows[2:]
    col = {h: i for i, h in enumerate(hdr)}
    out = []
    for r in data:
        d = {"name": r[col["Kernel Name"]][:60]}
        for k, (m, scale) in KEYS.items():
            if m not in col:
                continue
            v = to_float(r[col[m]])
            if v is None:
                continue
            u = units[col[m]]
            if k.endswith("_MB"):
                mult = {"byte": 1e-6, "Kbyte": 1e-3, "Mbyte": 1.0, "Gbyte": 1e3}.get(u, 1.0)
                v = v * mult
            elif k == "time_us":
                v = v * {"nsecond": 1e-3, "ns": 1e-3, "usecond": 1.0, "us": 1.0, "msecond": 1e3, "ms": 1e3}.get(u, 1.0)
            d[k] = round(v, 3)
        st = {}
        for s in STALLS:
            m = f"smsp__average_warps_issue_stalled_{s}_per_issue_active.ratio"
            if m in col:
                v = to_float(r[col[m]])
                if v:
                    st[s] = round(v, 2)
        d["stalls_top"] = dict(sorted(st.items(), key=lambda kv: -kv[1])[:5])
        out.append(d)
    return out


if __name__ == "__main__":
    args = sys.argv[1:]
    jout = None
    if "--json" in args:
        i = args.index("--json")
        jout = args[i + 1]
        args = args[:i] + args[i + 2:]
    res = {}
    for p in args:
        res[p.split("/")[-1].replace(".ncu-rep", "")] = summarize(p)
    for k, v in res.items():
        for d in v:
            print(k, json.dumps(d))
    if jout:
        json.dump(res, open(jout, "w"), indent=1)
