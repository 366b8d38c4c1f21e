"""Summarise ncu captures into profiles/ (run here, no GPU needed).

  python tools/ncu_summary.py full   gpurun_out/p2p_full_r1.ncu-rep  profiles/r1_p2p_kernel_ncu.txt [--traffic C2 128]
  python tools/ncu_summary.py launches gpurun_out/launches_r1.csv   profiles/r1_launches.txt
"""
import csv
import io
import json
import os
import subprocess
import sys
from collections import defaultdict

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

KEYS = [
    "gpu__time_duration.sum", "sm__cycles_elapsed.avg.per_second", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
    "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fmaheavy_cycles_active.avg.pct_of_peak_sustained_elapsed",
    "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
    "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
    "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_fp64_cycles_active.avg.pct_of_peak_sustained_active",
    "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
    "smsp__issue_active.avg.pct_of_peak_sustained_active", "sm__warps_active.avg.pct_of_peak_sustained_active",
    "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum.pct_of_peak_sustained_elapsed",
    "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum", "launch__registers_per_thread",
    "launch__grid_size", "launch__block_size", "smsp__inst_executed.sum",
]


def raw(rep):
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    return rows[0], rows[1], rows[2:]


def full(rep, dst, traffic=None):
    hdr, units, data = raw(rep)
    lines = [f"# ncu --set full summary of {os.path.basename(rep)}"]
    for d in data:
        kv = dict(zip(hdr, d))
        lines.append(f"kernel: {kv.get('Kernel Name')}")
        for k in KEYS:
            if k in kv:
                lines.append(f"  {k:75s} {kv[k]} {units[hdr.index(k)]}")
        stalls = []
        for i, h in enumerate(hdr):
            if h.startswith("smsp__average_warps_issue_stalled_") and h.endswith("_per_issue_active.ratio"):
                try:
                    stalls.append((float(d[i]), h[len("smsp__average_warps_issue_stalled_"):-len("_per_issue_active.ratio")]))
                except ValueError:
                    pass
        stalls.sort(reverse=True)
        lines.append("  stall reasons (warp-cycles per issued instruction):")
        for v, nm in stalls[:10]:
            lines.append(f"    {nm:30s} {v:.3f}")
        if traffic:
            def num(k):
                v = float(kv[k])
                u = units[hdr.index(k)].lower()
                return v * {"byte": 1, "kbyte": 1e3, "mbyte": 1e6, "gbyte": 1e9}.get(u, 1)
            tb = num("dram__bytes_read.sum") + num("dram__bytes_write.sum")
            with open(os.path.join(ROOT, "profiles", "traffic.json"), "w") as f:
                json.dump({"config": traffic[0], "S": int(traffic[1]), "dram_bytes_per_launch": tb,
                           "source": os.path.basename(dst)}, f)
            lines.append(f"  dram bytes per launch (read+write): {tb:.4g}")
    open(dst, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


def launches(src, dst):
    txt = open(src).read()
    i = txt.find('"ID"')
    rows = list(csv.DictReader(io.StringIO(txt[i:])))
    tot = defaultdict(float)
    cnt = defaultdict(int)
    order = []
    for r in rows:
        if r.get("Metric Name") != "gpu__time_duration.sum":
            continue
        nm = r["Kernel Name"].split("(")[0]
        if nm not in cnt:
            order.append(nm)
        v = float(r["Metric Value"])
        unit = r["Metric Unit"]
        v *= {"ns": 1e-3, "us": 1, "usecond": 1, "ms": 1e3, "msecond": 1e3, "nsecond": 1e-3}.get(unit, 1)
        tot[nm] += v
        cnt[nm] += 1
    allt = sum(tot.values())
    lines = [f"# ncu launch list ({os.path.basename(src)}): gpu__time_duration.sum, --clock-control none",
             "# cold-cache, serialised per launch: compare SHARES, not absolutes",
             f"{'kernel':60s} {'launches':>8s} {'total_us':>12s} {'mean_us':>10s} {'share':>7s}"]
    for nm in sorted(order, key=lambda k: -tot[k]):
        lines.append(f"{nm[:60]:60s} {cnt[nm]:8d} {tot[nm]:12.1f} {tot[nm] / cnt[nm]:10.2f} {tot[nm] / allt:7.1%}")
    open(dst, "w").write("\n".join(lines) + "\n")
    print("\n".join(lines))


if __name__ == "__main__":
    mode, src, dst = sys.argv[1:4]
    if mode == "full":
        tr = sys.argv[5:7] if len(sys.argv) > 5 and sys.argv[4] == "--traffic" else None
        full(src, dst, tr)
    else:
        launches(src, dst)
