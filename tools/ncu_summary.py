#!/usr/bin/env python
"""Summarise `ncu --set full` reports (and a launch list) into profiles/.

    python tools/ncu_summary.py --tag r1 --n 67108864 gpurun_out/prof_*_T4.ncu-rep \
        --launches gpurun_out/launches.csv

Writes profiles/ncu_summary.json (read by bench.py for roofline.traffic) and
profiles/ncu_<tag>.md. Per-object counters divide by --n (objects per launch).
Runs here (no GPU needed): `ncu -i <rep> --page raw --csv`.
"""
import argparse
import csv
import io
import json
import os
import re
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

METRICS = {
    "duration_ns": "gpu__time_duration.sum",
    "dram_read": "dram__bytes_read.sum",
    "dram_write": "dram__bytes_write.sum",
    "dram_pct": "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
    "regs": "launch__registers_per_thread",
    "grid": "launch__grid_size",
    "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active",
    "issue_active_pct": "smsp__issue_active.avg.pct_of_peak_sustained_active",
    "inst": "smsp__inst_executed.sum",
    "simt_eff": "smsp__thread_inst_executed_per_inst_executed.ratio",
    "global_ld": "smsp__sass_inst_executed_op_global_ld.sum",
    "global_st": "smsp__sass_inst_executed_op_global_st.sum",
    "local_ld": "smsp__sass_inst_executed_op_local_ld.sum",
    "local_st": "smsp__sass_inst_executed_op_local_st.sum",
    "branch": "smsp__inst_executed_op_branch.sum",
    "div_targets": "smsp__sass_branch_targets_threads_divergent.sum",
    "uniform_pct": "smsp__sass_average_branch_targets_threads_uniform.pct",
    "l1_hit": "l1tex__t_sector_hit_rate.pct",
    "l2_hit": "lts__t_sector_hit_rate.pct",
    "ld_sectors": "l1tex__t_sectors_pipe_lsu_mem_global_op_ld.sum",
    "stall_long_sb": "smsp__average_warps_issue_stalled_long_scoreboard_per_issue_active.ratio",
    "stall_barrier": "smsp__average_warps_issue_stalled_barrier_per_issue_active.ratio",
    "stall_wait": "smsp__average_warps_issue_stalled_wait_per_issue_active.ratio",
}


def raw(rep):
    if rep.endswith(".csv"):  # a `--page raw --csv` export made on the GPU box
        out = open(rep).read()
    else:
        out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr, units = rows[0], rows[1]
    res = []
    for r in rows[2:]:
        d = {"kernel": r[hdr.index("Kernel Name")]}
        for k, m in METRICS.items():
            if m in hdr:
                i = hdr.index(m)
                v = r[i].replace(",", "")
                try:
                    v = float(v)
                    u = units[i]
                    scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "KB": 1e3, "MB": 1e6,
                             "GB": 1e9, "nsecond": 1, "usecond": 1e3, "msecond": 1e6, "ns": 1, "us": 1e3,
                             "ms": 1e6}
                    if k in ("duration_ns", "dram_read", "dram_write") and u in scale:
                        v *= scale[u]
                except ValueError:
                    pass
                d[k] = v
        res.append(d)
    return res


def sass_counts(so, pattern):
    """CALL / BRX count in the SASS of kernels matching `pattern` (static check)."""
    out = subprocess.run(["cuobjdump", "-sass", so], capture_output=True, text=True).stdout
    res, cur = {}, None
    for line in out.splitlines():
        m = re.search(r"Function : (\S+)", line)
        if m:
            cur = m.group(1) if re.search(pattern, m.group(1)) else None
            if cur:
                res[cur] = {"CALL": 0, "BRX": 0, "UBLKCP": 0}
            continue
        if cur:
            for op in ("CALL", "BRX", "UBLKCP"):
                if re.search(rf"\b{op}\b", line):
                    res[cur][op] += 1
    return res


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("reports", nargs="+")
    ap.add_argument("--tag", default="r1")
    ap.add_argument("--n", type=int, default=1 << 26)
    ap.add_argument("--launches", default=None)
    ap.add_argument("--key-suffix", default="T4_random")
    a = ap.parse_args()
    summ_path = os.path.join(ROOT, "profiles", "ncu_summary.json")
    summ = json.load(open(summ_path)) if os.path.exists(summ_path) else {"kernels": {}}
    md = [f"# ncu summary ({a.tag}) — `ncu --set full --clock-control none`, one launch each, "
          f"n = {a.n} objects, B200\n",
          "Per-object columns divide by n. DRAM bytes are per launch; the algorithmic floor is "
          "16 B/call (SURVEY §8d) and the 16 B-object layout floor 40 B/call.\n",
          "| variant | kernel | µs | DRAM rd+wr GB | B/call | DRAM % | regs | warps act % | SIMT eff | "
          "glob ld/obj | glob st/obj | local ld+st | branches/obj | div. targets | L1 hit % | L2 hit % | "
          "stall long-sb | stall barrier |",
          "|" + "---|" * 18]
    for rep in a.reports:
        variant = os.path.basename(rep).split("_")[1]  # prof_<variant>_T4[.ncu-rep|.raw.csv]
        for d in raw(rep):
            n = a.n
            traffic = d.get("dram_read", 0) + d.get("dram_write", 0)
            key = f"micro_{variant}_{a.key_suffix}"
            summ["kernels"][key] = {"kernel": d["kernel"], "dram_bytes_per_launch": traffic,
                                    "duration_ns": d.get("duration_ns"), "source": os.path.basename(rep),
                                    "round": a.tag, **{k: v for k, v in d.items() if k != "kernel"}}
            f = lambda k, s=1.0, fmt="{:.2f}": fmt.format(d[k] / s) if isinstance(d.get(k), float) else "—"
            md.append(f"| {variant} | `{d['kernel'][:60]}` | {f('duration_ns', 1e3, '{:.1f}')} | "
                      f"{traffic / 1e9:.3f} | {traffic / n:.1f} | {f('dram_pct', 1, '{:.1f}')} | {f('regs', 1, '{:.0f}')} | "
                      f"{f('warps_active_pct', 1, '{:.1f}')} | {f('simt_eff', 1, '{:.1f}')} | {f('global_ld', n / 32, '{:.2f}')} | "
                      f"{f('global_st', n / 32, '{:.2f}')} | {f('local_ld', 1, '{:.0f}')}+{f('local_st', 1, '{:.0f}')} | "
                      f"{f('branch', n / 32, '{:.2f}')} | {f('div_targets', 1, '{:.0f}')} | {f('l1_hit', 1, '{:.1f}')} | "
                      f"{f('l2_hit', 1, '{:.1f}')} | {f('stall_long_sb')} | {f('stall_barrier')} |")
    md.append("\n`glob ld/obj` counts warp-level SASS global-load instructions × 32 / n, i.e. per-object "
              "load instructions issued. The embedded-vTable path (sharedoa) issues its vTable* load (A) and "
              "vFunc* slot load (B) per object; the COAL/TypePointer kernels issue only the pointer, the "
              "object warm-up and the body's own field load.\n")
    so = os.path.join(ROOT, "paper_conf_asplos_zhangar21_b200", "libvf.so")
    if os.path.exists(so):
        sc = sass_counts(so, r"k_dispatch_(sorted|grouped|virtual)INS_5micro3AppELi0E")
        md.append("## Static SASS check (cuobjdump -sass libvf.so, micro kernels)\n")
        md.append("| kernel | CALL | BRX | UBLKCP |\n|---|---|---|---|")
        for k, v in sorted(sc.items()):
            md.append(f"| `{k[:90]}` | {v['CALL']} | {v['BRX']} | {v['UBLKCP']} |")
        summ["sass"] = {k: v for k, v in sc.items()}
    if a.launches and os.path.exists(a.launches):
        rows = [r for r in csv.reader(l for l in open(a.launches) if l.startswith('"'))]
        hdr = rows[0]
        ki, vi = hdr.index("Kernel Name"), hdr.index("Metric Value")
        tot = {}
        for r in rows[1:]:
            tot.setdefault(r[ki].split("(")[0], []).append(float(r[vi]))
        allt = sum(sum(v) for v in tot.values())
        md.append("\n## Launch list of the bench command (ncu gpu__time_duration, cold-cache, serialised)\n")
        md.append("| kernel | launches | mean µs | share of all |\n|---|---|---|---|")
        for k, v in sorted(tot.items(), key=lambda kv: -sum(kv[1])):
            md.append(f"| `{k[:80]}` | {len(v)} | {sum(v) / len(v) / 1e3:.1f} | {sum(v) / allt:.1%} |")
        summ["launch_list"] = {k: {"launches": len(v), "mean_ns": sum(v) / len(v)} for k, v in tot.items()}
    os.makedirs(os.path.join(ROOT, "profiles"), exist_ok=True)
    json.dump(summ, open(summ_path, "w"), indent=1)
    open(os.path.join(ROOT, "profiles", f"ncu_{a.tag}.md"), "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
