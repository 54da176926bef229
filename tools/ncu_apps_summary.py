#!/usr/bin/env python
"""Summarise `ncu --set full` raw-page CSV exports of app kernels into a table.

    python tools/ncu_apps_summary.py --title "graph kernels (RMAT-24, typeptr)" \
        --out profiles/ncu_graph_r1.md gpurun_out/prof_graph-*.raw.csv

(The GPU box exports `ncu -i rep --page raw --csv`; reports themselves are too
large to bring back.)
"""
import argparse
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))
from ncu_summary import raw  # noqa: E402

COLS = [("duration_ns", "µs", 1e3, "{:.1f}"), ("dram_gbs", "DRAM GB/s", 1, "{:.0f}"), ("dram_pct", "DRAM %", 1, "{:.1f}"),
        ("global_ld", "global ld insts", 1, "{:.3g}"), ("branch", "branch insts", 1, "{:.3g}"),
        ("div_targets", "divergent branch targets", 1, "{:.3g}"), ("uniform_pct", "uniform branch %", 1, "{:.1f}"),
        ("regs", "regs", 1, "{:.0f}"), ("warps_active_pct", "warps act %", 1, "{:.1f}"),
        ("simt_eff", "SIMT eff (thr/inst)", 1, "{:.1f}"), ("issue_active_pct", "issue act %", 1, "{:.1f}"),
        ("l1_hit", "L1 hit %", 1, "{:.1f}"), ("l2_hit", "L2 hit %", 1, "{:.1f}"),
        ("stall_long_sb", "stall long-sb", 1, "{:.2f}")]


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("csvs", nargs="+")
    ap.add_argument("--out", required=True)
    ap.add_argument("--title", default="app kernels")
    a = ap.parse_args()
    md = [f"# ncu summary — {a.title}\n",
          "`ncu --set full --clock-control none`, one launch per kernel (cold cache, serialised: "
          "compare shares and counters, not absolute step times).\n",
          "| capture | kernel | DRAM rd+wr GB | " + " | ".join(c[1] for c in COLS) + " |",
          "|" + "---|" * (3 + len(COLS))]
    for path in a.csvs:
        name = os.path.basename(path).replace(".raw.csv", "")
        for d in raw(path):
            traffic = d.get("dram_read", 0) + d.get("dram_write", 0)
            if isinstance(d.get("duration_ns"), float) and d["duration_ns"] > 0:
                d["dram_gbs"] = traffic / d["duration_ns"]
            cells = []
            for k, _, s, fmt in COLS:
                v = d.get(k)
                cells.append(fmt.format(v / s) if isinstance(v, float) else "—")
            md.append(f"| {name} | `{d['kernel'][:70]}` | {traffic / 1e9:.3f} | " + " | ".join(cells) + " |")
    open(a.out, "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
