#!/usr/bin/env python
"""Render the `apps` block (and the config-2 variants) of a bench.py JSON line as
a markdown table for profiles/.

    python tools/apps_table.py gpurun_out/bench.json --out profiles/apps_r2.md
"""
import argparse
import json


def fmt(x, f="{:.3g}"):
    return "—" if x is None else f.format(x)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("bench_json")
    ap.add_argument("--out", required=True)
    ap.add_argument("--title", default="per-app block of bench.py (BASELINE configs 1, 3, 4, 5)")
    a = ap.parse_args()
    line = [l for l in open(a.bench_json).read().splitlines() if l.startswith("{")][-1]
    d = json.loads(line)
    md = [f"# {a.title}\n",
          f"One B200, `python bench.py` (driver contract run), {d.get('n_gpus')} GPU(s). "
          "Time = CUDA events around the step loop after warm-up, per-app clocks sampled during the "
          "app's runs. speedup = t_cuda / t_variant on the same config (device-heap CUDA arm).\n"]
    v = d.get("variants") or {}
    if v:
        md.append("## Config 2 (dispatch microbenchmark)\n")
        md.append(f"headline: {d['value'] / 1e9:.2f} Gcalls/s ({d['config']['variant']}, n = {d['config']['n']}, "
                  f"T = {d['config']['T']}, {d['config']['order']}); roofline frac {d['roofline']['frac']:.3f} "
                  f"(16 B/call algorithmic), {d['roofline'].get('layout_floor_frac', 0):.3f} of the 40 B/call "
                  f"layout floor; clocks {d.get('clocks')}\n")
        md.append("| variant | n | Gcalls/s |\n|---|---|---|")
        for k in ("cuda_packed", "sharedoa", "coal", "typeptr"):
            if k in v:
                md.append(f"| {k} | {v[k]['n']} | {v[k]['calls_per_s'] / 1e9:.2f} |")
        at = v.get("at_cuda_n")
        if at:
            md.append(f"\nSame config with the device-heap CUDA arm (n = {at['n']}, {at.get('l2')}):\n")
            md.append("| variant | Gcalls/s | speedup vs cuda |\n|---|---|---|")
            for k, s in at["speedup_vs_cuda"].items():
                md.append(f"| {k} | {at[k] / 1e9:.2f} | {s:.2f} |")
    apps = d.get("apps") or {}
    md.append("\n## Per-app (BASELINE sizes)\n")
    md.append("| app | config | variant | ms/step | Gcalls/s | speedup vs cuda | roofline (best variant) | "
              "oracle on host |")
    md.append("|---|---|---|---|---|---|---|---|")
    for name, row in apps.items():
        sp = row.get("speedup_vs_cuda", {})
        rf = row.get("roofline", {})
        cpu = row.get("cpu_baseline")
        first = True
        for var, x in row["variants"].items():
            md.append(f"| {name if first else ''} | {row['config'][:90] if first else ''} | {var} | "
                      f"{x['ms_per_step']:.4g} | {x['calls_per_s'] / 1e9:.4g} | {fmt(sp.get(var), '{:.2f}')} | "
                      + (f"{rf.get('frac', 0):.3f} of {rf.get('peak', 0):.0f} {rf.get('unit', '')} ({rf.get('bound')})"
                         if first else "")
                      + " | " + (f"{cpu['value'] / 1e9:.3g} Gcalls/s ({cpu['cores']} cores; {cpu['sample']})"
                                 if (first and cpu) else "") + " |")
            first = False
        for sub in ("bfs", "cc", "pr"):
            if sub in row:
                s = row[sub]
                md.append(f"| | {name}-{sub} | " + ", ".join(
                    f"{k} {x['ms_per_step']:.3g} ms" for k, x in s["variants"].items()) + " | | | " +
                    ", ".join(f"{k} {v_:.2f}" for k, v_ in s.get("speedup_vs_cuda", {}).items()) + " | | |")
        if "same_config_with_heap_cuda" in row:
            s = row["same_config_with_heap_cuda"]
            md.append(f"| | {s['config'][:90]} | " + ", ".join(
                f"{k} {x['ms_per_step']:.3g} ms" for k, x in s["variants"].items()) + " | | | " +
                ", ".join(f"{k} {v_:.2f}" for k, v_ in s.get("speedup_vs_cuda", {}).items()) + " | | |")
        md.append(f"| | clocks: {row.get('clocks')}; variants agree: {row.get('variants_agree')} | | | | | | |")
    open(a.out, "w").write("\n".join(md) + "\n")
    print("\n".join(md))


if __name__ == "__main__":
    main()
